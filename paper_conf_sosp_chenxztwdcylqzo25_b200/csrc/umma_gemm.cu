// umma_gemm.cu -- persistent grouped expert GEMM on the 5th-gen tensor cores.
//
//   routed:  C[rows of expert e] = A[rows of expert e] . B_e^T
//   shared:  C[token rows]       = A[token rows] . B_s^T
//
// GEMM1 (EPI_SWIGLU): A = x_perm (tokens sorted by expert), B = W13 with rows
// interleaved per 128 (W1 block b, W3 block b), so one 256-wide N tile holds
// matching gate/up columns and the epilogue computes h = silu(g) * u from the
// fp32 accumulators -- the fused gate+up batch of PAPER.md L179.  FP8: h is
// requantised to e4m3 with a 1x128 UE8M0 scale straight from fp32 (DESIGN.md
// reading R11), written together with the scale image GEMM2 consumes.
// GEMM2 (EPI_PLAIN):  A = h, B = W2 -> bf16 rows.
//
// Work units = (expert m-tile of 128 rows, 256-wide n-block), ordered expert-
// major then n-block then m-tile so CTAs running concurrently share one weight
// slab through L2 (the device-side analog of PAPER.md L181's co-scheduling of
// same-expert tasks).  Roles per CTA (320 threads, one CTA per SM):
//   warp 0     TMA producer (A/B tiles, FP8 scale images) into a 4-stage ring
//   warp 1     TMEM allocator + single-thread tcgen05.mma issuer
//   warps 2-9  epilogue: tcgen05.ld -> registers (TMEM released) -> math -> global
#include <cuda.h>

#include "common.cuh"
#include "kernels.h"
#include "sm100.cuh"

namespace moe {
using namespace sm100;

constexpr int UG_BM = 128, UG_BN = 256, UG_STAGES = 4, UG_THREADS = 320;
constexpr int UG_A_BYTES = UG_BM * 128;        // 16 KB (128 rows x 128 B)
constexpr int UG_B_BYTES = UG_BN * 128;        // 32 KB
constexpr int UG_SFA_BYTES = 512;              // 128 rows x 4 B image
constexpr int UG_SFB_BYTES = 1024;             // 256 rows x 4 B image
constexpr uint32_t UG_TMEM_COLS = 512;
constexpr uint32_t UG_SFA_COL = 256, UG_SFB_COL = 264;
constexpr int UG_UQ = 4;                       // depth of the in-CTA work-unit queue
constexpr size_t UG_SMEM = 1024 + (size_t)UG_STAGES * (UG_A_BYTES + UG_B_BYTES + UG_SFA_BYTES + UG_SFB_BYTES) + 512 + 2048;

struct UnitInfo {
  int valid, group, expert, row0, row_end, nb;
};

__device__ __forceinline__ UnitInfo decode_unit(const UmmaParams &p, int u, int n_routed_units) {
  UnitInfo r{};
  if (u < n_routed_units) {
    const int nb_r = p.nb_r;
    const int4 t_any = p.tiles[u / nb_r];
    const int t0 = t_any.w & 0xFFFF, nt = t_any.w >> 16;
    const int local = u - t0 * nb_r;
    const int4 tl = p.tiles[t0 + local % nt];
    r.valid = 1; r.group = 0; r.expert = tl.x; r.row0 = tl.y; r.row_end = tl.z; r.nb = local / nt;
    return r;
  }
  const int us = u - n_routed_units;
  const int mt = (p.T_shared + UG_BM - 1) / UG_BM;
  if (p.T_shared > 0 && us < mt * p.nb_s) {
    r.valid = 1; r.group = 1; r.expert = 0; r.nb = us / mt;
    r.row0 = (us % mt) * UG_BM; r.row_end = p.T_shared;
  }
  return r;
}

template <bool FP8, int EPI>
__global__ void __launch_bounds__(UG_THREADS, 1) umma_grouped_gemm(const __grid_constant__ UmmaParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t *sA = smem;
  uint8_t *sB = sA + UG_STAGES * UG_A_BYTES;
  uint8_t *sSFA = sB + UG_STAGES * UG_B_BYTES;
  uint8_t *sSFB = sSFA + UG_STAGES * UG_SFA_BYTES;
  uint64_t *full = reinterpret_cast<uint64_t *>(sSFB + UG_STAGES * UG_SFB_BYTES);
  uint64_t *empty = full + UG_STAGES;
  uint64_t *tmem_full = empty + UG_STAGES;
  uint64_t *tmem_empty = tmem_full + 1;
  uint64_t *uq_full = tmem_empty + 1;
  uint64_t *uq_empty = uq_full + UG_UQ;
  uint32_t *tmem_base_smem = reinterpret_cast<uint32_t *>(uq_empty + UG_UQ);
  int *unit_q = reinterpret_cast<int *>(tmem_base_smem + 4);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n_routed_units = p.tiles ? (*p.n_tiles) * p.nb_r : 0;

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&p.g[0].a_map); prefetch_tmap(&p.g[1].a_map);
    if (EPI == GEMM_LOGITS) prefetch_tmap(&p.g[0].b_map);
    for (int s = 0; s < UG_STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    mbar_init(tmem_full, 1);
    mbar_init(tmem_empty, 8);
    for (int i = 0; i < UG_UQ; ++i) { mbar_init(&uq_full[i], 1); mbar_init(&uq_empty[i], 9); }
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc(tmem_base_smem, UG_TMEM_COLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_base_smem;

  if (warp == 0) {
    // ============================ TMA producer ============================
    if (lane == 0) {
      int stage = 0; uint32_t phase = 0;
      int qs = 0; uint32_t qph = 0;
      for (;;) {
        // dynamic tile scheduler (PAPER.md L181 analog): units are claimed in
        // index order by whichever CTA is free, so CTAs sharing an expert's
        // weight slab run at the same time and reuse it through L2
        const int u = atomicAdd(p.sched, 1);
        mbar_wait(&uq_empty[qs], qph ^ 1);
        unit_q[qs] = u;
        mbar_arrive(&uq_full[qs]);
        if (++qs == UG_UQ) { qs = 0; qph ^= 1; }
        const UnitInfo ui = decode_unit(p, u, n_routed_units);
        if (!ui.valid) break;
        const UmmaGroup &g = p.g[ui.group];
        const int brow = ui.expert * g.n_total + ui.nb * UG_BN;
        const uint8_t *btiles = g.b_tiles + ((size_t)ui.expert * g.b_ntiles_n + ui.nb) * g.kblocks * UG_B_BYTES;
        if (EPI != GEMM_LOGITS)
          for (int kb = 0; kb < p.pf_dist && kb < g.kblocks; ++kb) bulk_prefetch_l2(btiles + (size_t)kb * UG_B_BYTES, UG_B_BYTES);
        for (int kb = 0; kb < g.kblocks; ++kb) {
          if (EPI != GEMM_LOGITS && p.pf_dist > 0 && kb + p.pf_dist < g.kblocks)
            bulk_prefetch_l2(btiles + (size_t)(kb + p.pf_dist) * UG_B_BYTES, UG_B_BYTES);
          mbar_wait(&empty[stage], phase ^ 1);
          if (p.debug_mode == 3 || p.debug_mode == 4) {   // timing experiment: MMAs on stale smem, no loads
            mbar_arrive(&full[stage]);
            if (++stage == UG_STAGES) { stage = 0; phase ^= 1; }
            continue;
          }
          uint32_t bytes = UG_A_BYTES + UG_B_BYTES;
          if (FP8) bytes += UG_SFA_BYTES + UG_SFB_BYTES;
          mbar_expect_tx(&full[stage], bytes);
          const int kc = kb * (FP8 ? 128 : 64);   // element coordinate along K
          tma_load_2d(sA + stage * UG_A_BYTES, &g.a_map, &full[stage], kc, ui.row0);
          if (EPI == GEMM_LOGITS) {
            tma_load_2d(sB + stage * UG_B_BYTES, &g.b_map, &full[stage], kc, brow);
          } else {
            // pre-tiled weights: one contiguous 32 KB read per k-block (L157 load-time layout)
            const uint8_t *bt = g.b_tiles + (((size_t)ui.expert * g.b_ntiles_n + ui.nb) * g.kblocks + kb) * UG_B_BYTES;
            bulk_load(sB + stage * UG_B_BYTES, bt, UG_B_BYTES, &full[stage]);
          }
          if (FP8) {
            const uint8_t *sfa = g.sfa + ((size_t)(kb >> 2) * g.sfa_tile_stride + (ui.row0 >> 7)) * 512;
            const uint8_t *sfb = g.sfb + (size_t)ui.expert * g.sfb_expert_stride +
                                 ((size_t)(kb >> 2) * g.sfb_rb + ui.nb * 2) * 512;
            bulk_load(sSFA + stage * UG_SFA_BYTES, sfa, UG_SFA_BYTES, &full[stage]);
            bulk_load(sSFB + stage * UG_SFB_BYTES, sfb, UG_SFB_BYTES, &full[stage]);
          }
          if (++stage == UG_STAGES) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ============================ MMA issuer ============================
    int stage = 0; uint32_t phase = 0; uint32_t acc_phase = 0;
    int qs = 0; uint32_t qph = 0;
    for (;;) {
      mbar_wait(&uq_full[qs], qph);
      const int u = unit_q[qs];
      __syncwarp();
      if (lane == 0) mbar_arrive(&uq_empty[qs]);
      if (++qs == UG_UQ) { qs = 0; qph ^= 1; }
      const UnitInfo ui = decode_unit(p, u, n_routed_units);
      if (!ui.valid) break;
      const int kblocks = p.g[ui.group].kblocks;
      mbar_wait(tmem_empty, acc_phase ^ 1);
      tc_fence_after();
      for (int kb = 0; kb < kblocks; ++kb) {
        mbar_wait(&full[stage], phase);
        tc_fence_after();
        if (lane == 0 && p.debug_mode != 1) {
          const uint32_t a0 = smem_u32(sA + stage * UG_A_BYTES);
          const uint32_t b0 = smem_u32(sB + stage * UG_B_BYTES);
          // a scale image holds 4 k-blocks (one UE8M0 byte each, selected by the
          // instruction descriptor's sf id): copy it to TMEM once per 4 k-blocks,
          // alternating between two column sets so the copy never targets
          // columns the previous group's MMAs still read
          const uint32_t sf_set = FP8 ? ((kb >> 2) & 1) * 16 : 0;
          const bool do_cp = FP8 && p.debug_mode != 4 && p.debug_mode != 6 && ((kb & 3) == 0 || p.debug_mode == 7);
          if (do_cp) {
            tmem_cp_32x128b_x4(tmem + UG_SFA_COL + sf_set, sf_desc(smem_u32(sSFA + stage * UG_SFA_BYTES)));
            tmem_cp_32x128b_x4(tmem + UG_SFB_COL + sf_set, sf_desc(smem_u32(sSFB + stage * UG_SFB_BYTES)));
            tmem_cp_32x128b_x4(tmem + UG_SFB_COL + sf_set + 4, sf_desc(smem_u32(sSFB + stage * UG_SFB_BYTES + 512)));
          }
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const uint64_t ad = sw128_kmajor_desc(a0 + k * 32);
            const uint64_t bd = sw128_kmajor_desc(b0 + k * 32);
            const uint32_t acc = (kb | k) != 0;
            if (FP8)
              mma_mxf8(tmem, ad, bd, idesc_mxf8(UG_BM, UG_BN, kb & 3, kb & 3), acc, tmem + UG_SFA_COL + sf_set,
                       tmem + UG_SFB_COL + sf_set);
            else
              mma_bf16(tmem, ad, bd, idesc_bf16(UG_BM, UG_BN), acc);
          }
          mma_commit(&empty[stage]);
          if (kb == kblocks - 1) mma_commit(tmem_full);
        } else if (lane == 0) {            // debug_mode 1: load pipeline only
          mbar_arrive(&empty[stage]);
          if (kb == kblocks - 1) mbar_arrive(tmem_full);
        }
        __syncwarp();
        if (++stage == UG_STAGES) { stage = 0; phase ^= 1; }
      }
      acc_phase ^= 1;
    }
  } else {
    // ============================ epilogue ============================
    // 8 warps: two per TMEM lane quadrant, each owning half of the columns.
    // Each thread pulls its accumulator columns into registers, releases TMEM
    // at once (so the next unit's MMAs overlap the math), then computes.
    const int ew = warp - 2;                      // 0..7
    const int q = warp & 3;                       // TMEM lane quadrant of this warp
    const int half = ew >> 2;                     // column half
    const uint32_t lane_base = (uint32_t)(q * 32) << 16;
    float *red = reinterpret_cast<float *>(unit_q + UG_UQ);   // [2 parity][2 half][128 rows]
    uint32_t acc_phase = 0;
    int qs = 0; uint32_t qph = 0;
    for (;;) {
      mbar_wait(&uq_full[qs], qph);
      const int u = unit_q[qs];
      __syncwarp();
      if (lane == 0) mbar_arrive(&uq_empty[qs]);
      if (++qs == UG_UQ) { qs = 0; qph ^= 1; }
      const UnitInfo ui = decode_unit(p, u, n_routed_units);
      if (!ui.valid) break;
      const UmmaGroup &g = p.g[ui.group];
      mbar_wait(tmem_full, acc_phase);
      tc_fence_after();
      const int row = ui.row0 + q * 32 + lane;
      const bool live = row < ui.row_end;
      if (p.debug_mode >= 1 && p.debug_mode <= 5) {   // debug: no epilogue work
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(tmem_empty);
        acc_phase ^= 1;
        continue;
      }
      if constexpr (EPI == GEMM_SWIGLU) {
        // gate columns [64*half, +64), up columns [128 + 64*half, +64)
        uint32_t gr[64], ur[64];
        tmem_ld_32x32b_x32(tmem + lane_base + half * 64, *reinterpret_cast<uint32_t(*)[32]>(gr));
        tmem_ld_32x32b_x32(tmem + lane_base + half * 64 + 32, *reinterpret_cast<uint32_t(*)[32]>(gr + 32));
        tmem_ld_32x32b_x32(tmem + lane_base + 128 + half * 64, *reinterpret_cast<uint32_t(*)[32]>(ur));
        tmem_ld_32x32b_x32(tmem + lane_base + 128 + half * 64 + 32, *reinterpret_cast<uint32_t(*)[32]>(ur + 32));
        tmem_ld_wait();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(tmem_empty);
        float h[64];
        float amax = 0.f;
#pragma unroll
        for (int i = 0; i < 64; ++i) {
          h[i] = silu_f(__uint_as_float(gr[i])) * __uint_as_float(ur[i]);
          amax = fmaxf(amax, fabsf(h[i]));
        }
        const int f0 = ui.nb * 128 + half * 64;
        if (FP8) {
          // the 1x128 block of h spans both halves: exchange partial amax
          float *rb = red + (acc_phase * 2) * 128;
          rb[half * 128 + q * 32 + lane] = amax;
          asm volatile("bar.sync 1, 256;" ::: "memory");
          amax = fmaxf(amax, rb[(half ^ 1) * 128 + q * 32 + lane]);
          const int e = ue8m0_exponent(amax);
          const float inv = exp2i(-e);
          if (live) {
            uint4 *dst = reinterpret_cast<uint4 *>(reinterpret_cast<uint8_t *>(g.out) + (size_t)row * g.ldc + f0);
#pragma unroll
            for (int v = 0; v < 4; ++v) {
              uint32_t w[4];
#pragma unroll
              for (int j = 0; j < 4; ++j) {
                const int b = v * 16 + j * 4;
                w[j] = (uint32_t)f32_to_e4m3(h[b] * inv) | ((uint32_t)f32_to_e4m3(h[b + 1] * inv) << 8) |
                       ((uint32_t)f32_to_e4m3(h[b + 2] * inv) << 16) | ((uint32_t)f32_to_e4m3(h[b + 3] * inv) << 24);
              }
              dst[v] = make_uint4(w[0], w[1], w[2], w[3]);
            }
            if (half == 0) g.out_sf[sf_img_off(row, ui.nb, g.out_sf_tile_stride)] = (uint8_t)(e + 127);
          }
        } else if (live) {
          uint4 *dst = reinterpret_cast<uint4 *>(reinterpret_cast<__nv_bfloat16 *>(g.out) + (size_t)row * g.ldc + f0);
#pragma unroll
          for (int v = 0; v < 8; ++v) {
            uint32_t w[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              __nv_bfloat162 b2 = __floats2bfloat162_rn(h[v * 8 + 2 * j], h[v * 8 + 2 * j + 1]);
              w[j] = *reinterpret_cast<uint32_t *>(&b2);
            }
            dst[v] = make_uint4(w[0], w[1], w[2], w[3]);
          }
        }
      } else {
        // PLAIN (bf16 rows) / LOGITS (fp32 rows): columns [128*half, +128)
        uint32_t r[128];
#pragma unroll
        for (int c = 0; c < 4; ++c)
          tmem_ld_32x32b_x32(tmem + lane_base + half * 128 + c * 32, *reinterpret_cast<uint32_t(*)[32]>(r + 32 * c));
        tmem_ld_wait();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(tmem_empty);
        const int n0 = ui.nb * UG_BN + half * 128;
        if constexpr (EPI == GEMM_LOGITS) {
          // router logits: fp32 columns n < n_valid (PAPER.md L187 gating network)
          if (live) {
            float *crow = reinterpret_cast<float *>(g.out) + (size_t)row * g.ldc;
            if ((g.ldc & 3) == 0 && n0 + 128 <= g.n_valid) {
              // 16-byte stores (4-byte stores put 32 rows x 4 B in every warp store)
              float4 *c4 = reinterpret_cast<float4 *>(crow + n0);
#pragma unroll
              for (int i = 0; i < 32; ++i)
                c4[i] = make_float4(__uint_as_float(r[4 * i]), __uint_as_float(r[4 * i + 1]),
                                    __uint_as_float(r[4 * i + 2]), __uint_as_float(r[4 * i + 3]));
            } else {
#pragma unroll
              for (int i = 0; i < 128; ++i)
                if (n0 + i < g.n_valid) crow[n0 + i] = __uint_as_float(r[i]);
            }
          }
        } else if (live) {
          uint4 *dst = reinterpret_cast<uint4 *>(reinterpret_cast<__nv_bfloat16 *>(g.out) + (size_t)row * g.ldc + n0);
#pragma unroll
          for (int v = 0; v < 16; ++v) {
            uint32_t w[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              __nv_bfloat162 b2 = __floats2bfloat162_rn(__uint_as_float(r[v * 8 + 2 * j]),
                                                        __uint_as_float(r[v * 8 + 2 * j + 1]));
              w[j] = *reinterpret_cast<uint32_t *>(&b2);
            }
            dst[v] = make_uint4(w[0], w[1], w[2], w[3]);
          }
        }
      }
      acc_phase ^= 1;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc(tmem, UG_TMEM_COLS);
}

template <bool FP8, int EPI>
static cudaError_t launch_one(const UmmaParams &p, int grid, cudaStream_t st) {
  auto k = umma_grouped_gemm<FP8, EPI>;
  static bool attr_set = false;
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)UG_SMEM);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  k<<<grid, UG_THREADS, UG_SMEM, st>>>(p);
  return cudaGetLastError();
}

cudaError_t launch_umma_gemm(bool fp8, int epi, const UmmaParams &p, int grid, cudaStream_t st) {
  if (grid <= 0) return cudaSuccess;
  if (epi == GEMM_LOGITS && !fp8) return launch_one<false, GEMM_LOGITS>(p, grid, st);
  return cudaErrorInvalidValue;   // expert GEMMs run in umma_swap.cu
}

// ------------------------------------------------------------------ weight tiling
// one thread per 16-byte chunk of the destination
__global__ void tile_weights_kernel(const uint8_t *__restrict__ src, uint8_t *__restrict__ dst, int nexp, int rows,
                                    int kbytes, int interleave_f, int es) {
  const int nt = rows / 256, kbn = kbytes / 128;
  const int64_t per_exp = (int64_t)rows * kbytes / 16;
  const int64_t total = per_exp * nexp;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < total; c += (int64_t)gridDim.x * blockDim.x) {
    const int64_t e = c / per_exp;
    int64_t rem = c % per_exp;
    const int64_t tile = rem / (256 * 8);          // 2048 chunks of 16 B per tile
    const int in = (int)(rem % (256 * 8));
    const int r = in >> 3, j = in & 7;              // tile row, 16-byte chunk slot (swizzled)
    const int nb = (int)(tile / kbn), kb = (int)(tile % kbn);
    const int jsrc = j ^ (r & 7);                    // chunk j of row r holds source chunk j ^ (r % 8)
    int srow;
    if (interleave_f > 0) {
      // W13 tile nb = h block nb (128 h columns); 128-row half c holds, per
      // 32-row lane quadrant q, [gate | up | gate | up] of columns
      // 128 nb + 64 c + 32 (q >> 1) + i  (umma_swap.cu / umma_decode.cu epilogues)
      const int c = r >> 7, q = (r >> 5) & 3, i = r & 31;
      const int f = nb * 128 + c * 64 + (q >> 1) * 32 + i;
      srow = (q & 1) ? interleave_f + f : f;
    } else {
      srow = nb * 256 + r;
    }
    const uint4 v = *reinterpret_cast<const uint4 *>(src + ((int64_t)e * rows + srow) * kbytes + (int64_t)kb * 128 +
                                                     jsrc * 16);
    *reinterpret_cast<uint4 *>(dst + c * 16) = v;
  }
  (void)nt; (void)es;
}

cudaError_t launch_tile_weights(const void *src, void *dst, int nexp, int rows, int kbytes, int interleave_f,
                                cudaStream_t st) {
  tile_weights_kernel<<<148 * 8, 256, 0, st>>>(reinterpret_cast<const uint8_t *>(src),
                                              reinterpret_cast<uint8_t *>(dst), nexp, rows, kbytes, interleave_f, 1);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ tensor maps
static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    void *ptr = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(ptr);
  }
  return fn;
}

// plain 2-D view of a pre-tiled / scale-image buffer: rows of row_elems
// elements (uint8 or uint32), box = (row_elems, box_rows), no swizzle
bool make_rows_map(CUtensorMap *m, const void *base, bool u32, int64_t rows, int row_elems, int box_rows) {
  auto enc = get_encode();
  if (!enc) return false;
  const int es = u32 ? 4 : 1;
  cuuint64_t dims[2] = {(cuuint64_t)row_elems, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)row_elems * es};
  cuuint32_t box[2] = {(cuuint32_t)row_elems, (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(m, u32 ? CU_TENSOR_MAP_DATA_TYPE_UINT32 : CU_TENSOR_MAP_DATA_TYPE_UINT8, 2,
                   const_cast<void *>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

// contiguous buffer viewed as rows of row_bytes (8-byte elements), box = box_rows
// whole rows: few, long TMA rows for pre-tiled (already swizzled) operands
bool make_blocks_map(CUtensorMap *m, const void *base, int64_t total_bytes, int row_bytes, int box_rows) {
  auto enc = get_encode();
  if (!enc) return false;
  cuuint64_t dims[2] = {(cuuint64_t)(row_bytes / 8), (cuuint64_t)(total_bytes / row_bytes)};
  cuuint64_t strides[1] = {(cuuint64_t)row_bytes};
  cuuint32_t box[2] = {(cuuint32_t)(row_bytes / 8), (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_UINT64, 2, const_cast<void *>(base), dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

// 2-D row-major [rows, cols] K-major operand, box = (128 bytes of K, box_rows), 128B swizzle
bool make_kmajor_map(CUtensorMap *m, const void *base, bool fp8, int64_t rows, int64_t cols, int box_rows) {
  auto enc = get_encode();
  if (!enc) return false;
  const int es = fp8 ? 1 : 2;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)(cols * es)};
  cuuint32_t box[2] = {(cuuint32_t)(128 / es), (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(m, fp8 ? CU_TENSOR_MAP_DATA_TYPE_UINT8 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2,
                   const_cast<void *>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

}  // namespace moe
