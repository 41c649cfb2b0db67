// umma_gemm2.cu -- the grouped expert GEMM on CTA pairs (tcgen05 cta_group::2).
//
// Same work as umma_gemm.cu (routed experts over the expert-sorted rows +
// the shared expert, SwiGLU / plain epilogues), but a cluster of two CTAs on
// two SMs of a TPC runs one 256 x 256 MMA tile: each CTA stages its own 128
// activation rows and HALF of the 256 weight rows; the pair leader issues
// tcgen05.mma.cta_group::2, which reads the other half of B from the peer's
// shared memory.  Per SM this halves the weight bytes moved per MMA, so the
// load pipeline (the limiter of the 1-CTA kernel) keeps up with
// the tensor cores; the freed shared memory buys a 6-stage ring.
//   work unit = (expert, 256-wide n block, pair of 128-row tiles), claimed
//   by the leader from a global counter (the L181 dynamic scheduler) and
//   forwarded to the peer through distributed shared memory.
#include <cuda.h>

#include "common.cuh"
#include "kernels.h"
#include "sm100.cuh"

namespace moe {
using namespace sm100;

constexpr int P2_BM = 128, P2_BN = 256, P2_STAGES = 6, P2_THREADS = 320;
constexpr int P2_A_BYTES = P2_BM * 128;          // this CTA's 128 rows x 128 B
constexpr int P2_B_BYTES = 128 * 128;            // this CTA's half of the 256 weight rows
constexpr int P2_SFA_BYTES = 512, P2_SFB_BYTES = 1024;
constexpr int P2_UQ = 4;
constexpr uint32_t P2_TMEM_COLS = 512;
constexpr uint32_t P2_SFA_COL = 256, P2_SFB_COL = 264;
constexpr size_t P2_SMEM =
    1024 + (size_t)P2_STAGES * (P2_A_BYTES + P2_B_BYTES + P2_SFA_BYTES + P2_SFB_BYTES) + 512 + 2048;

struct PairUnit {
  int valid, group, expert, row0, row_end, nb;   // row0 = first row of the pair (CTA c adds 128 c)
};

__device__ __forceinline__ PairUnit decode_pair_unit(const UmmaParams &p, int u, int n_routed_units) {
  PairUnit r{};
  if (u < n_routed_units) {
    const int nb_r = p.nb_r;
    const int4 any = p.pairs[u / nb_r];
    const int p0 = any.w & 0xFFFF, np = any.w >> 16;
    const int local = u - p0 * nb_r;
    const int4 pr = p.pairs[p0 + local % np];
    r.valid = 1; r.group = 0; r.expert = pr.x; r.row0 = pr.y; r.row_end = pr.z; r.nb = local / np;
    return r;
  }
  const int us = u - n_routed_units;
  const int npair = (p.T_shared + 2 * P2_BM - 1) / (2 * P2_BM);
  if (p.T_shared > 0 && us < npair * p.nb_s) {
    r.valid = 1; r.group = 1; r.expert = 0; r.nb = us / npair;
    r.row0 = (us % npair) * 2 * P2_BM; r.row_end = p.T_shared;
  }
  return r;
}

template <bool FP8, int EPI>
__global__ void __launch_bounds__(P2_THREADS, 1) umma_pair_gemm(const __grid_constant__ UmmaParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t *sA = smem;
  uint8_t *sB = sA + P2_STAGES * P2_A_BYTES;
  uint8_t *sSFA = sB + P2_STAGES * P2_B_BYTES;
  uint8_t *sSFB = sSFA + P2_STAGES * P2_SFA_BYTES;
  uint64_t *full = reinterpret_cast<uint64_t *>(sSFB + P2_STAGES * P2_SFB_BYTES);
  uint64_t *empty = full + P2_STAGES;
  uint64_t *tmem_full = empty + P2_STAGES;
  uint64_t *tmem_empty = tmem_full + 1;
  uint64_t *uq_full = tmem_empty + 1;
  uint64_t *uq_empty = uq_full + P2_UQ;
  uint32_t *tmem_base_smem = reinterpret_cast<uint32_t *>(uq_empty + P2_UQ);
  int *unit_q = reinterpret_cast<int *>(tmem_base_smem + 4);
  float *red = reinterpret_cast<float *>(unit_q + P2_UQ);    // [2 parity][2 half][128 rows]

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t crank = cluster_rank();
  const bool leader = crank == 0;
  const int n_routed_units = p.pairs ? (*p.n_pairs) * p.nb_r : 0;

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&p.g[0].a_map); prefetch_tmap(&p.g[1].a_map);
    prefetch_tmap(&p.g[0].b_map); prefetch_tmap(&p.g[1].b_map);
    for (int s = 0; s < P2_STAGES; ++s) { mbar_init(&full[s], 2); mbar_init(&empty[s], 1); }
    mbar_init(tmem_full, 1);
    mbar_init(tmem_empty, 16);                   // 8 epilogue warps x 2 CTAs (leader's copy is used)
    // leader's uq_empty: MMA warp + 8 epilogue warps (leader) + producer + 8 epilogue warps (peer)
    for (int i = 0; i < P2_UQ; ++i) { mbar_init(&uq_full[i], 1); mbar_init(&uq_empty[i], 18); }
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc_pair(tmem_base_smem, P2_TMEM_COLS);
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  const uint32_t tmem = *tmem_base_smem;

  // consumers hand a unit-queue slot back to the leader
  auto release_slot = [&](int qs) {
    if (leader) mbar_arrive(&uq_empty[qs]);
    else mbar_arrive_cluster(map_to_rank(&uq_empty[qs], 0));
  };
  auto next_unit = [&](int &qs, uint32_t &qph) {
    if (leader) mbar_wait(&uq_full[qs], qph);
    else mbar_wait_cluster(&uq_full[qs], qph);   // unit id was written by the leader (DSMEM)
    const int u = unit_q[qs];
    __syncwarp();
    if (lane == 0) release_slot(qs);
    if (++qs == P2_UQ) { qs = 0; qph ^= 1; }
    return u;
  };

  if (warp == 0) {
    // ============================ TMA producer (both CTAs) ============================
    if (lane == 0) {
      int stage = 0; uint32_t phase = 0;
      int qs = 0; uint32_t qph = 0;
      for (;;) {
        int u;
        if (leader) {
          // dynamic scheduler: claim the next unit, publish it to both CTAs
          u = atomicAdd(p.sched, 1);
          mbar_wait(&uq_empty[qs], qph ^ 1);
          unit_q[qs] = u;
          st_cluster_u32(map_to_rank(&unit_q[qs], 1), (uint32_t)u);
          mbar_arrive(&uq_full[qs]);
          mbar_arrive_cluster(map_to_rank(&uq_full[qs], 1));
          if (++qs == P2_UQ) { qs = 0; qph ^= 1; }
        } else {
          mbar_wait_cluster(&uq_full[qs], qph);
          u = unit_q[qs];
          mbar_arrive_cluster(map_to_rank(&uq_empty[qs], 0));
          if (++qs == P2_UQ) { qs = 0; qph ^= 1; }
        }
        const PairUnit ui = decode_pair_unit(p, u, n_routed_units);
        if (!ui.valid) break;
        const UmmaGroup &g = p.g[ui.group];
        const int arow = ui.row0 + (int)crank * P2_BM;
        // tiled weights: 256-row tile (expert, nb, kb), this CTA's 128-row half
        const int64_t btile = ((int64_t)ui.expert * g.b_ntiles_n + ui.nb) * g.kblocks;
        for (int kb = 0; kb < g.kblocks; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          const uint32_t bytes = P2_A_BYTES + P2_B_BYTES + (FP8 ? P2_SFA_BYTES + P2_SFB_BYTES : 0);
          if (leader) mbar_expect_tx(&full[stage], 2 * bytes);
          else mbar_arrive_cluster(map_to_rank(&full[stage], 0));
          const int kc = kb * (FP8 ? 128 : 64);
          tma_load_2d_pair(sA + stage * P2_A_BYTES, &g.a_map, &full[stage], kc, arow);
          tma_load_2d_pair(sB + stage * P2_B_BYTES, &g.b_map, &full[stage], 0, (int)((btile + kb) * 256 + crank * 128));
          if (FP8) {
            tma_load_2d_pair(sSFA + stage * P2_SFA_BYTES, &g.sfa_map, &full[stage], 0,
                             (kb >> 2) * g.sfa_tile_stride + (arow >> 7));
            tma_load_2d_pair(sSFB + stage * P2_SFB_BYTES, &g.sfb_map, &full[stage], 0,
                             (int)(((int64_t)ui.expert * ((g.kblocks + 3) >> 2) + (kb >> 2)) * g.sfb_rb + ui.nb * 2));
          }
          if (++stage == P2_STAGES) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ============================ MMA issuer (pair leader) ============================
    if (leader) {
      int stage = 0; uint32_t phase = 0; uint32_t acc_phase = 0;
      int qs = 0; uint32_t qph = 0;
      constexpr uint32_t kIdesc = FP8 ? 0u : idesc_bf16(2 * P2_BM, P2_BN);
      for (;;) {
        const int u = next_unit(qs, qph);
        const PairUnit ui = decode_pair_unit(p, u, n_routed_units);
        if (!ui.valid) break;
        const int kblocks = p.g[ui.group].kblocks;
        mbar_wait(tmem_empty, acc_phase ^ 1);
        tc_fence_after();
        for (int kb = 0; kb < kblocks; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          if (lane == 0 && p.debug_mode == 1) {       // timing experiment: loads only
            mbar_arrive(&empty[stage]);
            mbar_arrive_cluster(map_to_rank(&empty[stage], 1));
            if (kb == kblocks - 1) { mbar_arrive(tmem_full); mbar_arrive_cluster(map_to_rank(tmem_full, 1)); }
          } else if (lane == 0) {
            const uint32_t a0 = smem_u32(sA + stage * P2_A_BYTES);
            const uint32_t b0 = smem_u32(sB + stage * P2_B_BYTES);
            if (FP8) {
              tmem_cp_32x128b_x4_pair(tmem + P2_SFA_COL, sf_desc(smem_u32(sSFA + stage * P2_SFA_BYTES)));
              tmem_cp_32x128b_x4_pair(tmem + P2_SFB_COL, sf_desc(smem_u32(sSFB + stage * P2_SFB_BYTES)));
              tmem_cp_32x128b_x4_pair(tmem + P2_SFB_COL + 4, sf_desc(smem_u32(sSFB + stage * P2_SFB_BYTES + 512)));
            }
#pragma unroll
            for (int k = 0; k < 4; ++k) {
              const uint64_t ad = sw128_kmajor_desc(a0 + k * 32);
              const uint64_t bd = sw128_kmajor_desc(b0 + k * 32);
              const uint32_t acc = (kb | k) != 0;
              if (FP8)
                mma_mxf8_pair(tmem, ad, bd, idesc_mxf8(2 * P2_BM, P2_BN, kb & 3, kb & 3), acc, tmem + P2_SFA_COL,
                              tmem + P2_SFB_COL);
              else
                mma_bf16_pair(tmem, ad, bd, kIdesc, acc);
            }
            mma_commit_pair(&empty[stage]);
            if (kb == kblocks - 1) mma_commit_pair(tmem_full);
          }
          __syncwarp();
          if (++stage == P2_STAGES) { stage = 0; phase ^= 1; }
        }
        acc_phase ^= 1;
      }
    }
  } else {
    // ============================ epilogue (8 warps, both CTAs) ============================
    const int ew = warp - 2;
    const int q = warp & 3;
    const int half = ew >> 2;
    const uint32_t lane_base = (uint32_t)(q * 32) << 16;
    const uint32_t tmem_empty_leader = map_to_rank(tmem_empty, 0);
    auto release_tmem = [&]() {
      if (leader) mbar_arrive(tmem_empty);
      else mbar_arrive_cluster(tmem_empty_leader);
    };
    uint32_t acc_phase = 0;
    int qs = 0; uint32_t qph = 0;
    for (;;) {
      const int u = next_unit(qs, qph);
      const PairUnit ui = decode_pair_unit(p, u, n_routed_units);
      if (!ui.valid) break;
      const UmmaGroup &g = p.g[ui.group];
      mbar_wait(tmem_full, acc_phase);
      tc_fence_after();
      const int row = ui.row0 + (int)crank * P2_BM + q * 32 + lane;
      const bool live = row < ui.row_end;
      if (p.debug_mode >= 1) {                   // timing experiment: no epilogue work
        tc_fence_before();
        __syncwarp();
        if (lane == 0) release_tmem();
        acc_phase ^= 1;
        continue;
      }
      if constexpr (EPI == GEMM_SWIGLU) {
        uint32_t gr[64], ur[64];
        tmem_ld_32x32b_x32(tmem + lane_base + half * 64, *reinterpret_cast<uint32_t(*)[32]>(gr));
        tmem_ld_32x32b_x32(tmem + lane_base + half * 64 + 32, *reinterpret_cast<uint32_t(*)[32]>(gr + 32));
        tmem_ld_32x32b_x32(tmem + lane_base + 128 + half * 64, *reinterpret_cast<uint32_t(*)[32]>(ur));
        tmem_ld_32x32b_x32(tmem + lane_base + 128 + half * 64 + 32, *reinterpret_cast<uint32_t(*)[32]>(ur + 32));
        tmem_ld_wait();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) release_tmem();
        float h[64];
        float amax = 0.f;
#pragma unroll
        for (int i = 0; i < 64; ++i) {
          h[i] = silu_f(__uint_as_float(gr[i])) * __uint_as_float(ur[i]);
          amax = fmaxf(amax, fabsf(h[i]));
        }
        const int f0 = ui.nb * 128 + half * 64;
        if (FP8) {
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
        uint32_t r[128];
#pragma unroll
        for (int c = 0; c < 4; ++c)
          tmem_ld_32x32b_x32(tmem + lane_base + half * 128 + c * 32, *reinterpret_cast<uint32_t(*)[32]>(r + 32 * c));
        tmem_ld_wait();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) release_tmem();
        const int n0 = ui.nb * P2_BN + half * 128;
        if (live) {
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
  cluster_sync();
  if (warp == 1) tmem_dealloc_pair(tmem, P2_TMEM_COLS);
}

template <bool FP8, int EPI>
static cudaError_t launch_pair(const UmmaParams &p, int grid, cudaStream_t st) {
  auto k = umma_pair_gemm<FP8, EPI>;
  static bool set = false;
  if (!set) {
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)P2_SMEM);
    if (e != cudaSuccess) return e;
    set = true;
  }
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid & ~1);
  cfg.blockDim = dim3(P2_THREADS);
  cfg.dynamicSmemBytes = P2_SMEM;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k, p);
}

cudaError_t launch_umma_pair_gemm(bool fp8, int epi, const UmmaParams &p, int grid, cudaStream_t st) {
  if (grid < 2) grid = 2;
  if (fp8) return epi == GEMM_SWIGLU ? launch_pair<true, GEMM_SWIGLU>(p, grid, st) : launch_pair<true, GEMM_PLAIN>(p, grid, st);
  return epi == GEMM_SWIGLU ? launch_pair<false, GEMM_SWIGLU>(p, grid, st) : launch_pair<false, GEMM_PLAIN>(p, grid, st);
}

}  // namespace moe
