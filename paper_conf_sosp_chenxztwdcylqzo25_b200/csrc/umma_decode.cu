// umma_decode.cu -- decode expert FFNs on the tensor cores, swap-AB.
//
// With <= 16 tokens per expert the FFN is HBM-bound:
// each active expert's weights must stream through once.  Here the weights
// are the tcgen05 A operand (M = 128 weight rows per MMA, TMA-fed through a
// 6-stage ring) and the expert's token rows the B operand (N = 16), so the
// tensor cores do the dot products and the kernel is a pure weight stream.
// (The paper's AVX-512 low-ARI kernel, L170, recast for B200: same memory
// layout as the prefill GEMM, a different instruction shape.)
//   MODE 1: unit = (slot, 128 h columns b): the 256-row W13 tile b, whose
//           128-row halves c hold per lane quadrant [gate | up | gate | up] of
//           h columns 128b + 64c + [0, 64) -> two 128x16 accumulators; the up
//           quadrants hand their values to the gate quadrants through shared
//           memory -> SwiGLU -> h (FP8: 1x128 UE8M0 requant from fp32 + image)
//   MODE 2: unit = (slot, 128 rows of W2) -> y rows (bf16)
// Slots: active routed experts (act_list) + the shared expert (last slot).
#include <cuda.h>

#include "common.cuh"
#include "kernels.h"
#include "sm100.cuh"

namespace moe {
using namespace sm100;

constexpr int UD_N = 16, UD_STAGES = 6, UD_THREADS = 192;
constexpr int UD_A_BYTES = 2 * 128 * 128;     // up to two 128-row weight tiles
constexpr int UD_B_BYTES = UD_N * 128;        // 16 token rows x 128 B
constexpr int UD_SFA_BYTES = 512, UD_SFB_BYTES = 512;
constexpr int UD_XCH_FLOATS = 2 * 2 * UD_N * 32;   // up -> gate exchange [gate warp][acc][token][lane]
constexpr size_t UD_SMEM = 1024 + (size_t)UD_STAGES * (UD_A_BYTES + UD_B_BYTES + UD_SFA_BYTES + UD_SFB_BYTES) +
                           UD_XCH_FLOATS * 4 + 1024;
constexpr uint32_t UD_TMEM_COLS = 128;        // 2 acc stages x 32 cols + scale factors
constexpr uint32_t UD_SFA_COL = 64, UD_SFB_COL = 72;

// state: 0 = past the end (stop), 1 = empty slot/block (skip), 3 = work
struct UdUnit {
  int valid, shared, expert, n, row0, blk;
};

// slot 0 = the shared expert (its weights were prefetched into L2 during
// routing, so the first units run from L2), then the active routed experts
__device__ __forceinline__ UdUnit ud_unit(const UmmaDecodeParams &p, int u) {
  UdUnit r{};
  const int slot = u / p.nblk;
  if (slot >= p.max_slots) return r;            // valid = 0
  r.valid = 1;
  r.blk = u % p.nblk;
  const int rs = slot - p.has_shared;           // routed slot index
  if (rs < 0) {
    r.shared = 1; r.expert = 0; r.n = p.T; r.row0 = 0;
  } else if (rs < *p.n_active) {
    const int e = p.act_list[rs];
    r.expert = e; r.n = p.counts[e]; r.row0 = p.offs_pad[e];
  } else {
    return r;
  }
  if (r.blk < p.g_nblk[r.shared]) r.valid = 3;
  return r;
}

template <bool FP8, int MODE>
__global__ void __launch_bounds__(UD_THREADS, 1) umma_decode_kernel(const __grid_constant__ UmmaDecodeParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t *sA = smem;
  uint8_t *sB = sA + UD_STAGES * UD_A_BYTES;
  uint8_t *sSFA = sB + UD_STAGES * UD_B_BYTES;
  uint8_t *sSFB = sSFA + UD_STAGES * UD_SFA_BYTES;
  uint64_t *full = reinterpret_cast<uint64_t *>(sSFB + UD_STAGES * UD_SFB_BYTES);
  uint64_t *empty = full + UD_STAGES;
  uint64_t *tfull = empty + UD_STAGES;          // [2]
  uint64_t *tempty = tfull + 2;                 // [2]
  uint64_t *uq_full = tempty + 2;               // [4]
  uint64_t *uq_empty = uq_full + 4;             // [4]
  uint32_t *tmem_base_smem = reinterpret_cast<uint32_t *>(uq_empty + 4);
  int *unit_q = reinterpret_cast<int *>(tmem_base_smem + 4);
  float *red = reinterpret_cast<float *>(unit_q + 4);   // [4 warps][16 tokens]
  float *xch = red + 4 * UD_N;                           // MODE 1 up -> gate exchange

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  constexpr int NA = MODE == 1 ? 2 : 1;         // weight tiles per unit
  if (warp == 0 && lane == 0) {
    for (int s = 0; s < UD_STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    for (int s = 0; s < 2; ++s) { mbar_init(&tfull[s], 1); mbar_init(&tempty[s], 4); }
    for (int i = 0; i < 4; ++i) { mbar_init(&uq_full[i], 1); mbar_init(&uq_empty[i], 5); }
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc(tmem_base_smem, UD_TMEM_COLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_base_smem;
  pdl_trigger();                                // the next kernel may start its prologue
  pdl_wait();                                   // routing / activations of the predecessor

  if (warp == 0) {
    // ============================ producer ============================
    if (lane == 0) {
      int stage = 0; uint32_t phase = 0, qs = 0, qph = 0;
      for (;;) {
        const int u = atomicAdd(p.sched, 1);
        const UdUnit ui = ud_unit(p, u);
        if (ui.valid == 1) continue;            // empty slot / block: claim the next
        mbar_wait(&uq_empty[qs], qph ^ 1);
        unit_q[qs] = u;
        mbar_arrive(&uq_full[qs]);
        if (++qs == 4) { qs = 0; qph ^= 1; }
        if (!ui.valid) break;
        const UmmaGroup &g = p.g[ui.shared];
        const uint32_t bytes = NA * 128 * 128 + UD_B_BYTES + (FP8 ? UD_SFA_BYTES + UD_SFB_BYTES : 0);
        for (int kb = 0; kb < g.kblocks; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          mbar_expect_tx(&full[stage], bytes);
          const int kc = kb * (FP8 ? 128 : 64);
          // pre-tiled weights: MODE 1 = a whole 256-row tile (gate + up), MODE 2 = one half
          const uint8_t *wt = g.b_tiles +
                              (((size_t)ui.expert * g.b_ntiles_n + (MODE == 1 ? ui.blk : ui.blk >> 1)) * g.kblocks + kb) *
                                  (256 * 128) +
                              (MODE == 1 ? 0 : (ui.blk & 1) * (128 * 128));
          bulk_load(sA + stage * UD_A_BYTES, wt, NA * 128 * 128, &full[stage]);
          tma_load_2d(sB + stage * UD_B_BYTES, &g.a_map, &full[stage], kc, ui.row0);
          if (FP8) {
            // MODE 1: one W13 image per 256-row tile (both halves); MODE 2: per 128-row block
            const uint8_t *sfa = g.sfb + (size_t)ui.expert * g.sfb_expert_stride +
                                 ((size_t)(kb >> 2) * g.sfb_rb + ui.blk) * 512;
            const uint8_t *sfb = g.sfa + ((size_t)(kb >> 2) * g.sfa_tile_stride + (ui.row0 >> 7)) * 512;
            bulk_load(sSFA + stage * UD_SFA_BYTES, sfa, UD_SFA_BYTES, &full[stage]);
            bulk_load(sSFB + stage * UD_SFB_BYTES, sfb, UD_SFB_BYTES, &full[stage]);
          }
          if (++stage == UD_STAGES) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ============================ MMA issuer ============================
    int stage = 0; uint32_t phase = 0, qs = 0, qph = 0;
    int acc = 0; uint32_t acc_ph = 0;
    for (;;) {
      mbar_wait(&uq_full[qs], qph);
      const int u = unit_q[qs];
      __syncwarp();
      if (lane == 0) mbar_arrive(&uq_empty[qs]);
      if (++qs == 4) { qs = 0; qph ^= 1; }
      const UdUnit ui = ud_unit(p, u);
      if (!ui.valid) break;
      const int kblocks = p.g[ui.shared].kblocks;
      mbar_wait(&tempty[acc], acc_ph ^ 1);
      tc_fence_after();
      const uint32_t d0 = tmem + acc * 32;
      for (int kb = 0; kb < kblocks; ++kb) {
        mbar_wait(&full[stage], phase);
        tc_fence_after();
        if (lane == 0) {
          const uint32_t a0 = smem_u32(sA + stage * UD_A_BYTES);
          const uint32_t b0 = smem_u32(sB + stage * UD_B_BYTES);
          if (FP8) {
            tmem_cp_32x128b_x4(tmem + UD_SFA_COL, sf_desc(smem_u32(sSFA + stage * UD_SFA_BYTES)));
            tmem_cp_32x128b_x4(tmem + UD_SFB_COL, sf_desc(smem_u32(sSFB + stage * UD_SFB_BYTES)));
          }
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const uint64_t bd = sw128_kmajor_desc(b0 + k * 32);
            const uint32_t accum = (kb | k) != 0;
#pragma unroll
            for (int t = 0; t < NA; ++t) {
              const uint64_t ad = sw128_kmajor_desc(a0 + t * 128 * 128 + k * 32);
              if (FP8)
                mma_mxf8(d0 + t * 16, ad, bd, idesc_mxf8(128, UD_N, kb & 3, kb & 3), accum,
                         tmem + UD_SFA_COL, tmem + UD_SFB_COL);
              else
                mma_bf16(d0 + t * 16, ad, bd, idesc_bf16(128, UD_N), accum);
            }
          }
          mma_commit(&empty[stage]);
          if (kb == kblocks - 1) mma_commit(&tfull[acc]);
        }
        __syncwarp();
        if (++stage == UD_STAGES) { stage = 0; phase ^= 1; }
      }
      if (++acc == 2) { acc = 0; acc_ph ^= 1; }
    }
  } else {
    // ============================ epilogue (4 warps, lanes = weight rows) ============================
    const int q = warp & 3;
    const uint32_t lane_base = (uint32_t)(q * 32) << 16;
    int acc = 0; uint32_t acc_ph = 0, qs = 0, qph = 0;
    for (;;) {
      mbar_wait(&uq_full[qs], qph);
      const int u = unit_q[qs];
      __syncwarp();
      if (lane == 0) mbar_arrive(&uq_empty[qs]);
      if (++qs == 4) { qs = 0; qph ^= 1; }
      const UdUnit ui = ud_unit(p, u);
      if (!ui.valid) break;
      const UmmaGroup &g = p.g[ui.shared];
      mbar_wait(&tfull[acc], acc_ph);
      tc_fence_after();
      uint32_t r0[16], r1[16];
      tmem_ld_32x32b_x16(tmem + lane_base + acc * 32, r0);
      if (MODE == 1) tmem_ld_32x32b_x16(tmem + lane_base + acc * 32 + 16, r1);
      tmem_ld_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[acc]);
      const int n = ui.n;
      const int wr = q * 32 + lane;             // weight row within the 128-row tile
      if (MODE == 1) {
        // quadrant q of accumulator c: gate (q even) / up (q odd) rows of h
        // column 128 blk + 64 c + 32 (q >> 1) + lane
        const int qg = q >> 1;
        float *xb = xch + qg * (2 * UD_N * 32);
        if (q & 1) {
#pragma unroll
          for (int t = 0; t < UD_N; ++t) {
            xb[t * 32 + lane] = __uint_as_float(r0[t]);
            xb[(UD_N + t) * 32 + lane] = __uint_as_float(r1[t]);
          }
        }
        asm volatile("bar.sync 1, 128;" ::: "memory");
        float h0[UD_N], h1[UD_N];
        if (!(q & 1)) {
#pragma unroll
          for (int t = 0; t < UD_N; ++t) {
            h0[t] = silu_f(__uint_as_float(r0[t])) * xb[t * 32 + lane];
            h1[t] = silu_f(__uint_as_float(r1[t])) * xb[(UD_N + t) * 32 + lane];
          }
        }
        const int f0 = ui.blk * 128 + qg * 32 + lane;       // accumulator 0; accumulator 1 at + 64
        if (FP8) {
          // per token: amax over the 128 h values of this block (2 gate warps x 2 accumulators)
          if (!(q & 1)) {
#pragma unroll
            for (int t = 0; t < UD_N; ++t) {
              const float m = warp_max(fmaxf(fabsf(h0[t]), fabsf(h1[t])));
              if (lane == 0) red[qg * UD_N + t] = m;
            }
          }
          asm volatile("bar.sync 1, 128;" ::: "memory");
          if (!(q & 1)) {
#pragma unroll
            for (int t = 0; t < UD_N; ++t) {
              if (t < n) {
                const int e = ue8m0_exponent(fmaxf(red[t], red[UD_N + t]));
                const float inv = exp2i(-e);
                const int64_t row = (int64_t)ui.row0 + t;
                uint8_t *o = reinterpret_cast<uint8_t *>(g.out) + row * g.ldc;
                o[f0] = f32_to_e4m3(h0[t] * inv);
                o[f0 + 64] = f32_to_e4m3(h1[t] * inv);
                if (qg == 0 && lane == 0) g.out_sf[sf_img_off(row, ui.blk, g.out_sf_tile_stride)] = (uint8_t)(e + 127);
              }
            }
          }
        } else if (!(q & 1)) {
#pragma unroll
          for (int t = 0; t < UD_N; ++t)
            if (t < n) {
              __nv_bfloat16 *o = reinterpret_cast<__nv_bfloat16 *>(g.out) + ((int64_t)ui.row0 + t) * g.ldc;
              o[f0] = __float2bfloat16_rn(h0[t]);
              o[f0 + 64] = __float2bfloat16_rn(h1[t]);
            }
        }
        asm volatile("bar.sync 1, 128;" ::: "memory");   // exchange / red buffers free for the next unit
      } else {
        const int c = ui.blk * 128 + wr;
#pragma unroll
        for (int t = 0; t < UD_N; ++t)
          if (t < n)
            reinterpret_cast<__nv_bfloat16 *>(g.out)[((int64_t)ui.row0 + t) * g.ldc + c] =
                __float2bfloat16_rn(__uint_as_float(r0[t]));
      }
      if (++acc == 2) { acc = 0; acc_ph ^= 1; }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc(tmem, UD_TMEM_COLS);
}

template <bool FP8, int MODE>
static cudaError_t ud_launch(const UmmaDecodeParams &p, int grid, cudaStream_t st) {
  auto k = umma_decode_kernel<FP8, MODE>;
  static bool set = false;
  if (!set) {
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)UD_SMEM);
    if (e != cudaSuccess) return e;
    set = true;
  }
  return launch_pdl(k, dim3(grid), dim3(UD_THREADS), UD_SMEM, st, p);
}

cudaError_t launch_umma_decode(bool fp8, int mode, const UmmaDecodeParams &p, int grid, cudaStream_t st) {
  if (grid <= 0) return cudaSuccess;
  if (fp8) return mode == 1 ? ud_launch<true, 1>(p, grid, st) : ud_launch<true, 2>(p, grid, st);
  return mode == 1 ? ud_launch<false, 1>(p, grid, st) : ud_launch<false, 2>(p, grid, st);
}

}  // namespace moe
