// umma_decode_fused.cu -- decode expert FFNs as ONE weight stream per unit.
//
// Decode (<= 16 tokens per expert) is HBM-bound: every
// active expert's W13 and W2 must stream through once.  The two-launch chain
// (umma_decode.cu: W13 -> h in HBM -> W2) pays a launch drain, a W2 tail wave
// (9 x 56 row blocks on 148 SMs) and the h round trip.  Here a unit is
// (slot, 128-column chunk c of the expert's FFN dimension):
//   phase A: stream the 256-row W13 tile c (gate + up rows of h columns
//            128c .. 128c+127, all H) through the swap-AB MMA (weights = the
//            M = 128 operand, the slot's <= 16 token rows the N = 16 operand),
//            SwiGLU from fp32 TMEM, FP8: 1x128 UE8M0 requant -- exactly the
//            128-column block of R10/R11, so the scale is local to the unit --
//            and write h_c [16 tokens x 128] into shared memory as the B
//            operand of phase B (SW128 K-major image, no HBM round trip);
//   phase B: stream W2[:, 128c .. 128c+127] (H/256 tiles of 256 rows x 128 B)
//            against h_c: one k-block per 128-row M tile, so the MMA is the
//            unscaled kind::f8f6f4 and the W2 block scale x the h scale are
//            applied in the epilogue, which adds w_tj * partial into an fp32
//            [T, H] accumulator (red.global.add; immediate or deferred sum,
//            PAPER.md L219-241) -- the k-sum over chunks and the weighted
//            combine over a token's experts (L187) happen in the same adds.
// Units are claimed from a device counter (the L181 dynamic task queue): the
// shared expert's chunks first, then the active routed experts (ascending id).
// The kernel is PDL-launched while the router runs; every warp waits for the
// router's completion before touching routing data or activations (an optional
// L2 prefetch of the shared expert before that wait, MOE_DECODE_PF=1, measured
// slower).  The weight stream uses an evict-first L2 policy.
// decode_finalize_kernel adds the residual / deferred input, writes bf16 y (and
// deferred_out) and re-zeroes the sums.
//
// Summation order across chunks is the order of the atomics (fp32; results
// are reproducible to fp32 rounding, not bitwise) -- DESIGN.md reading R22.
#include <cuda.h>
#include <cstdio>

#include "common.cuh"
#include "kernels.h"
#include "sm100.cuh"

namespace moe {
using namespace sm100;

constexpr int FD_N = 16, FD_STAGES = 5, FD_THREADS = 192, FD_UQ = 4, FD_ACCB = 4;
constexpr int FD_A_BYTES = 256 * 128;          // one 256-row weight tile k-block (two 128-row MMA tiles)
constexpr int FD_B_BYTES = FD_N * 128;         // 16 token rows x 128 B
constexpr int FD_SF_BYTES = 512;
constexpr int FD_H_BYTES = 2 * FD_B_BYTES;     // h_c: FP8 one k-block, BF16 two
constexpr size_t FD_SMEM = 1024 + (size_t)FD_STAGES * (FD_A_BYTES + FD_B_BYTES + 2 * FD_SF_BYTES) + FD_H_BYTES +
                           2 * 2 * FD_N * 32 * 4 +     // up -> gate exchange [gate warp][acc][token][lane]
                           1024;                       // barriers, queue, amax, scales
constexpr uint32_t FD_TMEM_COLS = 256;
constexpr uint32_t FD_ACCA = 0, FD_SFA_COL = 32, FD_SFB_COL = 40, FD_ACCB_COL = 64;   // + 32 per ring slot

// instruction descriptor, kind::f8f6f4 (E4M3 x E4M3 -> F32, no block scale), K-major A and B
__host__ __device__ constexpr uint32_t idesc_f8(int M, int N) {
  return (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
__device__ __forceinline__ void mma_f8(uint32_t d_tmem, uint64_t a_desc, uint64_t b_desc, uint32_t idesc,
                                       uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f8f6f4 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(a_desc), "l"(b_desc), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// unit -> (valid, group, expert, row0, n tokens, chunk).  valid: 0 = past the end
struct FdUnit {
  int valid, group, expert, row0, n, chunk;
};

__device__ __forceinline__ FdUnit fd_unit(const FusedDecodeParams &p, int u) {
  // decode TP (moe_layer_set_decode_tp): this rank streams the chunks c = tp_rank + tp_size * j
  // of every expert (W13 rows and W2 columns of the same 128 FFN columns), so its partial sum
  // over chunks is its share of every expert's output
  const int P = p.tp_size > 1 ? p.tp_size : 1, rk = P > 1 ? p.tp_rank : 0;
  const int nl0 = (p.nch[0] - rk + P - 1) / P, nl1 = (p.nch[1] - rk + P - 1) / P;
  FdUnit r{};
  const int ns = p.has_shared ? nl1 : 0;
  if (u < ns) {
    r.valid = 1; r.group = 1; r.expert = 0; r.row0 = 0; r.n = p.T; r.chunk = rk + P * u;
    return r;
  }
  const int v = u - ns;
  const int slot = v / nl0;
  if (slot >= *p.n_active) return r;
  const int e = p.act_list[slot];
  // token-order activations (all T <= 16 tokens are the N = 16 operand; the
  // epilogue keeps the columns of the tokens routed to e)
  r.valid = 1; r.group = 0; r.expert = e; r.row0 = 0; r.n = p.T; r.chunk = rk + P * (v % nl0);
  return r;
}

// y = bf16(residual + acc_imm + deferred_in); deferred_out = bf16(acc_def); sums re-zeroed.
// Elements first, first + stride, ... of the T*H/8 8-element groups.
__device__ __forceinline__ void decode_finalize_range(const DecodeFinalizeArgs &a, int64_t first, int64_t stride) {
  const int64_t n8 = (int64_t)a.T * a.H / 8;
  for (int64_t i = first; i < n8; i += stride) {
    float4 *s4 = reinterpret_cast<float4 *>(a.acc_imm) + 2 * i;
    float4 u0 = s4[0], u1 = s4[1];
    float v[8] = {u0.x, u0.y, u0.z, u0.w, u1.x, u1.y, u1.z, u1.w};
    s4[0] = make_float4(0.f, 0.f, 0.f, 0.f);
    s4[1] = make_float4(0.f, 0.f, 0.f, 0.f);
    if (a.residual) {
      float f[8];
      bf16x8_to_f32(reinterpret_cast<const uint4 *>(a.residual)[i], f);
#pragma unroll
      for (int j = 0; j < 8; ++j) v[j] += f[j];
    }
    if (a.deferred_in) {
      float f[8];
      bf16x8_to_f32(reinterpret_cast<const uint4 *>(a.deferred_in)[i], f);
#pragma unroll
      for (int j = 0; j < 8; ++j) v[j] += f[j];
    }
    uint4 o;
    __nv_bfloat162 *ob = reinterpret_cast<__nv_bfloat162 *>(&o);
#pragma unroll
    for (int j = 0; j < 4; ++j) ob[j] = __floats2bfloat162_rn(v[2 * j], v[2 * j + 1]);
    reinterpret_cast<uint4 *>(a.y)[i] = o;
    if (a.deferred_out) {
      float4 d0 = make_float4(0.f, 0.f, 0.f, 0.f), d1 = d0;
      if (a.use_def) {
        float4 *d4 = reinterpret_cast<float4 *>(a.acc_def) + 2 * i;
        d0 = d4[0]; d1 = d4[1];
        d4[0] = make_float4(0.f, 0.f, 0.f, 0.f);
        d4[1] = make_float4(0.f, 0.f, 0.f, 0.f);
      }
      {
        uint4 od;
        __nv_bfloat162 *db = reinterpret_cast<__nv_bfloat162 *>(&od);
        db[0] = __floats2bfloat162_rn(d0.x, d0.y); db[1] = __floats2bfloat162_rn(d0.z, d0.w);
        db[2] = __floats2bfloat162_rn(d1.x, d1.y); db[3] = __floats2bfloat162_rn(d1.z, d1.w);
        reinterpret_cast<uint4 *>(a.deferred_out)[i] = od;
      }
    }
  }
}

template <bool FP8>
__global__ void __launch_bounds__(FD_THREADS, 1) umma_decode_fused_kernel(const __grid_constant__ FusedDecodeParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t *sA = smem;
  uint8_t *sH = sA + FD_STAGES * FD_A_BYTES;                 // 1024-aligned
  uint8_t *sB = sH + FD_H_BYTES;
  uint8_t *sSFA = sB + FD_STAGES * FD_B_BYTES;
  uint8_t *sSFB = sSFA + FD_STAGES * FD_SF_BYTES;
  float *xch = reinterpret_cast<float *>(sSFB + FD_STAGES * FD_SF_BYTES);   // [2][2][16][32]
  uint64_t *full = reinterpret_cast<uint64_t *>(xch + 2 * 2 * FD_N * 32);
  uint64_t *empty = full + FD_STAGES;
  uint64_t *accA_full = empty + FD_STAGES;
  uint64_t *h_ready = accA_full + 1;
  uint64_t *accB_full = h_ready + 1;                         // [FD_ACCB]
  uint64_t *accB_empty = accB_full + FD_ACCB;                // [FD_ACCB]
  uint64_t *uq_full = accB_empty + FD_ACCB;                  // [FD_UQ]
  uint64_t *uq_empty = uq_full + FD_UQ;                      // [FD_UQ]
  uint32_t *tmem_base_smem = reinterpret_cast<uint32_t *>(uq_empty + FD_UQ);
  int4 *unit_q = reinterpret_cast<int4 *>(tmem_base_smem + 4);   // [FD_UQ] (expert, row0, n | chunk << 16, group | valid << 1)
  float *amax = reinterpret_cast<float *>(unit_q + FD_UQ);       // [2 gate warps][16]
  float *hsc = amax + 2 * FD_N;                                  // [2 unit parity][16] h scale per token (FP8)

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == 0 && lane == 0) {
    for (int s = 0; s < FD_STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    mbar_init(accA_full, 1);
    mbar_init(h_ready, 1);
    for (int s = 0; s < FD_ACCB; ++s) { mbar_init(&accB_full[s], 1); mbar_init(&accB_empty[s], 4); }
    for (int i = 0; i < FD_UQ; ++i) { mbar_init(&uq_full[i], 1); mbar_init(&uq_empty[i], 5); }
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc(tmem_base_smem, FD_TMEM_COLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_base_smem;

  constexpr int KDIV = FP8 ? 128 : 64;           // elements per 128-byte k-block
  constexpr int KBC = 128 / KDIV;                // W2 k-blocks per 128-column chunk
  const int KA = p.H / KDIV;                     // W13 k-blocks
  const int NT = p.H / 256;                      // W2 256-row tiles

  if (warp == 0) {
    // ============================ producer ============================
    if (lane == 0) {
      pdl_wait();                                // routing, xq / xperm of the route kernel
      const uint64_t pol = l2_evict_first_policy();   // weights are read once per forward
      int stage = 0; uint32_t phase = 0, qs = 0, qph = 0;
      for (;;) {
        const int u = atomicAdd(p.sched, 1);
        const FdUnit ui = fd_unit(p, u);
        mbar_wait(&uq_empty[qs], qph ^ 1);
        unit_q[qs] = make_int4(ui.expert, ui.row0, ui.n | (ui.chunk << 16), ui.group | (ui.valid << 1));
        mbar_arrive(&uq_full[qs]);
        if (++qs == FD_UQ) { qs = 0; qph ^= 1; }
        if (!ui.valid) {
          // every load of this CTA is issued: let the finalize kernel launch now, so
          // its launch latency overlaps the last stages (it waits for our completion)
          pdl_trigger();
          break;
        }
        const FdGroup &g = p.g[ui.group];
        // ---- phase A: W13 tile `chunk` (256 rows: gate + up of 128 h columns) ----
        const uint32_t bytes_a = FD_A_BYTES + FD_B_BYTES + (FP8 ? 2 * FD_SF_BYTES : 0);
        const uint8_t *w13 = g.w13 + ((size_t)ui.expert * p.nch[ui.group] + ui.chunk) * (size_t)KA * FD_A_BYTES;
        for (int kb = 0; kb < KA; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          mbar_expect_tx(&full[stage], bytes_a);
          bulk_load_hint(sA + stage * FD_A_BYTES, w13 + (size_t)kb * FD_A_BYTES, FD_A_BYTES, &full[stage], pol);
          tma_load_2d(sB + stage * FD_B_BYTES, &g.x_map, &full[stage], kb * KDIV, ui.row0);
          if (FP8) {
            const uint8_t *sfa = g.w13_img + (size_t)ui.expert * g.w13_img_stride +
                                 ((size_t)(kb >> 2) * p.nch[ui.group] + ui.chunk) * 512;
            const uint8_t *sfb = g.x_img + ((size_t)(kb >> 2) * g.x_img_stride + (ui.row0 >> 7)) * 512;
            bulk_load(sSFA + stage * FD_SF_BYTES, sfa, FD_SF_BYTES, &full[stage]);
            bulk_load(sSFB + stage * FD_SF_BYTES, sfb, FD_SF_BYTES, &full[stage]);
          }
          if (++stage == FD_STAGES) { stage = 0; phase ^= 1; }
        }
        // ---- phase B: W2 column block `chunk`, H/256 tiles of 256 rows ----
        const int KB2 = p.nch[ui.group] * KBC;     // W2 k-blocks per tile row
        const uint8_t *w2 = g.w2 + (size_t)ui.expert * NT * KB2 * FD_A_BYTES;
        for (int n = 0; n < NT; ++n) {
          for (int kk = 0; kk < KBC; ++kk) {
            mbar_wait(&empty[stage], phase ^ 1);
            mbar_expect_tx(&full[stage], FD_A_BYTES);
            bulk_load_hint(sA + stage * FD_A_BYTES, w2 + ((size_t)n * KB2 + ui.chunk * KBC + kk) * FD_A_BYTES,
                           FD_A_BYTES, &full[stage], pol);
            if (++stage == FD_STAGES) { stage = 0; phase ^= 1; }
          }
        }
      }
    }
  } else if (warp == 1) {
    // ============================ MMA issuer ============================
    pdl_wait();                                  // sleep in the grid dependency, not on an mbarrier, during routing
    int stage = 0; uint32_t phase = 0, qs = 0, qph = 0, hph = 0;
    int ab = 0; uint32_t abph = 0;
    for (;;) {
      mbar_wait(&uq_full[qs], qph);
      const int4 uq = unit_q[qs];
      __syncwarp();
      if (lane == 0) mbar_arrive(&uq_empty[qs]);
      if (++qs == FD_UQ) { qs = 0; qph ^= 1; }
      if (!(uq.w >> 1)) break;
      // phase A (the accumulator is free: the epilogue read it before h_ready of the previous unit)
      for (int kb = 0; kb < KA; ++kb) {
        mbar_wait(&full[stage], phase);
        tc_fence_after();
        if (lane == 0) {
          const uint32_t a0 = smem_u32(sA + stage * FD_A_BYTES);
          const uint32_t b0 = smem_u32(sB + stage * FD_B_BYTES);
          // scale images hold 4 k-blocks (scale id kb & 3): copy once per 4 k-blocks, into
          // alternating column sets so the copy never overwrites scales in-flight MMAs read
          const uint32_t sfset = (uint32_t)((kb >> 2) & 1) * 4;
          if (FP8 && (kb & 3) == 0) {
            tmem_cp_32x128b_x4(tmem + FD_SFA_COL + sfset, sf_desc(smem_u32(sSFA + stage * FD_SF_BYTES)));
            tmem_cp_32x128b_x4(tmem + FD_SFB_COL + sfset, sf_desc(smem_u32(sSFB + stage * FD_SF_BYTES)));
          }
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const uint64_t bd = sw128_kmajor_desc(b0 + k * 32);
            const uint32_t accum = (kb | k) != 0;
#pragma unroll
            for (int t = 0; t < 2; ++t) {
              const uint64_t ad = sw128_kmajor_desc(a0 + t * 128 * 128 + k * 32);
              if (FP8)
                mma_mxf8(tmem + FD_ACCA + t * 16, ad, bd, idesc_mxf8(128, FD_N, kb & 3, kb & 3), accum,
                         tmem + FD_SFA_COL + sfset, tmem + FD_SFB_COL + sfset);
              else
                mma_bf16(tmem + FD_ACCA + t * 16, ad, bd, idesc_bf16(128, FD_N), accum);
            }
          }
          mma_commit(&empty[stage]);
          if (kb == KA - 1) mma_commit(accA_full);
        }
        __syncwarp();
        if (++stage == FD_STAGES) { stage = 0; phase ^= 1; }
      }
      // phase B: B operand = h_c in shared memory
      mbar_wait(h_ready, hph);
      hph ^= 1;
      tc_fence_after();
      const uint32_t h0 = smem_u32(sH);
      for (int n = 0; n < NT; ++n) {
        mbar_wait(&accB_empty[ab], abph ^ 1);
        tc_fence_after();
        for (int kk = 0; kk < KBC; ++kk) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          if (lane == 0) {
            const uint32_t a0 = smem_u32(sA + stage * FD_A_BYTES);
#pragma unroll
            for (int k = 0; k < 4; ++k) {
              const uint64_t bd = sw128_kmajor_desc(h0 + kk * FD_B_BYTES + k * 32);
              const uint32_t accum = (kk | k) != 0;
#pragma unroll
              for (int t = 0; t < 2; ++t) {
                const uint64_t ad = sw128_kmajor_desc(a0 + t * 128 * 128 + k * 32);
                const uint32_t d = tmem + FD_ACCB_COL + ab * 32 + t * 16;
                if (FP8) mma_f8(d, ad, bd, idesc_f8(128, FD_N), accum);
                else mma_bf16(d, ad, bd, idesc_bf16(128, FD_N), accum);
              }
            }
            mma_commit(&empty[stage]);
            if (kk == KBC - 1) mma_commit(&accB_full[ab]);
          }
          __syncwarp();
          if (++stage == FD_STAGES) { stage = 0; phase ^= 1; }
        }
        if (++ab == FD_ACCB) { ab = 0; abph ^= 1; }
      }
    }
  } else {
    // ============================ epilogue (4 warps, lanes = weight rows) ============================
    const int q = warp & 3;
    const int qg = q >> 1;
    const uint32_t lane_base = (uint32_t)(q * 32) << 16;
    uint32_t qs = 0, qph = 0, aph = 0;
    int ab = 0; uint32_t abph = 0;
    int ui_par = 0;
    // MOE_DEBUG_TRACE: per-CTA timeline (globaltimer ns) into p.trace[8 + 8 * cta ..] (timing experiments)
    unsigned long long *tr = (p.trace && warp == 2 && lane == 0) ? p.trace + 8 + 8 * blockIdx.x : nullptr;
    if (tr) {
      tr[0] = gtimer();
      unsigned smid;
      asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
      tr[7] = smid;
    }
    pdl_wait();
    if (tr) tr[1] = gtimer();                                  // routing results (tokens, weights) of the route kernel
    for (;;) {
      mbar_wait(&uq_full[qs], qph);
      const int4 uq = unit_q[qs];
      __syncwarp();
      if (lane == 0) mbar_arrive(&uq_empty[qs]);
      if (++qs == FD_UQ) { qs = 0; qph ^= 1; }
      if (!(uq.w >> 1)) break;
      const int group = uq.w & 1, expert = uq.x, row0 = uq.y, n = uq.z & 0xFFFF, chunk = uq.z >> 16;
      // lane t < n: token t -> destination row of the fp32 sums and its weight (routed:
      // only if the token chose this expert; canonical slot i >= n_imm -> deferred sum)
      float *dst_j = nullptr;
      float w_j = 0.f;
      if (lane < n) {
        if (group) {
          dst_j = p.acc_imm + (size_t)lane * p.H;
          w_j = p.sgate ? p.sgate[lane] : 1.f;
        } else {
          const int ge = expert + p.e0;
          int hit = -1;
          for (int i = 0; i < p.k; ++i) hit = (hit < 0 && p.topk_idx[lane * p.k + i] == ge) ? i : hit;
          if (hit >= 0) {
            w_j = p.topk_w[lane * p.k + hit];
            dst_j = (hit < p.n_imm ? p.acc_imm : p.acc_def) + (size_t)lane * p.H;
          }
        }
      }
      const unsigned tmask = __ballot_sync(0xffffffffu, dst_j != nullptr);
      (void)row0;
      // ---- phase A epilogue: SwiGLU + requant -> h_c (B operand of phase B) ----
      if (tr) { tr[2] = gtimer(); tr[6] = (unsigned long long)(group << 30 | expert << 16 | chunk); }
      mbar_wait(accA_full, aph);
      if (tr) tr[3] = gtimer();
      aph ^= 1;
      tc_fence_after();
      uint32_t r0[16], r1[16];
      tmem_ld_32x32b_x16(tmem + lane_base + FD_ACCA, r0);
      tmem_ld_32x32b_x16(tmem + lane_base + FD_ACCA + 16, r1);
      tmem_ld_wait();
      tc_fence_before();
      float *xb = xch + qg * (2 * FD_N * 32);
      if (q & 1) {
#pragma unroll
        for (int t = 0; t < FD_N; ++t) {
          xb[t * 32 + lane] = __uint_as_float(r0[t]);
          xb[(FD_N + t) * 32 + lane] = __uint_as_float(r1[t]);
        }
      }
      asm volatile("bar.sync 1, 128;" ::: "memory");
      const int f0 = qg * 32 + lane;             // h column within the chunk (accumulator 1: + 64)
      if (!(q & 1)) {
        float h0[FD_N], h1[FD_N];
#pragma unroll
        for (int t = 0; t < FD_N; ++t) {
          h0[t] = t < n ? silu_f(__uint_as_float(r0[t])) * xb[t * 32 + lane] : 0.f;
          h1[t] = t < n ? silu_f(__uint_as_float(r1[t])) * xb[(FD_N + t) * 32 + lane] : 0.f;
        }
        if (FP8) {
#pragma unroll
          for (int t = 0; t < FD_N; ++t) {
            const float m = warp_max(fmaxf(fabsf(h0[t]), fabsf(h1[t])));
            if (lane == 0) amax[qg * FD_N + t] = m;
          }
          asm volatile("bar.sync 2, 64;" ::: "memory");   // the two gate warps
#pragma unroll
          for (int t = 0; t < FD_N; ++t) {
            const int e = ue8m0_exponent(fmaxf(amax[t], amax[FD_N + t]));
            const float inv = exp2i(-e);
            uint8_t *row = sH + t * 128;
            row[(((f0 >> 4) ^ (t & 7)) << 4) | (f0 & 15)] = f32_to_e4m3(h0[t] * inv);
            const int f1 = f0 + 64;
            row[(((f1 >> 4) ^ (t & 7)) << 4) | (f1 & 15)] = f32_to_e4m3(h1[t] * inv);
            if (qg == 0 && lane == 0) hsc[ui_par * FD_N + t] = exp2i(e);
          }
        } else {
          // two 64-column k-blocks of bf16: column f0 -> block 0, f0 + 64 -> block 1 (same in-block column)
#pragma unroll
          for (int t = 0; t < FD_N; ++t) {
            const int off = t * 128 + ((((f0 >> 3) ^ (t & 7)) << 4) | ((f0 & 7) << 1));
            *reinterpret_cast<__nv_bfloat16 *>(sH + off) = __float2bfloat16_rn(h0[t]);
            *reinterpret_cast<__nv_bfloat16 *>(sH + FD_B_BYTES + off) = __float2bfloat16_rn(h1[t]);
          }
        }
        fence_proxy_async_smem();                 // generic-proxy h writes -> the MMA's async-proxy reads
      }
      asm volatile("bar.sync 1, 128;" ::: "memory");
      if (q == 0 && lane == 0) mbar_arrive(h_ready);
      if (tr) tr[4] = gtimer();
      // ---- phase B epilogue: scaled, weighted partial sums of W2 row tiles ----
      const FdGroup &g = p.g[group];
      const int nchg = p.nch[group];
      // the unit's W2 block scales (H/128 <= 64 row blocks) into registers up front:
      // a global load per tile would put HBM latency on the epilogue's critical path
      float s2a = 1.f, s2b = 1.f;
      if (FP8) {
        const float *w2s = g.w2_s + (size_t)expert * (p.H / 128) * nchg + chunk;
        if (lane < p.H / 128) s2a = w2s[(size_t)lane * nchg];
        if (lane + 32 < p.H / 128) s2b = w2s[(size_t)(lane + 32) * nchg];
      }
      for (int nt = 0; nt < NT; ++nt) {
        mbar_wait(&accB_full[ab], abph);
        tc_fence_after();
        uint32_t v0[16], v1[16];
        tmem_ld_32x32b_x16(tmem + lane_base + FD_ACCB_COL + ab * 32, v0);
        tmem_ld_32x32b_x16(tmem + lane_base + FD_ACCB_COL + ab * 32 + 16, v1);
        tmem_ld_wait();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&accB_empty[ab]);
        if (++ab == FD_ACCB) { ab = 0; abph ^= 1; }
        const int rA = nt * 256 + q * 32 + lane, rB = rA + 128;
        float sA_ = 1.f, sB_ = 1.f;
        if (FP8) {
          const int rb = 2 * nt;                  // row blocks rb, rb + 1 (warp-uniform)
          sA_ = __shfl_sync(0xffffffffu, rb < 32 ? s2a : s2b, rb & 31);
          sB_ = __shfl_sync(0xffffffffu, rb + 1 < 32 ? s2a : s2b, (rb + 1) & 31);
        }
#pragma unroll
        for (int t = 0; t < FD_N; ++t) {
          if ((tmask >> t) & 1u) {
            float *d = reinterpret_cast<float *>(
                __shfl_sync(0xffffffffu, (unsigned long long)reinterpret_cast<uintptr_t>(dst_j), t));
            const float wt = __shfl_sync(0xffffffffu, w_j, t) * (FP8 ? hsc[ui_par * FD_N + t] : 1.f);
            atomicAdd(d + rA, __uint_as_float(v0[t]) * (sA_ * wt));
            atomicAdd(d + rB, __uint_as_float(v1[t]) * (sB_ * wt));
          }
        }
      }
      ui_par ^= 1;
      if (tr) tr[5] = gtimer();
    }
  }
  // only now may the finalize kernel launch: its CTAs wait in griddepcontrol.wait, which
  // takes issue slots from a co-resident CTA still streaming (measured: a 2.4 us SwiGLU
  // epilogue stretched to 14.5 us on an SM shared with a waiting finalize CTA)
  pdl_trigger();
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc(tmem, FD_TMEM_COLS);
  __shared__ int last_cta;
  if (threadIdx.x == 0) {
    // the last CTA out re-arms the work counter for the next forward (graph replay)
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
    last_cta = atomicAdd(p.done, 1) == (int)gridDim.x - 1;
    if (last_cta) {
      asm volatile("fence.acq_rel.gpu;" ::: "memory");
      atomicExch(p.sched, 0);
      atomicExch(p.done, 0);
    }
  }
}

__global__ void decode_finalize_kernel(const __grid_constant__ DecodeFinalizeArgs a) {
  pdl_trigger();                                 // the next layer's router may start loading its weights
  pdl_wait();
  if (a.trace && blockIdx.x == 0 && threadIdx.x == 0) a.trace[2000] = gtimer();
  decode_finalize_range(a, (int64_t)blockIdx.x * blockDim.x + threadIdx.x, (int64_t)gridDim.x * blockDim.x);
  if (a.trace && blockIdx.x == 0 && threadIdx.x == 0) a.trace[2001] = gtimer();
}

template <bool FP8>
static cudaError_t fd_launch(const FusedDecodeParams &p, int grid, cudaStream_t st) {
  auto k = umma_decode_fused_kernel<FP8>;
  cudaError_t e = set_kernel_attr((const void *)k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)FD_SMEM);
  if (e != cudaSuccess) return e;
  return launch_pdl(k, dim3(grid), dim3(FD_THREADS), FD_SMEM, st, p);
}

cudaError_t launch_umma_decode_fused(bool fp8, const FusedDecodeParams &p, int grid, cudaStream_t st) {
  if (grid <= 0) return cudaSuccess;
  return fp8 ? fd_launch<true>(p, grid, st) : fd_launch<false>(p, grid, st);
}

cudaError_t launch_decode_finalize(const DecodeFinalizeArgs &a, cudaStream_t st) {
  const int64_t n8 = (int64_t)a.T * a.H / 8;
  if (n8 <= 0) return cudaSuccess;
  const int grid = (int)std::min<int64_t>((n8 + 255) / 256, 148);
  return launch_pdl(decode_finalize_kernel, dim3(grid), dim3(256), 0, st, a);
}

}  // namespace moe
