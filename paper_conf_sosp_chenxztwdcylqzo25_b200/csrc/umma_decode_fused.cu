// umma_decode_fused.cu -- decode expert FFNs as ONE weight stream per unit.
//
// Decode (<= 16 tokens per expert) is HBM-bound: every
// active expert's W13 and W2 must stream through once.  A unit is (expert,
// 128-column chunk c of its FFN dimension):
//   phase A: stream the 256-row W13 tile c (gate + up rows of h columns
//            128c .. 128c+127, all H) through the swap-AB MMA (weights = the
//            M = 128 operand, the <= 16 token rows the N = 16 operand).
//            FP8: UNSCALED kind::f8f6f4 MMAs, one 128-K k-block per TMEM
//            accumulator slot of a 4-slot ring; the epilogue folds each slot
//            into fp32 registers with the k-block's 128x128 weight-block scale
//            x the token's 1x128 activation scale (the same products and
//            scales as the block-scaled MMA, summed per k-block -- reading
//            R23), so the MMA issue rate is the unscaled one (~75 vs ~117
//            cycles per 128x16x32 MMA, profiles/r01/mma_single_micro.txt).
//            Then SwiGLU from fp32, FP8: 1x128 UE8M0 requant of h -- exactly
//            the 128-column block of R10/R11, so the scale is local to the
//            unit -- written into shared memory as phase B's B operand (SW128
//            K-major image, no HBM round trip).  BF16: one kind::f16
//            accumulator over all of K.
//   phase B: stream W2[:, 128c .. 128c+127] (H/256 tiles of 256 rows x 128 B)
//            against h_c: one k-block per 128-row M tile, unscaled MMA, the W2
//            block scale x the h scale x the routing weight applied in the
//            epilogue, which red.adds into fp32 [T, H] sums (PAPER.md
//            L219-241) -- the k-sum over chunks and the weighted combine over a
//            token's experts (L187) happen in the same adds.
// Operand groups: 0 = this layer's routed experts, 1 = the shared expert,
// 2 = the PREVIOUS layer's deferred experts (Expert Deferral, PAPER.md L241:
// R^def_{k-1}(I_{k-1}) joins O_k).  Group-2 units depend only on the previous
// layer's routing and activations, which are complete when this kernel starts,
// so they are claimed first and stream while this layer's router is still
// running; every role waits for the router (griddepcontrol.wait) only when it
// reaches its first group-0/1 unit.  Units are claimed from a device counter
// (the L181 dynamic task queue): group 2, then the shared expert's chunks,
// then the routed experts (ascending id).  The weight stream uses an
// evict-first L2 policy.  decode_finalize_kernel adds the residual / deferred
// input, writes bf16 y (and deferred_out) and re-zeroes the sums.
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

constexpr int FD_N = 16, FD_STAGES = 5, FD_THREADS = 192, FD_UQ = 4, FD_ACCB = 4, FD_ACCA_SLOTS = 4;
static_assert(FD_STAGES > FD_ACCA_SLOTS, "phase-A epilogue waits on the stage barriers (no parity aliasing)");
constexpr int FD_A_BYTES = 256 * 128;          // one 256-row weight tile k-block (two 128-row MMA tiles)
constexpr int FD_B_BYTES = FD_N * 128;         // 16 token rows x 128 B
constexpr int FD_H_BYTES = 2 * FD_B_BYTES;     // h_c: FP8 one k-block, BF16 two
constexpr int FD_MAX_KB = 64;                  // H <= 8192: FP8 k-blocks of W13
constexpr size_t FD_SMEM = 1024 + (size_t)FD_STAGES * (FD_A_BYTES + FD_B_BYTES) + FD_H_BYTES +
                           2 * 2 * FD_N * 32 * 4 +     // up -> gate exchange [gate warp][acc][token][lane]
                           2 * 2 * FD_N * 32 * 4 +     // gate values, then h, [gate warp][acc][token][lane]
                           2 * FD_MAX_KB * FD_N * 4 +  // activation scales [this layer | previous layer][kb][token]
                           1024;                       // barriers, queue, amax, scales
constexpr uint32_t FD_TMEM_COLS = 256;
constexpr uint32_t FD_ACCA_COL = 0, FD_ACCB_COL = 128;   // + 32 per ring slot (two 16-column MMA tiles)
static_assert(FD_ACCA_SLOTS * 32 <= (int)FD_ACCB_COL && FD_ACCB_COL + FD_ACCB * 32 <= FD_TMEM_COLS, "TMEM map");

// instruction descriptor, kind::f8f6f4 (A E4M3 or E2M1 (a_fmt 5), B E4M3 -> F32, no block scale), K-major A and B
__host__ __device__ constexpr uint32_t idesc_f8(int M, int N, uint32_t a_fmt = 0) {
  return (1u << 4) | (a_fmt << 7) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
// TMA tile load with an L2 cache-policy hint (FP4 weights: unpacked to 16-byte
// aligned 4-bit groups in shared memory by the tensor map's 16U4_ALIGN16B type)
__device__ __forceinline__ void tma_load_2d_hint(void *dst, const void *map, uint64_t *bar, int c0, int c1, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%2, %3}], [%4], %5;" ::
          "r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
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
// fire-and-forget fp32 add to global memory.  (atomicAdd through a pointer that came out
// of a shuffle compiles to a generic-space ATOM with a returned value plus a shared-memory
// CAS fallback -- measured 3x slower for the phase-B epilogue)
__device__ __forceinline__ void red_add_global(float *p, float v) {
  asm volatile("red.global.add.f32 [%0], %1;" ::"l"(__cvta_generic_to_global(p)), "f"(v) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// 128-column chunks of a group this kernel streams
__device__ __forceinline__ int fd_units_per_expert(const FdGroup &g) { return g.nch; }

// cluster split: the peers' fp32 partials fit the leader's 8 KB exchange buffer
// ((csize - 1) peers x 128 threads x 2T floats) -> st.async into its shared memory
__device__ __forceinline__ bool fd_dsmem_partials(uint32_t csize, int T) { return (int)(csize - 1) * T <= 8; }

// unit -> (valid, group, expert, chunk).  Group 2 first (no dependency on this
// layer's router), then the shared expert (group 1), then the routed experts.
struct FdUnit {
  int valid, group, expert, chunk;
};
__device__ __forceinline__ int fd_prev_units(const FusedDecodeParams &p) {
  return p.has_prev ? (*p.g[2].n_list) * p.g[2].nch : 0;
}
// this layer's units (valid only after griddepcontrol.wait: n_list is the router's)
__device__ __forceinline__ FdUnit fd_unit(const FusedDecodeParams &p, int u, int n_prev) {
  FdUnit r{};
  if (u < n_prev) {
    const FdGroup &g = p.g[2];
    r.valid = 1; r.group = 2; r.expert = g.list[u / g.nch]; r.chunk = u % g.nch;
    return r;
  }
  u -= n_prev;
  const int ns = p.has_shared ? p.g[1].nch : 0;
  if (u < ns) {
    r.valid = 1; r.group = 1; r.expert = 0; r.chunk = u;
    return r;
  }
  u -= ns;
  const FdGroup &g = p.g[0];
  const int slot = u / g.nch;
  if (slot >= *g.n_list) return r;
  r.valid = 1; r.group = 0; r.expert = g.list[slot]; r.chunk = u % g.nch;
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

// W4: 4-bit (e2m1) expert weights -- streamed packed (half the bytes), unpacked by the
// TMA into the e4m3 tile geometry, consumed by the same kind::f8f6f4 MMA (A = E2M1)
template <bool FP8, bool W4>
__global__ void __launch_bounds__(FD_THREADS, 1) umma_decode_fused_kernel(const __grid_constant__ FusedDecodeParams p) {
  static_assert(!W4 || FP8, "4-bit weights take e4m3 activations");
  constexpr uint32_t A_TX = W4 ? FD_A_BYTES / 2 : FD_A_BYTES;   // global bytes of one weight k-block
  constexpr uint32_t A_FMT = W4 ? 5u : 0u;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t *sA = smem;
  uint8_t *sH = sA + FD_STAGES * FD_A_BYTES;                 // 1024-aligned
  uint8_t *sB = sH + FD_H_BYTES;
  float *xch = reinterpret_cast<float *>(sB + FD_STAGES * FD_B_BYTES);   // [2][2][16][32]
  float *xs_s = xch + 2 * 2 * FD_N * 32;                     // [2: this layer, previous layer][FD_MAX_KB][16]
  float *gbuf = xs_s + 2 * FD_MAX_KB * FD_N;                 // [2][2][16][32] gate values -> h (SwiGLU)
  uint64_t *full = reinterpret_cast<uint64_t *>(gbuf + 2 * 2 * FD_N * 32);
  uint64_t *empty = full + FD_STAGES;
  uint64_t *accA_full = empty + FD_STAGES;                   // [FD_ACCA_SLOTS]
  uint64_t *accA_empty = accA_full + FD_ACCA_SLOTS;          // [FD_ACCA_SLOTS]
  uint64_t *h_ready = accA_empty + FD_ACCA_SLOTS;
  uint64_t *accB_full = h_ready + 1;                         // [FD_ACCB]
  uint64_t *accB_empty = accB_full + FD_ACCB;                // [FD_ACCB]
  uint64_t *uq_full = accB_empty + FD_ACCB;                  // [FD_UQ]
  uint64_t *uq_empty = uq_full + FD_UQ;                      // [FD_UQ]
  uint64_t *part_bar = uq_empty + FD_UQ;                     // cluster leader: the peers' partials are in L2
  uint32_t *tmem_base_smem = reinterpret_cast<uint32_t *>(part_bar + 1);
  int4 *unit_q = reinterpret_cast<int4 *>((reinterpret_cast<uintptr_t>(tmem_base_smem + 1) + 15) & ~uintptr_t(15));   // [FD_UQ] (expert, chunk, group, valid)
  float *amax = reinterpret_cast<float *>(unit_q + FD_UQ);       // [2 gate warps][16]
  float *hsc = amax + 2 * FD_N;                                  // [2 unit parity][16] h scale per token (FP8)

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // Cluster split (csize > 1, few units: expert TP, small layers): the csize CTAs of a
  // cluster share one unit -- CTA r streams W13 k-blocks [r KA / csize, (r+1) KA / csize)
  // and W2 tiles [r NT / csize, ...); the peers' fp32 gate/up partials are summed by the
  // leader (rank 0) through L2, which computes SwiGLU + requant and pushes h_c (and its
  // scales) into every peer's shared memory with st.async.  The leader claims the units
  // and forwards them to the peers' queues.
  const uint32_t csize = cluster_size(), crank = cluster_rank();
  const bool leader = crank == 0;
  if (warp == 0 && lane == 0) {
    for (int s = 0; s < FD_STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    for (int s = 0; s < FD_ACCA_SLOTS; ++s) { mbar_init(&accA_full[s], 1); mbar_init(&accA_empty[s], 4); }
    mbar_init(h_ready, 1);
    for (int s = 0; s < FD_ACCB; ++s) { mbar_init(&accB_full[s], 1); mbar_init(&accB_empty[s], 4); }
    // a queue slot is free when the MMA warp and the 4 epilogue warps here and the
    // producer, MMA and epilogue warps of every peer have read it
    for (int i = 0; i < FD_UQ; ++i) { mbar_init(&uq_full[i], 1); mbar_init(&uq_empty[i], 5 + 6 * (csize - 1)); }
    // partials through the leader's shared memory (st.async; small T) or through L2
    mbar_init(part_bar, (csize > 1 && !fd_dsmem_partials(csize, p.T)) ? 4 * (csize - 1) : 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc(tmem_base_smem, FD_TMEM_COLS);
  tc_fence_before();
  __syncthreads();
  if (csize > 1) cluster_sync();                 // every barrier of the cluster initialised
  tc_fence_after();
  const uint32_t tmem = *tmem_base_smem;

  constexpr int KDIV = FP8 ? 128 : 64;           // elements per 128-byte k-block
  constexpr int KBC = 128 / KDIV;                // W2 k-blocks per 128-column chunk
  const int KA = p.H / KDIV;                     // W13 k-blocks
  const int NT = p.H / 256;                      // W2 256-row tiles
  const int kb0 = (int)(crank * KA / csize), kb1 = (int)((crank + 1) * KA / csize);   // this CTA's share
  const int nt0 = (int)(crank * NT / csize), nt1 = (int)((crank + 1) * NT / csize);
  // a consumer is done with queue slot qs (the leader's barrier counts the whole cluster)
  auto release_slot = [&](int qs_) {
    if (leader) mbar_arrive(&uq_empty[qs_]);
    else mbar_arrive_remote(map_to_rank(&uq_empty[qs_], 0));
  };

  if (warp == 0) {
    // ============================ producer ============================
    if (lane == 0) {
      const int n_prev = fd_prev_units(p);       // the previous layer's routing is complete
      bool waited = false;
      const uint64_t pol = l2_evict_first_policy();   // weights are read once per forward
      int stage = 0; uint32_t phase = 0, qs = 0, qph = 0;
      for (;;) {
        FdUnit ui;
        if (leader) {
          const int u = atomicAdd(p.sched, 1);
          if (u >= n_prev && !waited) {
            pdl_wait();                          // this layer's routing and xq (route kernel)
            waited = true;
          }
          ui = fd_unit(p, u, n_prev);
          mbar_wait(&uq_empty[qs], qph ^ 1);
          unit_q[qs] = make_int4(ui.expert, ui.chunk, ui.group, ui.valid);
          mbar_arrive(&uq_full[qs]);
          for (uint32_t r = 1; r < csize; ++r) {   // forward the unit to the peers
            const uint32_t pbar = map_to_rank(&uq_full[qs], r);
            mbar_arrive_expect_tx_remote(pbar, 16);
            st_async_v4u32(map_to_rank(&unit_q[qs], r),
                           make_uint4((uint32_t)ui.expert, (uint32_t)ui.chunk, (uint32_t)ui.group, (uint32_t)ui.valid),
                           pbar);
          }
        } else {
          mbar_wait(&uq_full[qs], qph);
          const int4 q4 = unit_q[qs];
          release_slot(qs);
          ui.expert = q4.x; ui.chunk = q4.y; ui.group = q4.z; ui.valid = q4.w;
          if (ui.valid && ui.group != 2 && !waited) {
            pdl_wait();                          // this layer's xq (TMA-loaded below)
            waited = true;
          }
        }
        if (++qs == FD_UQ) { qs = 0; qph ^= 1; }
        if (!ui.valid) {
          // every load of this CTA is issued: let the finalize kernel launch now, so
          // its launch latency overlaps the last stages (it waits for our completion)
          pdl_trigger();
          break;
        }
        const FdGroup &g = p.g[ui.group];
        // ---- phase A: W13 tile `chunk` (256 rows: gate + up of 128 h columns) ----
        const uint8_t *w13 = g.w13 + ((size_t)ui.expert * g.nch + ui.chunk) * (size_t)KA * FD_A_BYTES;
        for (int kb = kb0; kb < kb1; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          mbar_expect_tx(&full[stage], A_TX + FD_B_BYTES);
          if (W4)
            tma_load_2d_hint(sA + stage * FD_A_BYTES, &g.w13_map4, &full[stage], kb * 128,
                             (ui.expert * g.nch + ui.chunk) * 256, pol);
          else
            bulk_load_hint(sA + stage * FD_A_BYTES, w13 + (size_t)kb * FD_A_BYTES, FD_A_BYTES, &full[stage], pol);
          tma_load_2d(sB + stage * FD_B_BYTES, &g.x_map, &full[stage], kb * KDIV, 0);
          if (++stage == FD_STAGES) { stage = 0; phase ^= 1; }
        }
        // ---- phase B: W2 column block `chunk`, H/256 tiles of 256 rows ----
        const int KB2 = g.nch * KBC;               // W2 k-blocks per tile row
        const uint8_t *w2 = g.w2 + (size_t)ui.expert * NT * KB2 * FD_A_BYTES;
        for (int n = nt0; n < nt1; ++n) {
          for (int kk = 0; kk < KBC; ++kk) {
            mbar_wait(&empty[stage], phase ^ 1);
            mbar_expect_tx(&full[stage], A_TX);
            if (W4)
              tma_load_2d_hint(sA + stage * FD_A_BYTES, &g.w2_map4, &full[stage], ui.chunk * 128,
                               ui.expert * p.H + n * 256, pol);
            else
              bulk_load_hint(sA + stage * FD_A_BYTES, w2 + ((size_t)n * KB2 + ui.chunk * KBC + kk) * FD_A_BYTES,
                             FD_A_BYTES, &full[stage], pol);
            if (++stage == FD_STAGES) { stage = 0; phase ^= 1; }
          }
        }
      }
    }
  } else if (warp == 1) {
    // ============================ MMA issuer ============================
    // (touches only shared memory and TMEM: no griddepcontrol.wait needed)
    int stage = 0; uint32_t phase = 0, qs = 0, qph = 0, hph = 0;
    int ab = 0; uint32_t abph = 0;
    int as = 0; uint32_t asph = 0;
    for (;;) {
      mbar_wait(&uq_full[qs], qph);
      const int4 uq = unit_q[qs];
      __syncwarp();
      if (lane == 0) release_slot(qs);
      if (++qs == FD_UQ) { qs = 0; qph ^= 1; }
      if (!uq.w) break;
      // ---- phase A ----
      for (int kb = kb0; kb < kb1; ++kb) {
        if (kExperiments && (p.debug & 2)) {     // timing experiment: phase-A loads only (no MMAs)
          if (FP8) mbar_wait(&accA_empty[as], asph ^ 1);
          mbar_wait(&full[stage], phase);
          if (lane == 0) {
            mbar_arrive(&empty[stage]);
            if (!FP8 && kb == kb1 - 1) mbar_arrive(&accA_full[0]);
          }
          __syncwarp();
          if (++stage == FD_STAGES) { stage = 0; phase ^= 1; }
          if (FP8 && ++as == FD_ACCA_SLOTS) { as = 0; asph ^= 1; }
          continue;
        }
        if (FP8) {                               // this k-block's accumulator slot is free
          mbar_wait(&accA_empty[as], asph ^ 1);
          tc_fence_after();
        }
        mbar_wait(&full[stage], phase);
        tc_fence_after();
        if (lane == 0) {
          const uint32_t a0 = smem_u32(sA + stage * FD_A_BYTES);
          const uint32_t b0 = smem_u32(sB + stage * FD_B_BYTES);
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const uint64_t bd = sw128_kmajor_desc(b0 + k * 32);
#pragma unroll
            for (int t = 0; t < 2; ++t) {
              const uint64_t ad = sw128_kmajor_desc(a0 + t * 128 * 128 + k * 32);
              if (FP8)     // a fresh accumulator slot per k-block
                mma_f8(tmem + FD_ACCA_COL + as * 32 + t * 16, ad, bd, idesc_f8(128, FD_N, A_FMT), k != 0);
              else         // the accumulator is free: the epilogue read it before h_ready of the previous unit
                mma_bf16(tmem + FD_ACCA_COL + t * 16, ad, bd, idesc_bf16(128, FD_N), (kb != kb0) || (k != 0));
            }
          }
          // FP8: one commit per k-block serves the producer (stage free) and the epilogue
          // (slot `as` complete) -- a tcgen05.commit costs the tensor pipe ~100 cycles
          // (profiles/r02/mma_ring.txt), so the second commit per k-block was a bubble
          mma_commit(&empty[stage]);
          if (!FP8 && kb == kb1 - 1) mma_commit(&accA_full[0]);
        }
        __syncwarp();
        if (++stage == FD_STAGES) { stage = 0; phase ^= 1; }
        if (FP8 && ++as == FD_ACCA_SLOTS) { as = 0; asph ^= 1; }
      }
      // ---- phase B: B operand = h_c in shared memory ----
      mbar_wait(h_ready, hph);
      hph ^= 1;
      fence_proxy_async_smem();                  // a peer's h_c arrived by st.async
      tc_fence_after();
      const uint32_t h0 = smem_u32(sH);
      for (int n = nt0; n < nt1; ++n) {
        mbar_wait(&accB_empty[ab], abph ^ 1);
        tc_fence_after();
        for (int kk = 0; kk < KBC; ++kk) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          if (kExperiments && (p.debug & 8)) {   // timing experiment: phase-B loads only (no MMAs)
            if (lane == 0) {
              mbar_arrive(&empty[stage]);
              if (kk == KBC - 1) mbar_arrive(&accB_full[ab]);
            }
            __syncwarp();
            if (++stage == FD_STAGES) { stage = 0; phase ^= 1; }
            continue;
          }
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
                if (FP8) mma_f8(d, ad, bd, idesc_f8(128, FD_N, A_FMT), accum);
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
    const int et = threadIdx.x - 64;             // 0..127
    const uint32_t lane_base = (uint32_t)(q * 32) << 16;
    uint32_t qs = 0, qph = 0, aph = 0;
    int ab = 0; uint32_t abph = 0;
    int as = 0; uint32_t asph = 0;
    int es = 0; uint32_t eph = 0;                // FP8: the smem stage ring, followed (phase A waits)
    int ui_par = 0;
    uint32_t hph_e = 0, pph = 0;                 // cluster peers: h_ready phase; leader: part_bar phase
    bool waited = false;
    // MOE_DEBUG_TRACE: per-CTA timeline (globaltimer ns) into p.trace[8 + 8 * cta ..] (timing experiments)
    unsigned long long *tr = (p.trace && warp == 2 && lane == 0) ? p.trace + 8 + 8 * blockIdx.x : nullptr;
    if (tr) {
      tr[0] = gtimer();
      unsigned smid;
      asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
      tr[7] = smid;
    }
    // activation scales [kb][token] of a layer into shared memory (FP8; tokens >= T read 0)
    // (every load issued before the first store: one L2 round trip, not KA*16/128 of them --
    //  the phase-A MMAs can run only FD_ACCA_SLOTS k-blocks ahead of this warp group)
    auto load_xs = [&](const float *xs, float *dst) {
      constexpr int NI = FD_MAX_KB * FD_N / 128;
      float v[NI];
#pragma unroll
      for (int j = 0; j < NI; ++j) {
        const int i = et + 128 * j, kb = i / FD_N, t = i % FD_N;
        v[j] = (kb < KA && t < p.T) ? __ldg(xs + (size_t)t * KA + kb) : 0.f;
      }
#pragma unroll
      for (int j = 0; j < NI; ++j) dst[et + 128 * j] = v[j];
    };
    if (FP8 && p.has_prev) load_xs(p.g[2].xs, xs_s + FD_MAX_KB * FD_N);   // previous layer: complete
    asm volatile("bar.sync 3, 128;" ::: "memory");
    for (;;) {
      mbar_wait(&uq_full[qs], qph);
      const int4 uq = unit_q[qs];
      __syncwarp();
      if (lane == 0) release_slot(qs);
      if (++qs == FD_UQ) { qs = 0; qph ^= 1; }
      if (!uq.w) break;
      const int expert = uq.x, chunk = uq.y, group = uq.z;
      if (group != 2 && !waited) {
        pdl_wait();                              // this layer's routing results and activation scales
        if (tr) tr[1] = gtimer();
        if (FP8) load_xs(p.g[0].xs, xs_s);
        asm volatile("bar.sync 3, 128;" ::: "memory");
        waited = true;
      }
      const FdGroup &g = p.g[group];
      const float *xsg = xs_s + (group == 2 ? FD_MAX_KB * FD_N : 0);
      // lane t < T: token t -> destination row of the fp32 sums and its weight.
      // Routed groups: only if the token chose this expert, in a canonical slot of
      // [a0, a1) (-> acc_imm) or [a1, a2) (-> acc_def); shared: every token.
      float *dst_j = nullptr;
      float w_j = 0.f;
      if (lane < p.T) {
        if (group == 1) {
          dst_j = p.acc_imm + (size_t)lane * p.H;
          w_j = p.sgate ? p.sgate[lane] : 1.f;
        } else {
          // all k ids in flight together (a short-circuit scan would serialise k L2 round trips)
          const int ge = expert + g.e0;
          int ids[32];
#pragma unroll
          for (int i = 0; i < 32; ++i) ids[i] = i < g.k ? __ldg(g.topk_idx + lane * g.k + i) : -1;
          int hit = -1;
#pragma unroll
          for (int i = 31; i >= 0; --i) hit = ids[i] == ge ? i : hit;
          if (hit >= g.a0 && hit < g.a2) {
            w_j = g.topk_w[lane * g.k + hit];
            dst_j = (hit < g.a1 ? p.acc_imm : p.acc_def) + (size_t)lane * p.H;
          }
        }
      }
      const unsigned tmask = __ballot_sync(0xffffffffu, dst_j != nullptr);
      // ---- phase A epilogue: fp32 gate/up accumulators of this lane's two weight rows ----
      if (tr) { tr[2] = gtimer(); tr[6] = (unsigned long long)(group << 30 | expert << 16 | chunk); }
      float r0[FD_N], r1[FD_N];
      if constexpr (FP8) {
        // 128x128 weight-block scales of this warp's rows (gate or up rows of h block
        // `chunk`, interleaved per 128 rows: row block 2 chunk + (q & 1)), all k-blocks
        const float *ws = g.w13_s + ((size_t)expert * 2 * g.nch + 2 * chunk + (q & 1)) * KA;
        const float swa = lane < KA ? ws[lane] : 0.f, swb = lane + 32 < KA ? ws[lane + 32] : 0.f;
#pragma unroll
        for (int t = 0; t < FD_N; ++t) r0[t] = r1[t] = 0.f;
        for (int kb = kb0; kb < kb1; ++kb) {
          // the k-block's MMAs are complete when its smem stage is released (the MMA warp's
          // single commit per k-block); this warp group follows the stage ring: phase A takes
          // one stage per k-block, phase B (nt1 - nt0) * KBC (advanced below).  No parity
          // aliasing: the stage is reused only FD_STAGES > FD_ACCA_SLOTS k-blocks later, which
          // needs slot `as` released by this warp group first
          mbar_wait(&empty[es], eph);
          if (++es == FD_STAGES) { es = 0; eph ^= 1; }
          tc_fence_after();
          if (kExperiments && (p.debug & 1)) {   // timing experiment: no per-k-block fold
            __syncwarp();
            if (lane == 0) mbar_arrive(&accA_empty[as]);
            if (++as == FD_ACCA_SLOTS) { as = 0; asph ^= 1; }
            continue;
          }
          uint32_t v0[16], v1[16];
          tmem_ld_32x32b_x16(tmem + lane_base + FD_ACCA_COL + as * 32, v0);
          tmem_ld_32x32b_x16(tmem + lane_base + FD_ACCA_COL + as * 32 + 16, v1);
          tmem_ld_wait();
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive(&accA_empty[as]);
          if (++as == FD_ACCA_SLOTS) { as = 0; asph ^= 1; }
          const float sw = __shfl_sync(0xffffffffu, kb < 32 ? swa : swb, kb & 31);
          const float4 *xs4 = reinterpret_cast<const float4 *>(xsg + kb * FD_N);
#pragma unroll
          for (int t4 = 0; t4 < FD_N / 4; ++t4) {
            const float4 x4 = xs4[t4];
            const float sx[4] = {x4.x, x4.y, x4.z, x4.w};
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              const int t = 4 * t4 + j;
              const float s = sw * sx[j];
              r0[t] = fmaf(__uint_as_float(v0[t]), s, r0[t]);
              r1[t] = fmaf(__uint_as_float(v1[t]), s, r1[t]);
            }
          }
        }
      } else {
        mbar_wait(&accA_full[0], aph);
        aph ^= 1;
        tc_fence_after();
        uint32_t v0[16], v1[16];
        tmem_ld_32x32b_x16(tmem + lane_base + FD_ACCA_COL, v0);
        tmem_ld_32x32b_x16(tmem + lane_base + FD_ACCA_COL + 16, v1);
        tmem_ld_wait();
        tc_fence_before();
#pragma unroll
        for (int t = 0; t < FD_N; ++t) { r0[t] = __uint_as_float(v0[t]); r1[t] = __uint_as_float(v1[t]); }
      }
      if (tr) tr[3] = gtimer();
      constexpr uint32_t H_TX = FP8 ? 2 * FD_B_BYTES / 2 + 4 * FD_N : FD_H_BYTES;   // h_c (+ FP8 scales) bytes
      if (csize > 1) {
        // ---- cluster: the peers' partial gate/up sums -> the leader (through L2) ----
        float *scr = p.cl_scratch + (size_t)cluster_id_x() * 7 * 128 * 32;
        const bool dsm = fd_dsmem_partials(csize, p.T);
        if (!leader) {
          if (dsm) {
            // (token t of this thread's two rows) -> the leader's xch [peer][thread][2T]
            float *dst = xch + ((size_t)(crank - 1) * 128 + et) * 2 * p.T;
            const uint32_t bar = map_to_rank(part_bar, 0);
#pragma unroll
            for (int t = 0; t < FD_N; ++t)
              if (t < p.T) st_async_v2f32(map_to_rank(dst + 2 * t, 0), r0[t], r1[t], bar);
          } else {
            float4 *dst = reinterpret_cast<float4 *>(scr + ((size_t)(crank - 1) * 128 + et) * 32);
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              __stcg(dst + j, make_float4(r0[4 * j], r0[4 * j + 1], r0[4 * j + 2], r0[4 * j + 3]));
              __stcg(dst + 4 + j, make_float4(r1[4 * j], r1[4 * j + 1], r1[4 * j + 2], r1[4 * j + 3]));
            }
            __syncwarp();
            if (lane == 0) mbar_arrive_cluster(map_to_rank(part_bar, 0));   // release.cluster
          }
          // h_c of this unit comes from the leader (st.async into sH / hsc, complete_tx on h_ready)
          if (q == 0 && lane == 0) mbar_expect_tx(h_ready, H_TX);
          mbar_wait(h_ready, hph_e);
          hph_e ^= 1;
          if (tr) tr[4] = gtimer();
          goto phase_b;
        }
        unsigned long long *tl = (p.trace && warp == 2 && lane == 0) ? p.trace + 1300 + 4 * blockIdx.x : nullptr;
        if (dsm) {
          if (q == 0 && lane == 0) mbar_expect_tx(part_bar, (csize - 1) * 128 * 2 * p.T * 4);
          mbar_wait_cluster(part_bar, pph);
          if (tl) tl[0] = gtimer();
          pph ^= 1;
          for (uint32_t r = 1; r < csize; ++r) {
            const float *src = xch + ((size_t)(r - 1) * 128 + et) * 2 * p.T;
#pragma unroll
            for (int t = 0; t < FD_N; ++t)
              if (t < p.T) { r0[t] += src[2 * t]; r1[t] += src[2 * t + 1]; }
          }
          asm volatile("bar.sync 1, 128;" ::: "memory");   // xch is the SwiGLU exchange buffer next
        }
        if (!dsm) mbar_wait_cluster(part_bar, pph);
        if (!dsm) pph ^= 1;
        for (uint32_t r = 1; r < (dsm ? 1u : csize); ++r) {
          const float4 *src = reinterpret_cast<const float4 *>(scr + ((size_t)(r - 1) * 128 + et) * 32);
          float4 v[8];
#pragma unroll
          for (int j = 0; j < 8; ++j) v[j] = __ldcg(src + j);
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            r0[4 * j] += v[j].x; r0[4 * j + 1] += v[j].y; r0[4 * j + 2] += v[j].z; r0[4 * j + 3] += v[j].w;
            r1[4 * j] += v[4 + j].x; r1[4 * j + 1] += v[4 + j].y; r1[4 * j + 2] += v[4 + j].z;
            r1[4 * j + 3] += v[4 + j].w;
          }
        }
      }
      {
      unsigned long long *tl = (p.trace && csize > 1 && warp == 2 && lane == 0) ? p.trace + 1300 + 4 * blockIdx.x : nullptr;
      if (tl) tl[1] = gtimer();
      // ---- SwiGLU + requant -> h_c (B operand of phase B) ----
      // The accumulators go to shared memory once (unrolled: one store per live token), then
      // rolled loops over the T live tokens: this code runs once per unit with a cold
      // instruction cache while the weight streams load L2, so its footprint -- not its
      // instruction count -- is what the unit waits for (the 16-way unrolled form with
      // predicated-off token columns measured ~3.5 us here at T = 1).
      float *xb = xch + qg * (2 * FD_N * 32);      // up values
      float *gb = gbuf + qg * (2 * FD_N * 32);     // gate values, then h
      {
        float *dst = (q & 1) ? xb : gb;
#pragma unroll
        for (int t = 0; t < FD_N; ++t) {
          if (t < p.T) {                        // (warp-uniform: token columns >= T are never read)
            dst[t * 32 + lane] = r0[t];
            dst[(FD_N + t) * 32 + lane] = r1[t];
          }
        }
      }
      asm volatile("bar.sync 1, 128;" ::: "memory");
      unsigned long long *tq = (p.trace && csize > 1 && !(q & 1) && lane == 0) ? p.trace + 2100 + 8 * blockIdx.x + 4 * qg : nullptr;
      if (tq) tq[0] = gtimer();
      const int f0 = qg * 32 + lane;             // h column within the chunk (accumulator 1: + 64)
      if (!(q & 1)) {
#pragma unroll 1
        for (int t = 0; t < p.T; ++t) {
          const float h0 = silu_f(gb[t * 32 + lane]) * xb[t * 32 + lane];
          const float h1 = silu_f(gb[(FD_N + t) * 32 + lane]) * xb[(FD_N + t) * 32 + lane];
          gb[t * 32 + lane] = h0;
          gb[(FD_N + t) * 32 + lane] = h1;
          if (FP8) {
            const float m = warp_max(fmaxf(fabsf(h0), fabsf(h1)));
            if (lane == 0) amax[qg * FD_N + t] = m;
          }
        }
        if (tq) tq[1] = gtimer();
        if (FP8) {
          asm volatile("bar.sync 2, 64;" ::: "memory");   // the two gate warps
          if (tq) tq[2] = gtimer();
          const int f1 = f0 + 64;
#pragma unroll 1
          for (int t = 0; t < p.T; ++t) {
            const int e = ue8m0_exponent(fmaxf(amax[t], amax[FD_N + t]));
            const float inv = exp2i(-e);
            uint8_t *row = sH + t * 128;
            row[(((f0 >> 4) ^ (t & 7)) << 4) | (f0 & 15)] = f32_to_e4m3(gb[t * 32 + lane] * inv);
            row[(((f1 >> 4) ^ (t & 7)) << 4) | (f1 & 15)] = f32_to_e4m3(gb[(FD_N + t) * 32 + lane] * inv);
            if (qg == 0 && lane == 0) hsc[ui_par * FD_N + t] = exp2i(e);
          }
        } else {
          // two 64-column k-blocks of bf16: column f0 -> block 0, f0 + 64 -> block 1 (same in-block column)
#pragma unroll 1
          for (int t = 0; t < p.T; ++t) {
            const int off = t * 128 + ((((f0 >> 3) ^ (t & 7)) << 4) | ((f0 & 7) << 1));
            *reinterpret_cast<__nv_bfloat16 *>(sH + off) = __float2bfloat16_rn(gb[t * 32 + lane]);
            *reinterpret_cast<__nv_bfloat16 *>(sH + FD_B_BYTES + off) = __float2bfloat16_rn(gb[(FD_N + t) * 32 + lane]);
          }
        }
        if (tq) tq[3] = gtimer();
        fence_proxy_async_smem();                 // generic-proxy h writes -> the MMA's async-proxy reads
      }
      asm volatile("bar.sync 1, 128;" ::: "memory");
      if (tl) tl[2] = gtimer();
      if (csize > 1) {
        // push h_c (and the FP8 h scales) into every peer's shared memory
        constexpr int HV = (FP8 ? 2 * FD_B_BYTES / 2 : FD_H_BYTES) / 16;   // 16-byte vectors of h_c
        for (int i = et; i < HV; i += 128) {
          const uint4 v = *reinterpret_cast<const uint4 *>(sH + 16 * i);
          for (uint32_t r = 1; r < csize; ++r)
            st_async_v4u32(map_to_rank(sH + 16 * i, r), v, map_to_rank(h_ready, r));
        }
        if (FP8 && et < FD_N / 4) {
          const uint4 v = *reinterpret_cast<const uint4 *>(hsc + ui_par * FD_N + 4 * et);
          for (uint32_t r = 1; r < csize; ++r)
            st_async_v4u32(map_to_rank(hsc + ui_par * FD_N + 4 * et, r), v, map_to_rank(h_ready, r));
        }
      }
      if (q == 0 && lane == 0) mbar_arrive(h_ready);
      if (tr) tr[4] = gtimer();
      if (tl) tl[3] = gtimer();
      }
    phase_b:
      // ---- phase B epilogue: scaled, weighted partial sums of W2 row tiles ----
      // the unit's W2 block scales (H/128 <= 64 row blocks) into registers up front:
      // a global load per tile would put HBM latency on the epilogue's critical path
      float s2a = 1.f, s2b = 1.f;
      if (FP8) {
        const float *w2s = g.w2_s + (size_t)expert * (p.H / 128) * g.nch + chunk;
        if (lane < p.H / 128) s2a = w2s[(size_t)lane * g.nch];
        if (lane + 32 < p.H / 128) s2b = w2s[(size_t)(lane + 32) * g.nch];
      }
      for (int nt = nt0; nt < nt1; ++nt) {
        mbar_wait(&accB_full[ab], abph);
        tc_fence_after();
        if (kExperiments && (p.debug & 4)) {     // timing experiment: no phase-B epilogue work
          __syncwarp();
          if (lane == 0) mbar_arrive(&accB_empty[ab]);
          if (++ab == FD_ACCB) { ab = 0; abph ^= 1; }
          continue;
        }
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
            red_add_global(d + rA, __uint_as_float(v0[t]) * (sA_ * wt));
            red_add_global(d + rB, __uint_as_float(v1[t]) * (sB_ * wt));
          }
        }
      }
      ui_par ^= 1;
      for (int i = (nt1 - nt0) * KBC; i > 0; --i)   // the stages phase B consumed
        if (++es == FD_STAGES) { es = 0; eph ^= 1; }
      if (tr) tr[5] = gtimer();
    }
    if (!waited) pdl_wait();                     // (a CTA that only saw group-2 units: nothing left to read)
  }
  // only now may the finalize kernel launch: its CTAs wait in griddepcontrol.wait, which
  // takes issue slots from a co-resident CTA still streaming (measured: a 2.4 us SwiGLU
  // epilogue stretched to 14.5 us on an SM shared with a waiting finalize CTA)
  pdl_trigger();
  tc_fence_before();
  __syncthreads();
  if (csize > 1) cluster_sync();                 // no CTA leaves while a peer may still st.async into it
  if (warp == 1) tmem_dealloc(tmem, FD_TMEM_COLS);
  if (threadIdx.x == 0) {
    // the last CTA out re-arms the work counter for the next forward (graph replay)
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
    if (atomicAdd(p.done, 1) == (int)gridDim.x - 1) {
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

template <bool FP8, bool W4>
static cudaError_t fd_launch(const FusedDecodeParams &p, int grid, int csize, cudaStream_t st) {
  auto k = umma_decode_fused_kernel<FP8, W4>;
  cudaError_t e = set_kernel_attr((const void *)k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)FD_SMEM);
  if (e == cudaSuccess && csize > 1)
    e = set_kernel_attr((const void *)k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(FD_THREADS);
  cfg.dynamicSmemBytes = FD_SMEM;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  int na = 0;
  attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[na++].val.programmaticStreamSerializationAllowed = 1;
  if (csize > 1) {
    attr[na].id = cudaLaunchAttributeClusterDimension;
    attr[na].val.clusterDim.x = csize;
    attr[na].val.clusterDim.y = 1;
    attr[na++].val.clusterDim.z = 1;
  }
  cfg.attrs = attr;
  cfg.numAttrs = na;
  return cudaLaunchKernelEx(&cfg, k, p);
}

cudaError_t launch_umma_decode_fused(bool fp8, bool w4, const FusedDecodeParams &p, int grid, int csize,
                                     cudaStream_t st) {
  if (grid <= 0) return cudaSuccess;
  if (w4) return fd_launch<true, true>(p, grid, csize, st);
  return fp8 ? fd_launch<true, false>(p, grid, csize, st) : fd_launch<false, false>(p, grid, csize, st);
}

// clusters of `csize` fused-decode CTAs that can be resident at once (0 if none)
int fused_decode_max_clusters(bool fp8, int csize) {
  const void *k = fp8 ? (const void *)umma_decode_fused_kernel<true, false> : (const void *)umma_decode_fused_kernel<false, false>;
  if (set_kernel_attr(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)FD_SMEM) != cudaSuccess) return 0;
  if (csize > 8 && set_kernel_attr(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) != cudaSuccess) return 0;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(csize * 16);
  cfg.blockDim = dim3(FD_THREADS);
  cfg.dynamicSmemBytes = FD_SMEM;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = csize;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, k, &cfg) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return n;
}

cudaError_t launch_decode_finalize(const DecodeFinalizeArgs &a, cudaStream_t st) {
  const int64_t n8 = (int64_t)a.T * a.H / 8;
  if (n8 <= 0) return cudaSuccess;
  const int grid = (int)std::min<int64_t>((n8 + 255) / 256, 148);
  return launch_pdl(decode_finalize_kernel, dim3(grid), dim3(256), 0, st, a);
}

}  // namespace moe
