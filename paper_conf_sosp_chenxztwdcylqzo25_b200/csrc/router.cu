// router.cu -- score + group-limited top-k selection, one warp per token.
//
// PAPER.md L98 (§2.1): the gate "dynamically selects the most relevant experts
// to process each token, usually the top-k or its variants (e.g., grouped
// top-k in DeepSeek-V3/R1)".  Gate rules (reading R1):
//   s = sigmoid(logit) | softmax(logits);  sel = s + bias;
//   groups: keep the topk_group groups with the best max(sel) | top-2 sum(sel),
//           others excluded;  idx = top_k(sel)  (ties -> lower id, reading R2)
//   w = s[idx] (/ sum w if norm_topk) * routed_scale
//   slots written in canonical order: w descending, ties -> lower id (R4)
#include <algorithm>
#include <cub/block/block_scan.cuh>

#include "common.cuh"
#include "kernels.h"

namespace moe {

constexpr int RT_WARPS = 4;

// (v, i) better than (v2, i2): larger value, then smaller index
__device__ __forceinline__ bool better(float v, int i, float v2, int i2) {
  return v > v2 || (v == v2 && i < i2);
}

__device__ __forceinline__ void warp_argmax(float &v, int &i) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    float v2 = __shfl_xor_sync(0xffffffffu, v, o);
    int i2 = __shfl_xor_sync(0xffffffffu, i, o);
    if (better(v2, i2, v, i)) { v = v2; i = i2; }
  }
}

// One warp routes token t (scratch s/sel: 2 x E floats of shared memory).
__device__ void select_token(const RouterArgs &args, int t, float *s, float *sel, int lane) {
  // copy the arguments into registers: the stores below go through generic
  // pointers the compiler cannot prove disjoint from the argument struct, and
  // re-loading the fields in every loop iteration costs ~30x the work
  struct {
    int E, k, n_group, topk_group, group_score, score_fn, norm_topk, shared_gated;
    float routed_scale;
    const float *bias;
    int32_t *topk_idx;
    float *topk_w, *sgate;
  } a = {args.E, args.k, args.n_group, args.topk_group, args.group_score, args.score_fn, args.norm_topk,
         args.shared_gated, args.routed_scale, args.bias, args.topk_idx, args.topk_w, args.sgate};
  const int E = a.E;
  const float *lg = args.logits + (int64_t)t * args.ldl;

  // ---- scores ----
  // (compact rolled loops: this code runs once per token on one warp, so its
  //  instruction footprint -- cold in the i-cache -- sets the latency)
  if (a.score_fn == MOE_SCORE_SOFTMAX) {
    float m = -INFINITY;
#pragma unroll 1
    for (int e = lane; e < E; e += 32) m = fmaxf(m, lg[e]);
    m = warp_max(m);
    float sum = 0.f;
#pragma unroll 1
    for (int e = lane; e < E; e += 32) {
      const float v = expf(lg[e] - m);
      s[e] = v;
      sum += v;
    }
    sum = warp_sum(sum);
#pragma unroll 1
    for (int e = lane; e < E; e += 32) s[e] = s[e] / sum;
  } else {
#pragma unroll 1
    for (int e = lane; e < E; e += 32) s[e] = 1.f / (1.f + expf(-lg[e]));
  }
#pragma unroll 1
  for (int e = lane; e < E; e += 32) sel[e] = s[e] + (a.bias ? a.bias[e] : 0.f);
  __syncwarp();
  // ---- group limit ----
  if (a.n_group > 1) {
    const int G = a.n_group, gs = E / G;
    float gscore = -INFINITY;
    if (lane < G) {
      float m1 = -INFINITY, m2 = -INFINITY;
#pragma unroll 1
      for (int i = 0; i < gs; ++i) {
        float v = sel[lane * gs + i];
        if (v > m1) { m2 = m1; m1 = v; } else if (v > m2) { m2 = v; }
      }
      gscore = (a.group_score == MOE_GROUP_TOP2_SUM) ? (m1 + m2) : m1;
    }
    bool keep = false;
    float gv = (lane < G) ? gscore : -INFINITY;
#pragma unroll 1
    for (int r = 0; r < a.topk_group; ++r) {
      float v = (lane < G && !keep) ? gv : -INFINITY;
      int i = (lane < G && !keep) ? lane : 0x7fffffff;
      warp_argmax(v, i);
      if (lane == i) keep = true;
    }
    const unsigned keep_mask = __ballot_sync(0xffffffffu, keep);
#pragma unroll 1
    for (int e = lane; e < E; e += 32)
      if (!((keep_mask >> (e / gs)) & 1u)) sel[e] = -INFINITY;
    __syncwarp();
  }

  // ---- top-k ----
  int my_id = -1;
#pragma unroll 1
  for (int j = 0; j < a.k; ++j) {
    float v = -INFINITY;
    int i = 0x7fffffff;
#pragma unroll 1
    for (int e = lane; e < E; e += 32) {
      const float x = sel[e];
      if (better(x, e, v, i)) { v = x; i = e; }
    }
    warp_argmax(v, i);
    if (lane == j) my_id = i;
    if (lane == (i & 31)) sel[i] = -INFINITY;   // owner lane retires the winner
    __syncwarp();
  }

  // ---- combine weights ----
  float w = (lane < a.k) ? s[my_id] : 0.f;
  if (a.norm_topk) {
    const float sum = warp_sum(w);
    w = w / sum;
  }
  w = w * a.routed_scale;

  // ---- canonical order: w descending, ties -> lower id ----
  int rank = 0;
#pragma unroll 1
  for (int i = 0; i < a.k; ++i) {
    float wi = __shfl_sync(0xffffffffu, w, i);
    int ii = __shfl_sync(0xffffffffu, my_id, i);
    if (lane < a.k && i != lane && better(wi, ii, w, my_id)) ++rank;
  }
  if (lane < a.k) {
    a.topk_idx[(int64_t)t * a.k + rank] = my_id;
    a.topk_w[(int64_t)t * a.k + rank] = w;
  }
  if (a.shared_gated && lane == 0) a.sgate[t] = 1.f / (1.f + expf(-lg[E]));
}

__global__ void __launch_bounds__(RT_WARPS * 32)
router_select_kernel(const __grid_constant__ RouterArgs a) {
  extern __shared__ float smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int t = blockIdx.x * RT_WARPS + warp;
  if (t >= a.T) return;
  select_token(a, t, smem + warp * 2 * a.E, smem + warp * 2 * a.E + a.E, lane);
}

// Block-parallel routing of ONE token (decode): every thread owns <= 4 experts;
// selection by rank (rank(e) = #experts that beat e) instead of k sequential
// arg-max rounds, so the latency is a few short loops over shared memory.
// Same rules and tie-breaks as select_token.  Scratch: s[E], sel[E], gsc[32],
// ids[32], ws[32] in shared memory.
template <int NT>
__device__ void select_token_block(const RouterArgs &args, int t, float *s, float *sel, float *gsc, int *ids,
                                   float *ws, long long *ck = nullptr) {
  if (ck && threadIdx.x == 0) ck[0] = clock64();
  const int E = args.E, k = args.k, G = args.n_group, TG = args.topk_group;
  const float *lg = args.logits + (int64_t)t * args.ldl;
  const float *bias = args.bias;
  const int tid = threadIdx.x;
  __shared__ float red[NT / 32];
  // scores
  float lv[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) lv[i] = (tid + NT * i < E) ? lg[tid + NT * i] : -INFINITY;
  if (args.score_fn == MOE_SCORE_SOFTMAX) {
    float m = fmaxf(fmaxf(lv[0], lv[1]), fmaxf(lv[2], lv[3]));
    m = warp_max(m);
    if ((tid & 31) == 0) red[tid >> 5] = m;
    __syncthreads();
    m = red[0];
#pragma unroll 1
    for (int w = 1; w < NT / 32; ++w) m = fmaxf(m, red[w]);
    __syncthreads();
    float sum = 0.f;
#pragma unroll
    for (int i = 0; i < 4; ++i) { lv[i] = (tid + NT * i < E) ? expf(lv[i] - m) : 0.f; sum += lv[i]; }
    sum = warp_sum(sum);
    if ((tid & 31) == 0) red[tid >> 5] = sum;
    __syncthreads();
    sum = 0.f;
#pragma unroll 1
    for (int w = 0; w < NT / 32; ++w) sum += red[w];
#pragma unroll
    for (int i = 0; i < 4; ++i) lv[i] = lv[i] / sum;
  } else {
#pragma unroll
    for (int i = 0; i < 4; ++i) lv[i] = 1.f / (1.f + expf(-lv[i]));
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int e = tid + NT * i;
    if (e < E) { s[e] = lv[i]; sel[e] = lv[i] + (bias ? bias[e] : 0.f); }
  }
  __syncthreads();
  if (ck && threadIdx.x == 0) ck[1] = clock64();
  // group limit: thread g scores group g, then ranks it
  if (G > 1) {
    const int gs = E / G;
    if (gs == 32 && E <= NT) {
      // one warp per group (DeepSeek-V3: 256 experts / 8 groups): warp reductions
      const int lane = tid & 31, g = tid >> 5;
      if (g < G) {
        const float v = sel[tid];
        const float m1 = warp_max(v);
        const int nmax = __popc(__ballot_sync(0xffffffffu, v == m1));
        const float m2 = nmax >= 2 ? m1 : warp_max(v == m1 ? -INFINITY : v);
        if (lane == 0) gsc[g] = args.group_score == MOE_GROUP_TOP2_SUM ? m1 + m2 : m1;
      }
    } else if (tid < G) {
      float m1 = -INFINITY, m2 = -INFINITY;
#pragma unroll 1
      for (int i = 0; i < gs; ++i) {
        const float v = sel[tid * gs + i];
        if (v > m1) { m2 = m1; m1 = v; } else if (v > m2) { m2 = v; }
      }
      gsc[tid] = args.group_score == MOE_GROUP_TOP2_SUM ? m1 + m2 : m1;
    }
    __syncthreads();
    if (tid < G) {
      int rk = 0;
#pragma unroll 1
      for (int g = 0; g < G; ++g) rk += better(gsc[g], g, gsc[tid], tid);
      ids[tid] = rk < TG;                          // keep flag
    }
    __syncthreads();
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int e = tid + NT * i;
      if (e < E && !ids[e / gs]) sel[e] = -INFINITY;
    }
    __syncthreads();
    if (ck && threadIdx.x == 0) ck[2] = clock64();
  }
  // top-k in two warp-level rounds (short loops: this tail runs once, on one SM,
  // with a cold instruction cache): (1) every warp extracts the k best of its
  // <= 128 experts by k arg-max rounds; (2) warp 0 merges the NT/32 candidate
  // lists the same way.  Masked (-inf) experts never qualify.
  {
    __shared__ float cv[NT / 32][32];
    __shared__ int ci[NT / 32][32];
    const int lane = tid & 31, w = tid >> 5;
    float v[4];
    int id[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int e = tid + NT * i;
      const float x = e < E ? sel[e] : -INFINITY;
      v[i] = x; id[i] = x == -INFINITY ? 0x7fffffff : e;
    }
#pragma unroll 1
    for (int r = 0; r < k; ++r) {
      float bv = v[0]; int bi = id[0];
#pragma unroll
      for (int i = 1; i < 4; ++i) if (better(v[i], id[i], bv, bi)) { bv = v[i]; bi = id[i]; }
      warp_argmax(bv, bi);
      if (lane == 0) { cv[w][r] = bv; ci[w][r] = bi; }
#pragma unroll
      for (int i = 0; i < 4; ++i) if (id[i] == bi) { v[i] = -INFINITY; id[i] = 0x7fffffff; }
    }
    __syncthreads();
    if (ck && threadIdx.x == 0) ck[3] = clock64();
    if (w == 0) {
      // candidates: NT/32 lists of k <= 32 -> <= NT/32 per lane
      constexpr int NC = NT / 32;
      float mv[NC]; int mi[NC];
#pragma unroll
      for (int i = 0; i < NC; ++i) {
        const int c = lane + 32 * i;              // candidate index = list * k + rank
        const bool ok = c < (NT / 32) * k;
        mv[i] = ok ? cv[c / k][c % k] : -INFINITY;
        mi[i] = ok ? ci[c / k][c % k] : 0x7fffffff;
      }
#pragma unroll 1
      for (int r = 0; r < k; ++r) {
        float bv = mv[0]; int bi = mi[0];
#pragma unroll
        for (int i = 1; i < NC; ++i) if (better(mv[i], mi[i], bv, bi)) { bv = mv[i]; bi = mi[i]; }
        warp_argmax(bv, bi);
        if (lane == 0) { ids[r] = bi; ws[r] = s[bi]; }
#pragma unroll
        for (int i = 0; i < NC; ++i) if (mi[i] == bi) { mv[i] = -INFINITY; mi[i] = 0x7fffffff; }
      }
    }
  }
  __syncthreads();
  if (ck && threadIdx.x == 0) ck[4] = clock64();
  // weights + canonical order (warp 0)
  if (tid < 32) {
    const int lane = tid;
    const int my_id = lane < k ? ids[lane] : 0x7fffffff;
    float w = lane < k ? ws[lane] : 0.f;
    if (args.norm_topk) w = w / warp_sum(w);
    w = w * args.routed_scale;
    int rank = 0;
#pragma unroll 1
    for (int i = 0; i < k; ++i) {
      const float wi = __shfl_sync(0xffffffffu, w, i);
      const int ii = __shfl_sync(0xffffffffu, my_id, i);
      if (lane < k && i != lane && better(wi, ii, w, my_id)) ++rank;
    }
    if (lane < k) {
      args.topk_idx[(int64_t)t * k + rank] = my_id;
      args.topk_w[(int64_t)t * k + rank] = w;
    }
    if (args.shared_gated && lane == 0) args.sgate[t] = 1.f / (1.f + expf(-lg[E]));
  }
  __syncthreads();
  if (ck && threadIdx.x == 0) ck[5] = clock64();
}

// ------------------------------------------------------------------ small T (decode)
// One launch for T <= 16 tokens: every CTA computes the router logits of two
// router rows (128 threads per row, whole row loaded at once), the last CTA to
// finish routes the tokens (select_token) and builds the expert-sorted order
// (counts, offsets, active-expert list, stable positions) -- the launch chain
// logits -> select -> count/scan/assign collapsed for the latency-bound decode step.
constexpr int RS_THREADS = 256;

__global__ void __launch_bounds__(RS_THREADS) route_small_kernel(const __grid_constant__ RouteSmallArgs a) {
  extern __shared__ float rsm[];
  const RouterArgs &r = a.r;
  const int H = a.H, T = r.T;
  const int half = threadIdx.x >> 7, tid = threadIdx.x & 127;
  const int row = blockIdx.x * 2 + half;
  __shared__ float red[2][4][16];
  __shared__ int is_last;
  pdl_trigger();
  // the shared expert's weights do not depend on the routing: pull them into
  // L2 now (HBM is otherwise idle while the router runs), so the first units
  // of the decode weight stream hit L2
  if (threadIdx.x == 0) {
#pragma unroll 1
    for (int i = 0; i < 2; ++i) {
      if (!a.pf[i]) continue;
      const int64_t per = ((a.pf_bytes[i] + gridDim.x - 1) / gridDim.x + 4095) & ~int64_t(4095);
      const int64_t b0 = (int64_t)blockIdx.x * per, b1 = b0 + per < a.pf_bytes[i] ? b0 + per : a.pf_bytes[i];
#pragma unroll 1
      for (int64_t o = b0; o < b1; o += 32768)
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(reinterpret_cast<const uint8_t *>(a.pf[i]) + o),
                     "r"((uint32_t)(b1 - o < 32768 ? b1 - o : 32768))
                     : "memory");
    }
  }
  // ---- logits of router rows `row` for all T tokens ----
  // (H <= 8192: each thread's <= 8 16-byte chunks of the row are loaded once,
  //  then a runtime loop over the tokens -- no per-token register arrays)
  {
    const int w4 = tid >> 5, lane = threadIdx.x & 31;
    const int nv = H / 8;
    uint4 w[8];
    const bool live = row < a.rows && !(a.debug & 1);
    const uint4 *wr = reinterpret_cast<const uint4 *>(reinterpret_cast<const __nv_bfloat16 *>(a.wg) + (size_t)row * H);
#pragma unroll
    for (int u = 0; u < 8; ++u) w[u] = (live && tid + u * 128 < nv) ? __ldg(wr + tid + u * 128) : make_uint4(0, 0, 0, 0);
#pragma unroll 1
    for (int t = 0; t < T; ++t) {
      const uint4 *xr = reinterpret_cast<const uint4 *>(reinterpret_cast<const __nv_bfloat16 *>(a.x) + (size_t)t * H);
      float acc = 0.f;
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int c = tid + u * 128;
        if (c < nv) {
          float wf[8], xf[8];
          bf16x8_to_f32(w[u], wf);
          bf16x8_to_f32(__ldg(xr + c), xf);
#pragma unroll
          for (int j = 0; j < 8; ++j) acc = fmaf(wf[j], xf[j], acc);
        }
      }
      acc = warp_sum(acc);
      if (lane == 0) red[half][w4][t] = acc;
    }
    __syncthreads();
    if (row < a.rows && tid < T)
      const_cast<float *>(r.logits)[(size_t)tid * r.ldl + row] = red[half][0][tid] + red[half][1][tid] + red[half][2][tid] + red[half][3][tid];
  }
  // ---- FP8: quantise x -> xq (token order) across all CTAs, in parallel with routing ----
  if (a.fp8 && a.xq) {
    const int nc = H / 8;                       // 8-element chunks per row; a 1x128 block = 16 chunks
    const int64_t total = (int64_t)T * nc;
    const int lane = threadIdx.x & 31;
    for (int64_t base = ((int64_t)blockIdx.x * RS_THREADS + (threadIdx.x & ~31)); base < total;
         base += (int64_t)gridDim.x * RS_THREADS) {
      const int64_t gch = base + lane;
      const bool ok = gch < total;
      float f[8];
      float am = 0.f;
      if (ok) {
        const int64_t t = gch / nc, c = gch % nc;
        bf16x8_to_f32(__ldg(reinterpret_cast<const uint4 *>(reinterpret_cast<const __nv_bfloat16 *>(a.x) + t * H) + c),
                      f);
#pragma unroll
        for (int j = 0; j < 8; ++j) am = fmaxf(am, fabsf(f[j]));
      }
#pragma unroll
      for (int o = 8; o > 0; o >>= 1) am = fmaxf(am, __shfl_xor_sync(0xffffffffu, am, o));
      if (ok) {
        const int64_t t = gch / nc, c = gch % nc;
        const int ex = ue8m0_exponent(am);
        const float inv = exp2i(-ex);
        uint2 q;
        q.x = (uint32_t)f32_to_e4m3(f[0] * inv) | ((uint32_t)f32_to_e4m3(f[1] * inv) << 8) |
              ((uint32_t)f32_to_e4m3(f[2] * inv) << 16) | ((uint32_t)f32_to_e4m3(f[3] * inv) << 24);
        q.y = (uint32_t)f32_to_e4m3(f[4] * inv) | ((uint32_t)f32_to_e4m3(f[5] * inv) << 8) |
              ((uint32_t)f32_to_e4m3(f[6] * inv) << 16) | ((uint32_t)f32_to_e4m3(f[7] * inv) << 24);
        *reinterpret_cast<uint2 *>(reinterpret_cast<uint8_t *>(a.xq) + t * H + c * 8) = q;
        if ((lane & 15) == 0) {
          const int b = (int)(c >> 4);
          a.xs[t * (H / 128) + b] = exp2i(ex);
          if (a.xq_img) a.xq_img[sf_img_off(t, b, a.xq_img_stride)] = (uint8_t)(ex + 127);
        }
      }
    }
  }

  // ---- last CTA: route + permute ----
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) is_last = (atomicAdd(a.done, 1) == (int)gridDim.x - 1);
  __syncthreads();
  if (!is_last) return;
  long long ck0 = clock64();
  __shared__ long long cold_ck[8];
  if (a.debug & 2) { if (threadIdx.x == 0) *a.done = 0; return; }
  __threadfence();
  {
    float *s = rsm, *sel = rsm + r.E, *gsc = rsm + 2 * r.E, *ws = gsc + 32;
    int *ids = reinterpret_cast<int *>(ws + 32);
#pragma unroll 1
    for (int t = 0; t < T; ++t) select_token_block<RS_THREADS>(r, t, s, sel, gsc, ids, ws, (a.debug & 4) ? cold_ck : nullptr);
    if (a.debug & 8) {                           // MOE_DEBUG_ROUTE=12: time a second (warm i-cache) pass
      __syncthreads();
      const long long w0 = clock64();
      unsigned long long g0, g1;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g0));
      __shared__ long long ck[8];
#pragma unroll 1
      for (int t = 0; t < T; ++t) select_token_block<RS_THREADS>(r, t, s, sel, gsc, ids, ws, ck);
      __syncthreads();
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g1));
      if (threadIdx.x == 0)
        printf("route tail: warm select pass %lld cycles (%llu ns): scores %lld group %lld warp-topk %lld merge %lld weights %lld\n",
               clock64() - w0, g1 - g0, ck[1] - ck[0], ck[2] - ck[1], ck[3] - ck[2], ck[4] - ck[3], ck[5] - ck[4]);
    }
  }
  long long ck1 = clock64();
  {
  }
  // counts / offsets / active list over the local experts
  const PermuteArgs &p = a.p;
  int *cnt = reinterpret_cast<int *>(rsm);          // reuse scratch: [E] counts, [E] running
  int *run = cnt + p.E;
  for (int e = threadIdx.x; e < p.E; e += RS_THREADS) cnt[e] = 0;
  __syncthreads();
  for (int q = threadIdx.x; q < T * p.k; q += RS_THREADS) {
    const int e = p.topk_idx[q] - p.e0;
    p.pos[q] = -1;
    if (e >= 0 && e < p.E) atomicAdd(&cnt[e], 1);
  }
  __syncthreads();
  {
    // one exclusive scan over the experts of a packed triple (count | tiles << 11 |
    // active << 21): T*k <= 512 rows, <= 1024 tiles and experts -- 4 experts per thread
    using Scan = cub::BlockScan<int, RS_THREADS>;
    __shared__ typename Scan::TempStorage tmp;
    int v[4], o[4], tot;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int e = threadIdx.x * 4 + i;
      const int c = e < p.E ? cnt[e] : 0;
      v[i] = c | (((c + kPadM - 1) / kPadM) << 11) | ((c > 0) << 21);
    }
    Scan(tmp).ExclusiveSum(v, o, tot);
    if (threadIdx.x == 0) {
      p.offs[p.E] = tot & 2047;
      p.offs_pad[p.E] = ((tot >> 11) & 1023) * kPadM;
      *p.n_active = tot >> 21;
      *p.n_tiles = 0;
      *a.done = 0;                                 // re-arm the CTA counter (graph replay)
    }
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int e = threadIdx.x * 4 + i;
      if (e < p.E) {
        const int c = v[i] & 2047;
        p.counts[e] = c;
        if (p.dbg_counts) p.dbg_counts[e] = c;
        p.offs[e] = o[i] & 2047;
        p.offs_pad[e] = ((o[i] >> 11) & 1023) * kPadM;
        run[e] = 0;
        if (c > 0) p.act_list[o[i] >> 21] = e;
      }
    }
  }
  __syncthreads();
  long long ck2 = clock64();
  // stable assignment: tokens in order, a token's k experts are distinct
  for (int t = 0; t < T; ++t) {
    if (threadIdx.x < p.k) {
      const int q = t * p.k + threadIdx.x;
      const int e = p.topk_idx[q] - p.e0;
      if (e >= 0 && e < p.E) {
        const int i = run[e]++;
        const int rw = p.offs_pad[e] + i;
        p.row_token[rw] = t;
        p.pos[q] = rw;
        if (p.dbg_perm) p.dbg_perm[p.offs[e] + i] = t;
      }
    }
    __syncthreads();
  }
  if (!a.xperm) return;
  long long ck3 = clock64();
  // activations into expert order (replaces the quantise + gather launches)
  __shared__ int spos[32];
  ScatterDst d{};
  d.fp8 = a.fp8; d.xperm = a.xperm; d.xperm_img = a.xperm_img; d.xperm_img_stride = a.xperm_img_stride;
  d.xq = a.xq; d.xs = a.xs; d.xq_img = a.xq_img; d.xq_img_stride = a.xq_img_stride;
#pragma unroll 1
  for (int t = 0; t < T; ++t) {
    if (threadIdx.x < p.k) spos[threadIdx.x] = p.pos[t * p.k + threadIdx.x];
    __syncthreads();
    if (a.fp8) {
      // codes were quantised into xq by all CTAs: copy the row and its scale bytes
      // every thread loads its chunks (<= 4: H <= 16384) and scale byte once, then stores k times
      const uint4 *src = reinterpret_cast<const uint4 *>(reinterpret_cast<const uint8_t *>(a.xq) + (size_t)t * H);
      uint4 v[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int c = threadIdx.x + RS_THREADS * i;
        if (c < H / 16) v[i] = src[c];
      }
      const int b = threadIdx.x;
      const uint8_t sb = b < H / 128 ? (uint8_t)((__float_as_uint(a.xs[(size_t)t * (H / 128) + b]) >> 23) & 0xFF) : 0;
#pragma unroll 1
      for (int j = 0; j < p.k; ++j) {
        const int rw = spos[j];
        if (rw < 0) continue;
        uint4 *dst = reinterpret_cast<uint4 *>(reinterpret_cast<uint8_t *>(a.xperm) + (size_t)rw * H);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int c = threadIdx.x + RS_THREADS * i;
          if (c < H / 16) dst[c] = v[i];
        }
        if (b < H / 128) a.xperm_img[sf_img_off(rw, b, a.xperm_img_stride)] = sb;
      }
    } else {
      scatter_token_row<RS_THREADS>(reinterpret_cast<const __nv_bfloat16 *>(a.x) + (size_t)t * H, H, t, p.k, spos, d);
    }
    __syncthreads();
  }
  if ((a.debug & 4) && threadIdx.x == 0)       // MOE_DEBUG_ROUTE=4: phase cycle counts of the tail
    printf("route tail cycles: select %lld (scores %lld group %lld warp-topk %lld merge %lld weights %lld) scan %lld "
           "assign %lld rows %lld\n", ck1 - ck0, cold_ck[1] - cold_ck[0], cold_ck[2] - cold_ck[1],
           cold_ck[3] - cold_ck[2], cold_ck[4] - cold_ck[3], cold_ck[5] - cold_ck[4], ck2 - ck1, ck3 - ck2,
           clock64() - ck3);
}

cudaError_t launch_route_small(const RouteSmallArgs &a, cudaStream_t st) {
  if (a.r.T <= 0) return cudaSuccess;
  const size_t sm = std::max<size_t>((size_t)(RS_THREADS / 32) * 2 * a.r.E * sizeof(float), 2 * a.p.E * sizeof(int));
  if (sm > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(route_small_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
  }
  route_small_kernel<<<(a.rows + 1) / 2, RS_THREADS, sm, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_router_select(const RouterArgs &a, cudaStream_t st) {
  if (a.T <= 0) return cudaSuccess;
  const int grid = (a.T + RT_WARPS - 1) / RT_WARPS;
  const size_t sm = (size_t)RT_WARPS * 2 * a.E * sizeof(float);
  if (sm > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(router_select_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
  }
  router_select_kernel<<<grid, RT_WARPS * 32, sm, st>>>(a);
  return cudaGetLastError();
}

}  // namespace moe
