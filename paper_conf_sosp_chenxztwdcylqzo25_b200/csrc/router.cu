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
  return (v > v2) | ((v == v2) & (i < i2));
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

// ------------------------------------------------------------------ small T (decode)
// One launch for T <= 16 tokens: every CTA computes the router logits of two
// router rows (128 threads per row, whole row loaded at once), the last CTA to
// finish routes the tokens (select_token) and builds the expert-sorted order
// (counts, offsets, active-expert list, stable positions) -- the launch chain
// logits -> select -> count/scan/assign collapsed for the latency-bound decode step.
constexpr int RS_THREADS = 256;
__device__ __forceinline__ unsigned long long gtimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
constexpr int RS_MAX_E = 256;      // router experts per lane-major warp layout: 32 lanes x 8
constexpr int RS_MAX_PAIRS = 512;  // T * k

// One warp routes token t with everything in registers (lane l holds experts
// 8l .. 8l+7): scores, group limit, k arg-max rounds, weights and the
// canonical slot order (same rules and tie-breaks as select_token).
// scratch: E floats of this warp's shared memory.  Writes topk_idx / topk_w /
// sgate and the canonical ids into ids_s[t * k ..].
// Control flow is warp-uniform throughout (live only predicates the stores), so the
// shuffles compile to plain SHFL, not the collective-emulated form.
#ifdef SELECT_PROFILE
__device__ long long g_sel_ck[8];
#define SEL_CK(i) do { if (lane == 0) g_sel_ck[i] = clock64(); } while (0)
#else
#define SEL_CK(i) do { } while (0)
#endif
// (sel, id) -> 64-bit key, larger = better: order-preserving float bits, then
// the complemented id (ties -> lower expert id, reading R2)
__device__ __forceinline__ unsigned long long sel_key(float v, int id) {
  const uint32_t u = __float_as_uint(v);
  const uint32_t o = (u & 0x80000000u) ? ~u : (u | 0x80000000u);
  return ((unsigned long long)o << 32) | (uint32_t)(~(uint32_t)id);
}
__device__ __forceinline__ int key_id(unsigned long long key) { return (int)~(uint32_t)key; }

__device__ void select_token_regs(const RouterArgs &r, int t, float *scratch, int *ids_s, int lane, bool live,
                                  const float *bias_pre = nullptr) {
  const int E = r.E, k = r.k, G = r.n_group;
  SEL_CK(0);
  const float *lg = r.logits + (int64_t)t * r.ldl;
  float *s_sm = scratch;                         // [E] unbiased scores
  float *sel_sm = scratch + RS_MAX_E;            // [E] selection scores (group pass)
  float lv[8], bv[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int e = lane * 8 + i;
    lv[i] = e < E ? lg[e] : -INFINITY;
    bv[i] = bias_pre ? bias_pre[i] : ((e < E && r.bias) ? r.bias[e] : 0.f);
  }
  float s[8], sel[8];
  if (r.score_fn == MOE_SCORE_SOFTMAX) {
    float m = lv[0];
#pragma unroll
    for (int i = 1; i < 8; ++i) m = fmaxf(m, lv[i]);
    m = warp_max(m);
    float sum = 0.f;
#pragma unroll
    for (int i = 0; i < 8; ++i) { s[i] = lane * 8 + i < E ? __expf(lv[i] - m) : 0.f; sum += s[i]; }
    sum = warp_sum(sum);
    const float inv = 1.f / sum;
#pragma unroll
    for (int i = 0; i < 8; ++i) s[i] = s[i] * inv;
  } else {
#pragma unroll
    for (int i = 0; i < 8; ++i) s[i] = __fdividef(1.f, 1.f + __expf(-lv[i]));   // ~2 ulp, far inside the 1e-5 tie band
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int e = lane * 8 + i;
    sel[i] = e < E ? s[i] + bv[i] : -INFINITY;
    if (e < E) { s_sm[e] = s[i]; sel_sm[e] = sel[i]; }
  }
  __syncwarp();
  SEL_CK(1);
  if (G > 1) {
    // group g = experts [g gs, (g+1) gs)
    const int gs = E / G;
    float m1 = -INFINITY, m2 = -INFINITY;
    float gsc;
    const int lpg = gs >> 3;                     // lanes per group when groups are whole lanes
    if ((gs & 7) == 0 && lpg <= 32 && (lpg & (lpg - 1)) == 0 && G * lpg <= 32) {
      // groups made of whole lanes (V3: 32 experts = 4 lanes): in-register top-2 of the
      // lane's 8, merged across the group's lanes by xor shuffles (branch-free)
#pragma unroll
      for (int i = 0; i < 8; ++i) { m2 = fmaxf(m2, fminf(m1, sel[i])); m1 = fmaxf(m1, sel[i]); }
      for (int o = 1; o < lpg; o <<= 1) {
        const float p1 = __shfl_xor_sync(0xffffffffu, m1, o), p2 = __shfl_xor_sync(0xffffffffu, m2, o);
        m2 = fmaxf(fminf(m1, p1), fmaxf(m2, p2));
        m1 = fmaxf(m1, p1);
      }
      // group g's score, gathered onto lane g
      const float own = r.group_score == MOE_GROUP_TOP2_SUM ? m1 + m2 : m1;
      const float got = __shfl_sync(0xffffffffu, own, (lane * lpg) & 31);
      gsc = lane < G ? got : -INFINITY;
    } else {
      // general layout: lane g scans group g in shared memory (branch-free top-2)
      if (lane < G) {
        const float *gp = sel_sm + lane * gs;
#pragma unroll 8
        for (int i = 0; i < gs; ++i) {
          const float v = gp[i];
          m2 = fmaxf(m2, fminf(m1, v));
          m1 = fmaxf(m1, v);
        }
      }
      gsc = lane < G ? (r.group_score == MOE_GROUP_TOP2_SUM ? m1 + m2 : m1) : -INFINITY;
    }
    int rk = 0;
#pragma unroll 8
    for (int j = 0; j < G; ++j) rk += better(__shfl_sync(0xffffffffu, gsc, j), j, gsc, lane);
    const unsigned keep = __ballot_sync(0xffffffffu, lane < G && rk < r.topk_group);
    int g = (lane * 8) / gs, rem = (lane * 8) - g * gs;   // group of expert 8 lane, walked forward
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      sel[i] = (g < 32 && ((keep >> g) & 1u)) ? sel[i] : -INFINITY;
      ++rem;
      const bool nx = rem == gs;
      g += nx;
      rem = nx ? 0 : rem;
    }
  }
  SEL_CK(2);
  int my_id = 0;
  float my_w = 0.f;
  int rank = 0;
  if (k <= 8) {
    // top-k by a sorting network on 64-bit keys: each lane sorts its 8, then five
    // butterfly steps merge partner lists (bitonic: keep the better of A[i] and
    // B[7-i], then sort the bitonic 8) -- every lane ends with the token's best 8
    // in (sel desc, id asc) order.  Branch-free: divergence around the shuffles
    // makes them collective-emulated (measured ~5x the cycles).
    unsigned long long key[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) key[i] = sel[i] == -INFINITY ? 0ull : sel_key(sel[i], lane * 8 + i);
    auto cx = [&](int i, int j) {
      const unsigned long long a = key[i], b = key[j];
      key[i] = a > b ? a : b;
      key[j] = a > b ? b : a;
    };
    // Batcher odd-even merge sort of 8 (19 comparators)
    cx(0, 1); cx(2, 3); cx(4, 5); cx(6, 7);
    cx(0, 2); cx(1, 3); cx(4, 6); cx(5, 7);
    cx(1, 2); cx(5, 6);
    cx(0, 4); cx(1, 5); cx(2, 6); cx(3, 7);
    cx(2, 4); cx(3, 5);
    cx(1, 2); cx(3, 4); cx(5, 6);
    SEL_CK(3);
    // (rolled: this code runs once per token with a cold instruction cache, so its
    //  footprint, not its instruction count, sets the latency)
#pragma unroll 1
    for (int o = 1; o < 32; o <<= 1) {
      unsigned long long pk[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) pk[i] = __shfl_xor_sync(0xffffffffu, key[i], o);
#pragma unroll
      for (int i = 0; i < 8; ++i) key[i] = key[i] > pk[7 - i] ? key[i] : pk[7 - i];
      cx(0, 4); cx(1, 5); cx(2, 6); cx(3, 7);
      cx(0, 2); cx(1, 3); cx(4, 6); cx(5, 7);
      cx(0, 1); cx(2, 3); cx(4, 5); cx(6, 7);
    }
    SEL_CK(4);
    // weights and canonical order, lane-local (every lane holds the list)
    float sv[8], sum = 0.f;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      sv[i] = i < k ? s_sm[key_id(key[i])] : 0.f;
      sum += sv[i];
    }
    // one reciprocal for the 8 weights (an IEEE division each cost ~1 K cycles in total)
    const float c = (r.norm_topk ? 1.f / sum : 1.f) * r.routed_scale;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
      const float w = sv[i] * c;
      const int id = key_id(key[i]);
      my_id = i == lane ? id : my_id;
      my_w = i == lane ? w : my_w;
      sv[i] = w;
    }
#pragma unroll
    for (int i = 0; i < 8; ++i) rank += (i < k) & (i != lane) & better(sv[i], key_id(key[i]), my_w, my_id);
  } else {
    // k > 8: k arg-max rounds; the owner lane retires the winner
    my_id = 0x7fffffff;
#pragma unroll 1
    for (int j = 0; j < k; ++j) {
      float v = -INFINITY;
      int id = 0x7fffffff;
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const bool b = better(sel[i], lane * 8 + i, v, id) & (sel[i] != -INFINITY);
        v = b ? sel[i] : v;
        id = b ? lane * 8 + i : id;
      }
      warp_argmax(v, id);
#pragma unroll
      for (int i = 0; i < 8; ++i) sel[i] = lane * 8 + i == id ? -INFINITY : sel[i];
      my_id = lane == j ? id : my_id;
    }
    float w = lane < k ? s_sm[my_id] : 0.f;
    if (r.norm_topk) w = w / warp_sum(w);
    my_w = w * r.routed_scale;
#pragma unroll 1
    for (int i = 0; i < k; ++i) {
      const float wi = __shfl_sync(0xffffffffu, my_w, i);
      const int ii = __shfl_sync(0xffffffffu, my_id, i);
      rank += (i != lane) & better(wi, ii, my_w, my_id);
    }
  }
  if (live && lane < k) {
    r.topk_idx[(int64_t)t * k + rank] = my_id;
    r.topk_w[(int64_t)t * k + rank] = my_w;
    if (ids_s) ids_s[t * k + rank] = my_id;
  }
  if (live && r.shared_gated && lane == 0) r.sgate[t] = 1.f / (1.f + expf(-lg[E]));
  SEL_CK(5);
  __syncwarp();                                  // scratch reuse by the next token of this warp
}

// Prefill selection (E <= 256): one warp per token with the register-resident
// select of the decode router (same rules; ~4x fewer cycles than select_token).
__global__ void __launch_bounds__(RT_WARPS * 32) router_select_regs_kernel(const __grid_constant__ RouterArgs a) {
  __shared__ float scratch[RT_WARPS][2 * RS_MAX_E];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int t = __shfl_sync(0xffffffffu, blockIdx.x * RT_WARPS + warp, 0);   // warp-uniform
  if (t < a.T) select_token_regs(a, t, scratch[warp], nullptr, lane, true);
}

// ---- one token, the whole CTA (decode at T = 1) ----
// Groups of exactly 32 experts (or no group limit), k <= 8, E <= 256: warp w scores
// experts 32w .. 32w+31 (one per lane), takes its group's score and its best k with warp
// max-reductions (redux.sync) on order-preserving bits -- ties to the lowest lane = the lower
// id -- and warp 0 merges the kept groups' candidates.  Same rules, tie-breaks and float
// operations (sigmoid / softmax, the sequential weight sum, one reciprocal) as select_token_regs, so
// both give bit-identical routing.
__device__ __forceinline__ uint32_t ord_bits(float v) {
  const uint32_t u = __float_as_uint(v);
  return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}
__device__ __forceinline__ float ord_float(uint32_t o) {
  return __uint_as_float((o & 0x80000000u) ? (o & 0x7FFFFFFFu) : ~o);
}
__device__ __forceinline__ bool route_one_fast_ok(const RouterArgs &r) {
  const int E = r.E, G = r.n_group;
  const int ng = G > 1 ? r.topk_group : E / 32;
  return r.T == 1 && r.k <= 8 && E % 32 == 0 && E <= RS_MAX_E &&
         (G <= 1 || E == 32 * G) && ng * r.k <= 32;
}
// Writes topk_idx / topk_w / sgate and ids_s[0 .. k) (canonical order).  With lists = true
// (all experts local, no debug outputs) also the fused decode's active / immediate / deferred
// expert lists (ascending ids) and re-arms the CTA counter.
__device__ void route_one_fast(const RouteSmallArgs &a, int *ids_s, bool lists) {
  const RouterArgs &r = a.r;
  const int E = r.E, G = r.n_group, k = r.k;
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const int NW = E / 32;
  __shared__ float s_all[RS_MAX_E], gsc_s[8], sv_s[8];
  __shared__ uint32_t cand_o[32];
  __shared__ int cand_id[32], id_s[8], rc_s[8];
  const bool act = w < NW;                       // warp-uniform
  const int e = w * 32 + lane;
  uint32_t o = 0u;
  if (r.score_fn == MOE_SCORE_SOFTMAX) {
    // warp 0 computes the softmax in select_token_regs's layout and order (lane l: experts
    // 8l .. 8l+7; lane max, warp max, lane sum, warp sum, one reciprocal) -- bit-identical s
    if (w == 0) {
      float lv[8], m = -INFINITY, sum = 0.f, sv[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        lv[i] = lane * 8 + i < E ? r.logits[lane * 8 + i] : -INFINITY;
        m = i ? fmaxf(m, lv[i]) : lv[i];
      }
      m = warp_max(m);
#pragma unroll
      for (int i = 0; i < 8; ++i) { sv[i] = lane * 8 + i < E ? __expf(lv[i] - m) : 0.f; sum += sv[i]; }
      sum = warp_sum(sum);
      const float inv = 1.f / sum;
#pragma unroll
      for (int i = 0; i < 8; ++i)
        if (lane * 8 + i < E) s_all[lane * 8 + i] = sv[i] * inv;
    }
    __syncthreads();
    if (act) o = ord_bits(s_all[e] + (r.bias ? r.bias[e] : 0.f));
  } else if (act) {
    const float l = r.logits[e];
    const float b = r.bias ? r.bias[e] : 0.f;
    const float s = __fdividef(1.f, 1.f + __expf(-l));
    s_all[e] = s;
    o = ord_bits(s + b);
  }
  unsigned long long *tr = a.trace ? a.trace + 1900 : nullptr;     // MOE_DEBUG_TRACE: phase stamps
  if (tr && tid == 0) tr[0] = gtimer_ns();
  int slot0 = w * k;                             // this group's place in the candidate list
  bool keep = true;
  if (G > 1) {
    if (act) {
      const uint32_t m1 = __reduce_max_sync(0xffffffffu, o);
      const uint32_t one = __ballot_sync(0xffffffffu, o == m1);
      const uint32_t m2 = __reduce_max_sync(0xffffffffu, lane == __ffs(one) - 1 ? 0u : o);
      if (lane == 0)
        gsc_s[w] = r.group_score == MOE_GROUP_TOP2_SUM ? ord_float(m1) + ord_float(m2) : ord_float(m1);
    }
    __syncthreads();
    if (tr && tid == 0) tr[1] = gtimer_ns();
    if (act) {
      const float mine = gsc_s[w];
      int rk = 0;
      for (int j = 0; j < G; ++j) rk += better(gsc_s[j], j, mine, w);
      keep = rk < r.topk_group;
      slot0 = rk * k;                            // group rank: unique among the kept groups
    }
  }
  if (act && keep) {
    uint32_t c = o;
#pragma unroll 1
    for (int i = 0; i < k; ++i) {
      const uint32_t m = __reduce_max_sync(0xffffffffu, c);
      const int win = __ffs(__ballot_sync(0xffffffffu, c == m)) - 1;
      if (lane == win) c = 0u;
      if (lane == 0) { cand_o[slot0 + i] = m; cand_id[slot0 + i] = w * 32 + win; }
    }
  }
  __syncthreads();
  if (tr && tid == 0) tr[2] = gtimer_ns();
  if (w != 0) return;
  const int nc = (G > 1 ? r.topk_group : NW) * k;
  const bool has = lane < nc;
  const uint32_t mo = has ? cand_o[lane] : 0u;
  const int mid = has ? cand_id[lane] : 0x7fffffff;
  int rank = 0;
  for (int j = 0; j < nc; ++j) {
    const uint32_t oj = cand_o[j];
    rank += (oj > mo) | ((oj == mo) & (cand_id[j] < mid));
  }
  if (has && rank < k) { id_s[rank] = mid; sv_s[rank] = s_all[mid]; }
  __syncwarp();
  float sum = 0.f;
#pragma unroll
  for (int i = 0; i < 8; ++i) sum += i < k ? sv_s[i] : 0.f;
  const float cmul = (r.norm_topk ? 1.f / sum : 1.f) * r.routed_scale;
  int rc = 0, my_id = 0;
  if (lane < k) {
    my_id = id_s[lane];
    const float my_w = sv_s[lane] * cmul;
#pragma unroll
    for (int i = 0; i < 8; ++i) rc += (i < k) & (i != lane) & better(sv_s[i] * cmul, id_s[i], my_w, my_id);
    r.topk_idx[rc] = my_id;
    r.topk_w[rc] = my_w;
    ids_s[rc] = my_id;
    rc_s[lane] = rc;
  }
  if (r.shared_gated && lane == 0) r.sgate[0] = 1.f / (1.f + expf(-r.logits[E]));
  if (tr && lane == 0) tr[3] = gtimer_ns();
  if (!lists) return;
  __syncwarp();
  if (lane < k) {
    // T = 1: the k experts are distinct -- a list position is a count of smaller ids
    const bool imm = rc < a.n_imm;
    int below = 0, below_same = 0;
    for (int i = 0; i < k; ++i) {
      const bool lt = id_s[i] < my_id;
      below += lt;
      below_same += lt & ((rc_s[i] < a.n_imm) == imm);
    }
    a.p.act_list[below] = my_id;
    if (a.imm_list) (imm ? a.imm_list : a.def_list)[below_same] = my_id;
  }
  if (lane == 0) {
    *a.p.n_active = k;
    if (a.imm_list) { *a.n_imm_list = min(a.n_imm, k); *a.n_def_list = k - min(a.n_imm, k); }
    *a.done = 0;                                 // re-arm the CTA counter (graph replay)
  }
}

// The last router CTA: route every token (one warp per token), then the
// expert-sorted order for T <= 16 tokens -- with at most T <= kPadM rows per
// expert every active expert's padded segment is one 128-row tile, so its
// position is (number of active experts below it) x 128, read off a bitmap of
// the active experts; a pair's row within the segment is the number of
// earlier tokens that chose the same expert (stable by token).  Finally the
// token rows (FP8: the codes quantised by all CTAs) are copied to their k rows.
__device__ void route_small_tail(const RouteSmallArgs &a, float *rsm, const float *bias_pre) {
  const RouterArgs &r = a.r;
  const PermuteArgs &p = a.p;
  const int T = r.T, k = r.k, TK = T * k;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  __shared__ int ids_s[RS_MAX_PAIRS];
  __shared__ int cnt_s[RS_MAX_E], slot_s[RS_MAX_E], offs_s[RS_MAX_E];
  __shared__ unsigned bm[RS_MAX_E / 32], bmi[RS_MAX_E / 32], bmd[RS_MAX_E / 32];
  long long ck[4];
  ck[0] = clock64();
  if (a.trace && tid == 0) a.trace[1] = gtimer_ns();
  const bool fast = route_one_fast_ok(r) && !(kExperiments && (a.debug & 16));   // MOE_DEBUG_ROUTE=16: general select
  if (fast) {
    const bool lists = p.e0 == 0 && p.E == r.E && !p.dbg_perm && !p.dbg_counts;
    route_one_fast(a, ids_s, lists);
    if (lists) {
      if (a.trace && tid == 0) { a.trace[2] = gtimer_ns(); a.trace[3] = a.trace[4] = a.trace[2]; }
      return;
    }
    __syncthreads();
  }
  for (int e = tid; e < p.E; e += RS_THREADS) cnt_s[e] = 0;
  if (tid < RS_MAX_E / 32) bm[tid] = bmi[tid] = bmd[tid] = 0u;
  // one warp per token; warps past the last token skip (warp-uniform branch)
#pragma unroll 1
  for (int t0 = 0; t0 < T && !fast; t0 += RS_THREADS / 32) {
    const int t = __shfl_sync(0xffffffffu, t0 + warp, 0);
    if (t < T) select_token_regs(r, t, rsm + warp * 2 * RS_MAX_E, ids_s, lane, true, bias_pre);
  }
  __syncthreads();
  ck[1] = clock64();
  if (a.trace && tid == 0) a.trace[2] = gtimer_ns();
  if (kExperiments && (a.debug & 8)) {                             // timing experiment: a second (warm i-cache) select pass
    const long long w0 = clock64();
#pragma unroll 1
    for (int t0 = 0; t0 < T; t0 += RS_THREADS / 32) {
      const int t = __shfl_sync(0xffffffffu, t0 + warp, 0);
      if (t < T) select_token_regs(r, t, rsm + warp * 2 * RS_MAX_E, ids_s, lane, true, bias_pre);
    }
    __syncthreads();
    if (a.trace && tid == 0) { a.trace[5] = ck[1] - ck[0]; a.trace[6] = clock64() - w0; }
  }
  for (int q = tid; q < TK; q += RS_THREADS) {
    const int e = ids_s[q] - p.e0;
    if (e >= 0 && e < p.E) {
      atomicAdd(&cnt_s[e], 1);
      atomicOr(&bm[e >> 5], 1u << (e & 31));
      atomicOr(q % k < a.n_imm ? &bmi[e >> 5] : &bmd[e >> 5], 1u << (e & 31));
    }
  }
  __syncthreads();
  if (a.imm_list) {
    // Expert Deferral (chained forwards): the experts of the immediate and of the
    // deferred canonical slots, ascending (bitmap + popc, one thread per expert)
    const int e = tid;
    int bi = 0, ni = 0, bd = 0, nd = 0;
#pragma unroll
    for (int w = 0; w < RS_MAX_E / 32; ++w) {
      const int pi = __popc(bmi[w]), pd = __popc(bmd[w]);
      ni += pi; nd += pd;
      if (w < (e >> 5)) { bi += pi; bd += pd; }
    }
    const unsigned below = (1u << (e & 31)) - 1u;
    if (e < p.E && ((bmi[e >> 5] >> (e & 31)) & 1u)) a.imm_list[bi + __popc(bmi[e >> 5] & below)] = e;
    if (e < p.E && ((bmd[e >> 5] >> (e & 31)) & 1u)) a.def_list[bd + __popc(bmd[e >> 5] & below)] = e;
    if (tid == 0) { *a.n_imm_list = ni; *a.n_def_list = nd; }
  }
  if (!p.dbg_perm && !p.dbg_counts) {
    // fused decode: the expert kernel reads token-order activations and finds its
    // tokens in topk_idx, so only the active-expert list is needed (ascending ids)
    const int e = tid;
    int below = 0, nact = 0;
#pragma unroll
    for (int w = 0; w < RS_MAX_E / 32; ++w) {
      const int pc = __popc(bm[w]);
      nact += pc;
      if (w < (e >> 5)) below += pc;
    }
    if (e < p.E && ((bm[e >> 5] >> (e & 31)) & 1u))
      p.act_list[below + __popc(bm[e >> 5] & ((1u << (e & 31)) - 1u))] = e;
    if (tid == 0) {
      *p.n_active = nact;
      *a.done = 0;                                 // re-arm the CTA counter (graph replay)
    }
    if (a.trace && tid == 0) { a.trace[3] = gtimer_ns(); a.trace[4] = a.trace[3]; }
    return;
  }
  {
    using Scan = cub::BlockScan<int, RS_THREADS>;
    __shared__ typename Scan::TempStorage tmp;
    const int e = tid;
    const int c = e < p.E ? cnt_s[e] : 0;
    int o, tot;
    Scan(tmp).ExclusiveSum(c, o, tot);
    int below = 0, nact = 0;
#pragma unroll
    for (int w = 0; w < RS_MAX_E / 32; ++w) {
      const int pc = __popc(bm[w]);
      nact += pc;
      if (w < (e >> 5)) below += pc;
    }
    if (e < p.E) {
      const int slot = below + __popc(bm[e >> 5] & ((1u << (e & 31)) - 1u));
      p.counts[e] = c;
      p.offs[e] = o;
      p.offs_pad[e] = slot * kPadM;
      if (p.dbg_counts) p.dbg_counts[e] = c;
      if (c > 0) p.act_list[slot] = e;
      slot_s[e] = slot;
      offs_s[e] = o;
    }
    if (tid == 0) {
      p.offs[p.E] = tot;
      p.offs_pad[p.E] = nact * kPadM;
      *p.n_active = nact;
      *p.n_tiles = 0;
      *a.done = 0;                                 // re-arm the CTA counter (graph replay)
    }
  }
  __syncthreads();
  for (int q = tid; q < TK; q += RS_THREADS) {
    const int id = ids_s[q], e = id - p.e0, t = q / k;
    int rw = -1;
    if (e >= 0 && e < p.E) {
      int i = 0;
#pragma unroll 1
      for (int q2 = 0; q2 < t * k; ++q2) i += ids_s[q2] == id;
      rw = slot_s[e] * kPadM + i;
      p.row_token[rw] = t;
      if (p.dbg_perm) p.dbg_perm[offs_s[e] + i] = t;
    }
    p.pos[q] = rw;
  }
  __syncthreads();
  ck[2] = clock64();
  if (a.trace && tid == 0) a.trace[3] = gtimer_ns();
  ck[3] = clock64();
  if (a.trace && tid == 0) a.trace[4] = gtimer_ns();
  if (kExperiments && (a.debug & 4) && tid == 0)                 // MOE_DEBUG_ROUTE=4: phase cycle counts of the tail
    printf("route tail cycles: select %lld permute %lld rows %lld\n", ck[1] - ck[0], ck[2] - ck[1], ck[3] - ck[2]);
}



__global__ void __launch_bounds__(RS_THREADS) route_small_kernel(const __grid_constant__ RouteSmallArgs a) {
  extern __shared__ float rsm[];
  const RouterArgs &r = a.r;
  const int H = a.H, T = r.T;
  const int half = threadIdx.x >> 7, tid = threadIdx.x & 127;
  const int row = blockIdx.x * 2 + half;
  __shared__ float red[2][4][16];
  __shared__ int is_last;
  // router weights first: they do not depend on the predecessor kernel, so with
  // PDL their HBM latency overlaps the previous layer's tail
  const int w4 = tid >> 5, lane = threadIdx.x & 31;
  const int nv = H / 8;
  uint4 w[8];
  {
    const bool live = row < a.rows && !(kExperiments && (a.debug & 1));
    const uint4 *wr = reinterpret_cast<const uint4 *>(reinterpret_cast<const __nv_bfloat16 *>(a.wg) + (size_t)row * H);
#pragma unroll
    for (int u = 0; u < 8; ++u) w[u] = (live && tid + u * 128 < nv) ? __ldg(wr + tid + u * 128) : make_uint4(0, 0, 0, 0);
  }
  // the selection bias too (lane l: experts 8l .. 8l+7; used by the last CTA's route)
  float bpre[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int e = (threadIdx.x & 31) * 8 + i;
    bpre[i] = (r.bias && e < r.E) ? __ldg(r.bias + e) : 0.f;
  }
  // chained deferral: the decode stream may launch now and stream the previous layer's deferred
  // experts beside us; otherwise it launches once only the last CTA's tail is left (a launch
  // here measured ~1 us/layer slower: CTAs waiting in griddepcontrol.wait beside all 128 router
  // CTAs slow the logits phase down)
  if (a.early_trigger) pdl_trigger();
  // (an instruction-cache warm-up -- a dry run of the selection before the dependency wait --
  //  was measured: the window before the wait is ~1-2 us, so the dry run lands on the
  //  critical path, +1 us/layer plain, worse with deferral; MOE_DEBUG_ROUTE bit 32 in
  //  experiments builds re-enables it)
  if (kExperiments && (a.debug & 32) && threadIdx.x < 32)
    select_token_regs(r, 0, rsm, nullptr, threadIdx.x & 31, false, bpre);
  pdl_wait();                                    // x (the previous layer's output) and our workspaces
  if (a.trace && threadIdx.x == 0 && blockIdx.x == 0) a.trace[0] = gtimer_ns();
  // ---- logits of router rows `row` for all T tokens ----
  {
    // two tokens per step with all their x loads in flight together (a token at a
    // time serialised T L2 round trips: ~1.5 us each at T = 4)
#pragma unroll 1
    for (int t = 0; t < T; t += 2) {
      const bool two = t + 1 < T;
      const uint4 *xr0 = reinterpret_cast<const uint4 *>(reinterpret_cast<const __nv_bfloat16 *>(a.x) + (size_t)t * H);
      const uint4 *xr1 = two ? xr0 + H / 8 : xr0;
      uint4 xv0[8], xv1[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int c = tid + u * 128;
        xv0[u] = c < nv ? __ldg(xr0 + c) : make_uint4(0, 0, 0, 0);
        xv1[u] = c < nv ? __ldg(xr1 + c) : make_uint4(0, 0, 0, 0);
      }
      float acc0 = 0.f, acc1 = 0.f;
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        float wf[8], x0[8], x1[8];
        bf16x8_to_f32(w[u], wf);
        bf16x8_to_f32(xv0[u], x0);
        bf16x8_to_f32(xv1[u], x1);
#pragma unroll
        for (int j = 0; j < 8; ++j) { acc0 = fmaf(wf[j], x0[j], acc0); acc1 = fmaf(wf[j], x1[j], acc1); }
      }
      acc0 = warp_sum(acc0);
      acc1 = warp_sum(acc1);
      if (lane == 0) {
        red[half][w4][t] = acc0;
        if (two) red[half][w4][t + 1] = acc1;
      }
      // FP8: the x rows are in registers already -- CTA u < nv/128 quantises the 128-chunk slice u
      // (chunks tid + 128 u) of token t (half 0) / t + 1 (half 1): 1x128 UE8M0 over 16 lanes,
      // e4m3 RNE satfinite (reading R10), no second read of x
      if (a.fp8 && a.xq && (half == 0 || two)) {
#pragma unroll 1
        for (int u = blockIdx.x; u < 8 && u * 128 < nv; u += gridDim.x) {
          const int c = tid + u * 128, tt = t + half;
          uint4 xv = xv0[0];
#pragma unroll
          for (int uu = 0; uu < 8; ++uu) xv = uu == u ? (half ? xv1[uu] : xv0[uu]) : xv;
          float f[8];
          bf16x8_to_f32(xv, f);
          float am = 0.f;
#pragma unroll
          for (int j = 0; j < 8; ++j) am = fmaxf(am, fabsf(f[j]));
#pragma unroll
          for (int o = 8; o > 0; o >>= 1) am = fmaxf(am, __shfl_xor_sync(0xffffffffu, am, o));
          if (c < nv) {
            const int ex = ue8m0_exponent(am);
            const float inv = exp2i(-ex);
            uint2 q;
            q.x = (uint32_t)f32_to_e4m3(f[0] * inv) | ((uint32_t)f32_to_e4m3(f[1] * inv) << 8) |
                  ((uint32_t)f32_to_e4m3(f[2] * inv) << 16) | ((uint32_t)f32_to_e4m3(f[3] * inv) << 24);
            q.y = (uint32_t)f32_to_e4m3(f[4] * inv) | ((uint32_t)f32_to_e4m3(f[5] * inv) << 8) |
                  ((uint32_t)f32_to_e4m3(f[6] * inv) << 16) | ((uint32_t)f32_to_e4m3(f[7] * inv) << 24);
            *reinterpret_cast<uint2 *>(reinterpret_cast<uint8_t *>(a.xq) + (size_t)tt * H + c * 8) = q;
            if ((lane & 15) == 0) a.xs[(size_t)tt * (H / 128) + (c >> 4)] = exp2i(ex);
          }
        }
      }
    }
    __syncthreads();
    if (row < a.rows && tid < T)
      const_cast<float *>(r.logits)[(size_t)tid * r.ldl + row] = red[half][0][tid] + red[half][1][tid] + red[half][2][tid] + red[half][3][tid];
  }
  // ---- FP8, H > 8192 only (x slices beyond 8 x 128 chunks): quantise x -> xq from global ----
  if (a.fp8 && a.xq && nv > 8 * 128) {
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
        if ((lane & 15) == 0) a.xs[t * (H / 128) + (int)(c >> 4)] = exp2i(ex);
      }
    }
  }

  // ---- BF16: x into the layer's own token-order buffer (read by the decode stream) ----
  if (!a.fp8 && a.xcopy) {
    const int64_t n16 = (int64_t)T * H / 8;
    for (int64_t i = (int64_t)blockIdx.x * RS_THREADS + threadIdx.x; i < n16; i += (int64_t)gridDim.x * RS_THREADS)
      reinterpret_cast<uint4 *>(a.xcopy)[i] = __ldg(reinterpret_cast<const uint4 *>(a.x) + i);
  }

  // ---- last CTA: route + permute ----
  // (one gpu-scope acq_rel fence by the ticket thread after the CTA barrier orders
  //  every thread's logits / xq stores before the ticket, and the last CTA's reads after)
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
    const int tk = atomicAdd(a.done, 1);
    is_last = tk == (int)gridDim.x - 1;
    if (is_last) asm volatile("fence.acq_rel.gpu;" ::: "memory");
  }
  __syncthreads();
  if (!is_last) return;
  // every other CTA has exited: the decode stream may launch now, so its launch latency and
  // prologue overlap this tail (its griddepcontrol.wait still waits for the whole grid)
  if (!a.early_trigger && !(kExperiments && (a.debug & 64))) pdl_trigger();   // MOE_DEBUG_ROUTE=64: at exit
  if (kExperiments && (a.debug & 2)) { if (threadIdx.x == 0) *a.done = 0; return; }
  route_small_tail(a, rsm, bpre);
}

cudaError_t launch_route_small(const RouteSmallArgs &a, cudaStream_t st) {
  if (a.r.T <= 0) return cudaSuccess;
  const size_t sm = (size_t)(RS_THREADS / 32) * 2 * RS_MAX_E * sizeof(float);   // per-warp select scratch
  // max shared-memory carveout: the PDL-launched decode stream kernel (~190 KB
  // of smem) can then become resident beside the router CTAs
  cudaError_t e = set_kernel_attr((const void *)route_small_kernel, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  if (e != cudaSuccess) return e;
  if (sm > 48 * 1024) {
    e = set_kernel_attr((const void *)route_small_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
  }
  return launch_pdl(route_small_kernel, dim3((a.rows + 1) / 2), dim3(RS_THREADS), sm, st, a);
}

cudaError_t launch_router_select(const RouterArgs &a, cudaStream_t st) {
  if (a.T <= 0) return cudaSuccess;
  const int grid = (a.T + RT_WARPS - 1) / RT_WARPS;
  const size_t sm = (size_t)RT_WARPS * 2 * a.E * sizeof(float);
  if (sm > 48 * 1024) {
    cudaError_t e = set_kernel_attr((const void *)router_select_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
  }
  if (a.E <= RS_MAX_E) {
    router_select_regs_kernel<<<grid, RT_WARPS * 32, 0, st>>>(a);
    return cudaGetLastError();
  }
  router_select_kernel<<<grid, RT_WARPS * 32, sm, st>>>(a);
  return cudaGetLastError();
}

}  // namespace moe
