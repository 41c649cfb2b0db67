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

__global__ void __launch_bounds__(RT_WARPS * 32)
router_select_kernel(RouterArgs a) {
  extern __shared__ float smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int t = blockIdx.x * RT_WARPS + warp;
  if (t >= a.T) return;
  const int E = a.E;
  float *s = smem + warp * 2 * E;   // scores
  float *sel = s + E;               // selection scores
  const float *lg = a.logits + (int64_t)t * a.ldl;

  // ---- scores ----
  if (a.score_fn == MOE_SCORE_SOFTMAX) {
    float m = -INFINITY;
    for (int e = lane; e < E; e += 32) m = fmaxf(m, lg[e]);
    m = warp_max(m);
    float sum = 0.f;
    for (int e = lane; e < E; e += 32) {
      float v = expf(lg[e] - m);
      s[e] = v;
      sum += v;
    }
    sum = warp_sum(sum);
    for (int e = lane; e < E; e += 32) s[e] = s[e] / sum;
  } else {
    for (int e = lane; e < E; e += 32) s[e] = 1.f / (1.f + expf(-lg[e]));
  }
  for (int e = lane; e < E; e += 32) sel[e] = s[e] + (a.bias ? a.bias[e] : 0.f);
  __syncwarp();

  // ---- group limit ----
  if (a.n_group > 1) {
    const int G = a.n_group, gs = E / G;
    float gscore = -INFINITY;
    if (lane < G) {
      float m1 = -INFINITY, m2 = -INFINITY;
      for (int i = 0; i < gs; ++i) {
        float v = sel[lane * gs + i];
        if (v > m1) { m2 = m1; m1 = v; } else if (v > m2) { m2 = v; }
      }
      gscore = (a.group_score == MOE_GROUP_TOP2_SUM) ? (m1 + m2) : m1;
    }
    bool keep = false;
    float gv = (lane < G) ? gscore : -INFINITY;
    for (int r = 0; r < a.topk_group; ++r) {
      float v = (lane < G && !keep) ? gv : -INFINITY;
      int i = (lane < G && !keep) ? lane : 0x7fffffff;
      warp_argmax(v, i);
      if (lane == i) keep = true;
    }
    const unsigned keep_mask = __ballot_sync(0xffffffffu, keep);
    for (int e = lane; e < E; e += 32)
      if (!((keep_mask >> (e / gs)) & 1u)) sel[e] = -INFINITY;
    __syncwarp();
  }

  // ---- top-k ----
  int my_id = -1;
  for (int j = 0; j < a.k; ++j) {
    float v = -INFINITY;
    int i = 0x7fffffff;
    for (int e = lane; e < E; e += 32) {
      float x = sel[e];
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
