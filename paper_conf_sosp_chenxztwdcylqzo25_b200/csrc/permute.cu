// permute.cu -- token->expert count, prefix sum and stable permutation.
//
// Groups the (token, slot) pairs by expert so each expert's rows are one
// contiguous GEMM operand -- the "co-scheduling tasks targeting the same
// expert" of PAPER.md L181 and the per-expert batches of the fused MoE
// operator (L179).  Deterministic without atomics on the ordering path
// (DESIGN.md §5): the sorted order is (expert, token), each expert segment is
// padded to kPadM rows so the GEMM's M tiles never straddle two experts, and
// a work list of (expert, 128-row tile) units is written for the GEMMs (the
// device-side analog of the paper's dynamic task queue, L181).
#include <cub/block/block_scan.cuh>

#include "common.cuh"
#include "kernels.h"

namespace moe {

// (1) per-chunk histogram (order-free, smem atomics) + reset pos to -1
__global__ void __launch_bounds__(256) chunk_count_kernel(const __grid_constant__ PermuteArgs a) {
  extern __shared__ int32_t hist[];
  const int c = blockIdx.x;
  for (int e = threadIdx.x; e < a.E; e += blockDim.x) hist[e] = 0;
  __syncthreads();
  const int t0 = c * kChunkTokens;
  const int t1 = min(a.T, t0 + kChunkTokens);
  for (int p = t0 * a.k + threadIdx.x; p < t1 * a.k; p += blockDim.x) {
    const int e = a.topk_idx[p] - a.e0;
    a.pos[p] = -1;
    if (e >= 0 && e < a.E) atomicAdd(&hist[e], 1);
  }
  __syncthreads();
  for (int e = threadIdx.x; e < a.E; e += blockDim.x) a.chunk_cnt[(int64_t)c * a.E + e] = hist[e];
}

// (2) single CTA: per-expert totals, chunk bases, padded offsets, tile list
constexpr int SCAN_THREADS = 1024;
__global__ void __launch_bounds__(SCAN_THREADS) scan_kernel(const __grid_constant__ PermuteArgs a, int nchunk) {
  using Scan = cub::BlockScan<int, SCAN_THREADS>;
  __shared__ typename Scan::TempStorage tmp;
  __shared__ int tot[3];
  const int e = threadIdx.x;   // E <= 1024 (validated at create)
  int cnt = 0;
  if (e < a.E) {
    // chunk counts loaded 8 at a time (independent loads in flight) before the
    // running sum -- a load per step serialised nchunk L2 round trips
    for (int c0 = 0; c0 < nchunk; c0 += 8) {
      int v[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) v[j] = c0 + j < nchunk ? a.chunk_cnt[(int64_t)(c0 + j) * a.E + e] : 0;
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        if (c0 + j < nchunk) a.chunk_base[(int64_t)(c0 + j) * a.E + e] = cnt;
        cnt += v[j];
      }
    }
  }
  const int padded = (cnt + kPadM - 1) / kPadM * kPadM;
  int off, off_pad, tile_off, act_off, total;
  Scan(tmp).ExclusiveSum(cnt, off, total);
  __syncthreads();
  if (e == 0) tot[0] = total;
  Scan(tmp).ExclusiveSum(padded, off_pad, total);
  __syncthreads();
  if (e == 0) tot[1] = total;
  const int ntile = padded / kPadM;
  Scan(tmp).ExclusiveSum(ntile, tile_off, total);
  __syncthreads();
  if (e == 0) { *a.n_tiles = total; }
  Scan(tmp).ExclusiveSum(cnt > 0 ? 1 : 0, act_off, total);
  if (e == 0) *a.n_active = total;
  __syncthreads();
  // 2-CTA work list: pairs of consecutive 128-row tiles of one expert
  const int npair = (ntile + 1) / 2;
  int pair_off;
  Scan(tmp).ExclusiveSum(npair, pair_off, total);
  if (e == 0 && a.n_pairs) *a.n_pairs = total;
  __syncthreads();
  if (e < a.E) {
    a.counts[e] = cnt;
    if (a.dbg_counts) a.dbg_counts[e] = cnt;
    a.offs[e] = off;
    a.offs_pad[e] = off_pad;
    for (int m = 0; m < ntile; ++m)
      a.tiles[tile_off + m] = make_int4(e, off_pad + m * kPadM, off_pad + cnt, tile_off | (ntile << 16));
    if (a.pairs)
      for (int m = 0; m < npair; ++m)
        a.pairs[pair_off + m] = make_int4(e, off_pad + m * 2 * kPadM, off_pad + cnt, pair_off | (npair << 16));
    if (cnt > 0) a.act_list[act_off] = e;
  }
  if (e == 0) {
    a.offs[a.E] = tot[0];
    a.offs_pad[a.E] = tot[1];
  }
}

// (3) per chunk: assign rows in token order (stable).  Each expert gets a
// bitmask of the chunk's tokens that chose it; an entry's rank among the
// chunk's rows of its expert is the popcount of the mask below its token.
constexpr int kMaskWords = kChunkTokens / 32;
__global__ void __launch_bounds__(256) assign_kernel(const __grid_constant__ PermuteArgs a) {
  extern __shared__ uint32_t mask[];             // [E][kMaskWords]
  const int c = blockIdx.x;
  const int t0 = c * kChunkTokens;
  const int t1 = min(a.T, t0 + kChunkTokens);
  const int n = (t1 - t0) * a.k;
  for (int i = threadIdx.x; i < a.E * kMaskWords; i += blockDim.x) mask[i] = 0;
  __syncthreads();
  for (int p = threadIdx.x; p < n; p += blockDim.x) {
    const int e = a.topk_idx[(int64_t)t0 * a.k + p] - a.e0;
    const int tl = p / a.k;
    if (e >= 0 && e < a.E) atomicOr(&mask[e * kMaskWords + (tl >> 5)], 1u << (tl & 31));
  }
  __syncthreads();
  for (int p = threadIdx.x; p < n; p += blockDim.x) {
    const int e = a.topk_idx[(int64_t)t0 * a.k + p] - a.e0;
    if (e < 0 || e >= a.E) continue;
    const int tl = p / a.k;
    const uint32_t *m = mask + e * kMaskWords;
    int rank = __popc(m[tl >> 5] & ((1u << (tl & 31)) - 1u));
    for (int w = 0; w < (tl >> 5); ++w) rank += __popc(m[w]);
    const int cb = a.chunk_base[(int64_t)c * a.E + e] + rank;
    const int r = a.offs_pad[e] + cb;
    a.row_token[r] = t0 + tl;
    a.pos[(int64_t)t0 * a.k + p] = r;
    if (a.dbg_perm) a.dbg_perm[a.offs[e] + cb] = t0 + tl;
  }
  // the last chunk clears the padding rows of every expert segment
  if (c == gridDim.x - 1)
    for (int e = threadIdx.x; e < a.E; e += blockDim.x) {
      const int end = a.offs_pad[e + 1];
      for (int q = a.offs_pad[e] + a.counts[e]; q < end; ++q) a.row_token[q] = -1;
    }
}

cudaError_t launch_permute(const PermuteArgs &a, cudaStream_t st) {
  const int nchunk = (a.T + kChunkTokens - 1) / kChunkTokens;
  if (nchunk == 0) return cudaSuccess;
  chunk_count_kernel<<<nchunk, 256, a.E * sizeof(int32_t), st>>>(a);
  scan_kernel<<<1, SCAN_THREADS, 0, st>>>(a, nchunk);
  const size_t sm = (size_t)a.E * kMaskWords * sizeof(uint32_t);
  if (sm > 48 * 1024) {
    cudaError_t e = set_kernel_attr((const void *)assign_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
  }
  assign_kernel<<<nchunk, 256, sm, st>>>(a);
  return cudaGetLastError();
}

}  // namespace moe
