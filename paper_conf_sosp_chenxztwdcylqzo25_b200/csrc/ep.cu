// ep.cu -- expert parallelism: dispatch plan, pack, final combine kernels and
// the NCCL / in-process transports.
//
// Rank r of P owns experts [r E/P, (r+1) E/P) (Fig. 8a, EP as
// the deployment the paper contrasts with its NUMA TP).  Each rank routes its
// own tokens, sends every token row ONCE to each rank owning >= 1 of its k
// experts (with the k expert ids masked to that rank and the combine weights),
// the expert side runs the routed FFNs on the received rows and returns one
// pre-reduced partial row per (token, rank); the origin adds the partials, its
// shared expert output and the residual.
#include <nccl.h>

#include <cstring>

#include <cub/block/block_scan.cuh>

#include "common.cuh"
#include "kernels.h"

namespace moe {

// ------------------------------------------------------------------ plan
// single CTA: sendpos[t][d] = position of token t in the send list of rank d
// (-1 if none of t's experts lives on d), lists in token order; cnt[d] totals.
constexpr int EP_PLAN_THREADS = 1024;
__global__ void __launch_bounds__(EP_PLAN_THREADS) ep_plan_kernel(const int32_t *__restrict__ idx, int T, int k,
                                                                  int E_loc, int P, int32_t *__restrict__ sendpos,
                                                                  int32_t *__restrict__ cnt) {
  using Scan = cub::BlockScan<int, EP_PLAN_THREADS>;
  __shared__ typename Scan::TempStorage tmp;
  const int per = (T + EP_PLAN_THREADS - 1) / EP_PLAN_THREADS;
  const int t0 = threadIdx.x * per, t1 = min(T, t0 + per);
  for (int d = 0; d < P; ++d) {
    int c = 0;
    for (int t = t0; t < t1; ++t) {
      bool need = false;
      for (int j = 0; j < k; ++j) need |= (idx[(int64_t)t * k + j] / E_loc) == d;
      c += need;
    }
    int base, tot;
    Scan(tmp).ExclusiveSum(c, base, tot);
    __syncthreads();
    for (int t = t0; t < t1; ++t) {
      bool need = false;
      for (int j = 0; j < k; ++j) need |= (idx[(int64_t)t * k + j] / E_loc) == d;
      sendpos[(int64_t)t * P + d] = need ? base++ : -1;
    }
    if (threadIdx.x == 0) cnt[d] = tot;
  }
}

// ------------------------------------------------------------------ pack
// CTA per token: its bf16 row and metadata into the send list of every rank it needs
__global__ void __launch_bounds__(128) ep_pack_kernel(const __nv_bfloat16 *__restrict__ x, int H, int k,
                                                      const int32_t *__restrict__ idx, const float *__restrict__ w,
                                                      int E_loc, int P, int Tm, const int32_t *__restrict__ sendpos,
                                                      __nv_bfloat16 *__restrict__ send_x, int32_t *__restrict__ send_idx,
                                                      float *__restrict__ send_w) {
  const int t = blockIdx.x;
  const uint4 *src = reinterpret_cast<const uint4 *>(x + (size_t)t * H);
  for (int d = 0; d < P; ++d) {
    const int sp = sendpos[(int64_t)t * P + d];
    if (sp < 0) continue;
    const int64_t row = (int64_t)d * Tm + sp;
    uint4 *dst = reinterpret_cast<uint4 *>(send_x + row * H);
    for (int c = threadIdx.x; c < H / 8; c += blockDim.x) dst[c] = __ldg(src + c);
    if (threadIdx.x < k) {
      const int e = idx[(int64_t)t * k + threadIdx.x];
      send_idx[row * k + threadIdx.x] = (e / E_loc) == d ? e : -1;
      send_w[row * k + threadIdx.x] = w[(int64_t)t * k + threadIdx.x];
    }
  }
}

// FP8 layers: the token's e4m3 row (quantised once on the origin, 1x128 UE8M0, reading
// R10) + its H/128 exponent bytes -- H + H/128 bytes instead of 2H (round-2 EP v2)
__global__ void __launch_bounds__(128) ep_pack_fp8_kernel(const uint8_t *__restrict__ xq, const float *__restrict__ xs,
                                                          int H, int k, const int32_t *__restrict__ idx,
                                                          const float *__restrict__ w, int E_loc, int P, int Tm,
                                                          int row_bytes, const int32_t *__restrict__ sendpos,
                                                          uint8_t *__restrict__ send_x, int32_t *__restrict__ send_idx,
                                                          float *__restrict__ send_w) {
  const int t = blockIdx.x;
  const uint4 *src = reinterpret_cast<const uint4 *>(xq + (size_t)t * H);
  for (int d = 0; d < P; ++d) {
    const int sp = sendpos[(int64_t)t * P + d];
    if (sp < 0) continue;
    const int64_t row = (int64_t)d * Tm + sp;
    uint8_t *dst = send_x + row * row_bytes;
    for (int c = threadIdx.x; c < H / 16; c += blockDim.x) reinterpret_cast<uint4 *>(dst)[c] = __ldg(src + c);
    for (int b = threadIdx.x; b < H / 128; b += blockDim.x)
      dst[H + b] = (uint8_t)((__float_as_uint(xs[(size_t)t * (H / 128) + b]) >> 23) & 0xFF);
    if (threadIdx.x < k) {
      const int e = idx[(int64_t)t * k + threadIdx.x];
      send_idx[row * k + threadIdx.x] = (e / E_loc) == d ? e : -1;
      send_w[row * k + threadIdx.x] = w[(int64_t)t * k + threadIdx.x];
    }
  }
}

// expert side, FP8: a received row's codes into its k sorted rows (pos, -1 = not local)
// and its exponents into their scale images (one 32-bit word per 4 k-blocks, sf_img_off)
__global__ void __launch_bounds__(128) ep_scatter_fp8_kernel(const uint8_t *__restrict__ recv, int H, int k,
                                                             int row_bytes, const int32_t *__restrict__ pos,
                                                             uint8_t *__restrict__ xperm, uint8_t *__restrict__ img,
                                                             int img_stride) {
  const int r = blockIdx.x;
  __shared__ int sp[32];
  if (threadIdx.x < k) sp[threadIdx.x] = pos[(int64_t)r * k + threadIdx.x];
  __syncthreads();
  const uint8_t *src = recv + (int64_t)r * row_bytes;
  const int nb = H / 128, ng = (nb + 3) / 4;
  for (int j = 0; j < k; ++j) {
    const int rw = sp[j];
    if (rw < 0) continue;
    uint4 *dst = reinterpret_cast<uint4 *>(xperm + (int64_t)rw * H);
    for (int c = threadIdx.x; c < H / 16; c += blockDim.x) dst[c] = reinterpret_cast<const uint4 *>(src)[c];
    for (int g = threadIdx.x; g < ng; g += blockDim.x) {
      uint32_t wd = 0;
      for (int q = 0; q < 4; ++q) wd |= (4 * g + q < nb ? (uint32_t)src[H + 4 * g + q] : 127u) << (8 * q);
      *reinterpret_cast<uint32_t *>(img + sf_img_off(rw, 4 * g, img_stride)) = wd;
    }
  }
}

// expert side, FP8 decode: received rows in arrival order -> e4m3 codes [R, H] (the fused
// decode stream's token operand) + fp32 scales [R, H/128] (2^(e - 127) from the UE8M0 bytes)
__global__ void __launch_bounds__(128) ep_unpack_fp8_kernel(const uint8_t *__restrict__ recv, int H, int row_bytes,
                                                            uint8_t *__restrict__ xq, float *__restrict__ xs) {
  const int r = blockIdx.x;
  const uint8_t *src = recv + (int64_t)r * row_bytes;
  uint4 *dst = reinterpret_cast<uint4 *>(xq + (int64_t)r * H);
  for (int c = threadIdx.x; c < H / 16; c += blockDim.x) dst[c] = reinterpret_cast<const uint4 *>(src)[c];
  for (int b = threadIdx.x; b < H / 128; b += blockDim.x) xs[(int64_t)r * (H / 128) + b] = exp2i((int)src[H + b] - 127);
}

cudaError_t launch_ep_unpack_fp8(const void *recv, int R, int H, int row_bytes, void *xq, float *xs, cudaStream_t st) {
  if (R <= 0) return cudaSuccess;
  ep_unpack_fp8_kernel<<<R, 128, 0, st>>>(reinterpret_cast<const uint8_t *>(recv), H, row_bytes,
                                          reinterpret_cast<uint8_t *>(xq), xs);
  return cudaGetLastError();
}

cudaError_t launch_ep_pack_fp8(const void *xq, const float *xs, int T, int H, int k, const int32_t *idx,
                               const float *w, int E_loc, int P, int Tm, int row_bytes, const int32_t *sendpos,
                               void *send_x, int32_t *send_idx, float *send_w, cudaStream_t st) {
  if (T <= 0) return cudaSuccess;
  ep_pack_fp8_kernel<<<T, 128, 0, st>>>(reinterpret_cast<const uint8_t *>(xq), xs, H, k, idx, w, E_loc, P, Tm,
                                        row_bytes, sendpos, reinterpret_cast<uint8_t *>(send_x), send_idx, send_w);
  return cudaGetLastError();
}

cudaError_t launch_ep_scatter_fp8(const void *recv, int R, int H, int k, int row_bytes, const int32_t *pos,
                                  void *xperm, uint8_t *img, int img_stride, cudaStream_t st) {
  if (R <= 0) return cudaSuccess;
  ep_scatter_fp8_kernel<<<R, 128, 0, st>>>(reinterpret_cast<const uint8_t *>(recv), H, k, row_bytes, pos,
                                           reinterpret_cast<uint8_t *>(xperm), img, img_stride);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ final combine
// y[t] = residual + g_t * ys[t] + sum_d back[d][sendpos[t][d]] + deferred_in;
// deferred_out[t] = sum_d back_def[d][sendpos[t][d]]   (fp32 accumulation)
__global__ void __launch_bounds__(128) ep_final_combine_kernel(const __grid_constant__ EpCombineArgs a) {
  const int t = blockIdx.x;
  const int v = blockIdx.y * blockDim.x + threadIdx.x;
  if (v >= a.H / 8) return;
  const float g = a.sgate ? a.sgate[t] : 1.f;
  float acc[8], dacc[8], tmp[8];
#pragma unroll
  for (int i = 0; i < 8; ++i) { acc[i] = 0.f; dacc[i] = 0.f; }
  const int64_t off = (int64_t)t * a.H + v * 8;
  auto add = [&](const __nv_bfloat16 *p, float s, float *dst) {
    bf16x8_to_f32(*reinterpret_cast<const uint4 *>(p), tmp);
#pragma unroll
    for (int i = 0; i < 8; ++i) dst[i] = fmaf(s, tmp[i], dst[i]);
  };
  if (a.residual) add(a.residual + off, 1.f, acc);
  if (a.ysh) add(a.ysh + off, g, acc);
  for (int d = 0; d < a.P; ++d) {
    const int sp = a.sendpos[(int64_t)t * a.P + d];
    if (sp < 0) continue;
    const int64_t row = (int64_t)d * a.Tm + sp;
    add(a.back + row * a.H + v * 8, 1.f, acc);
    if (a.back_def) add(a.back_def + row * a.H + v * 8, 1.f, dacc);
  }
  if (a.deferred_in) add(a.deferred_in + off, 1.f, acc);
  uint4 o;
  __nv_bfloat162 *op = reinterpret_cast<__nv_bfloat162 *>(&o);
#pragma unroll
  for (int i = 0; i < 4; ++i) op[i] = __floats2bfloat162_rn(acc[2 * i], acc[2 * i + 1]);
  *reinterpret_cast<uint4 *>(a.y + off) = o;
  if (a.deferred_out) {
#pragma unroll
    for (int i = 0; i < 4; ++i) op[i] = __floats2bfloat162_rn(dacc[2 * i], dacc[2 * i + 1]);
    *reinterpret_cast<uint4 *>(a.deferred_out + off) = o;
  }
}

cudaError_t launch_ep_plan(const int32_t *idx, int T, int k, int E_loc, int P, int32_t *sendpos, int32_t *cnt,
                           cudaStream_t st) {
  if (T <= 0) return cudaMemsetAsync(cnt, 0, P * sizeof(int32_t), st);
  ep_plan_kernel<<<1, EP_PLAN_THREADS, 0, st>>>(idx, T, k, E_loc, P, sendpos, cnt);
  return cudaGetLastError();
}

cudaError_t launch_ep_pack(const void *x, int T, int H, int k, const int32_t *idx, const float *w, int E_loc, int P,
                           int Tm, const int32_t *sendpos, void *send_x, int32_t *send_idx, float *send_w,
                           cudaStream_t st) {
  if (T <= 0) return cudaSuccess;
  ep_pack_kernel<<<T, 128, 0, st>>>(reinterpret_cast<const __nv_bfloat16 *>(x), H, k, idx, w, E_loc, P, Tm, sendpos,
                                    reinterpret_cast<__nv_bfloat16 *>(send_x), send_idx, send_w);
  return cudaGetLastError();
}

cudaError_t launch_ep_final_combine(const EpCombineArgs &a, cudaStream_t st) {
  if (a.T <= 0) return cudaSuccess;
  ep_final_combine_kernel<<<dim3(a.T, (a.H / 8 + 127) / 128), 128, 0, st>>>(a);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ NCCL transport
int ep_nccl_get_unique_id(void *out128) {
  ncclUniqueId id;
  if (ncclGetUniqueId(&id) != ncclSuccess) return -1;
  memcpy(out128, &id, sizeof(id));
  return 0;
}

int ep_nccl_init(void **comm, int P, int rank, const void *uid128) {
  ncclUniqueId id;
  memcpy(&id, uid128, sizeof(id));
  ncclComm_t c;
  if (ncclCommInitRank(&c, P, id, rank) != ncclSuccess) return -1;
  *comm = c;
  return 0;
}

void ep_nccl_destroy(void *comm) {
  if (comm) ncclCommDestroy(reinterpret_cast<ncclComm_t>(comm));
}

const char *ep_nccl_error(void *comm) {
  ncclResult_t async;
  if (comm && ncclCommGetAsyncError(reinterpret_cast<ncclComm_t>(comm), &async) == ncclSuccess && async != ncclSuccess)
    return ncclGetErrorString(async);
  return "";
}

int ep_nccl_allreduce_f32(void *comm, float *buf, size_t n, cudaStream_t st) {
  return ncclAllReduce(buf, buf, n, ncclFloat32, ncclSum, reinterpret_cast<ncclComm_t>(comm), st) == ncclSuccess ? 0 : -1;
}

struct SumSrc { const float *p[31]; };
__global__ void sum_f32_kernel(float *__restrict__ dst, const __grid_constant__ SumSrc src, int nsrc, int64_t n) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    float v = dst[i];
    for (int j = 0; j < nsrc; ++j) v += src.p[j][i];
    dst[i] = v;
  }
}

cudaError_t launch_sum_f32(float *dst, const float *const *src, int nsrc, int64_t n, cudaStream_t st) {
  if (n <= 0 || nsrc <= 0) return cudaSuccess;
  if (nsrc > 31) return cudaErrorInvalidValue;
  SumSrc s{};
  for (int j = 0; j < nsrc; ++j) s.p[j] = src[j];
  sum_f32_kernel<<<(int)std::min<int64_t>((n + 255) / 256, 148 * 4), 256, 0, st>>>(dst, s, nsrc, n);
  return cudaGetLastError();
}

// exchange of the P send counts (one int32 to every peer)
int ep_nccl_counts(void *comm, const int32_t *send_cnt, int32_t *recv_cnt, int P, cudaStream_t st) {
  ncclComm_t c = reinterpret_cast<ncclComm_t>(comm);
  if (ncclGroupStart() != ncclSuccess) return -1;
  bool ok = true;                       // the group is always closed, even after a failed call
  for (int p = 0; p < P && ok; ++p) {
    ok = ncclSend(send_cnt + p, 1, ncclInt32, p, c, st) == ncclSuccess;
    ok = ok && ncclRecv(recv_cnt + p, 1, ncclInt32, p, c, st) == ncclSuccess;
  }
  const bool closed = ncclGroupEnd() == ncclSuccess;
  return ok && closed ? 0 : -1;
}

// all-to-all-v of up to 3 row-major buffers (bytes per row each): send_cnt[p]
// rows from row send_off[p] go to peer p, recv_cnt[p] rows from peer p land at
// row recv_off[p]
int ep_nccl_rows(void *comm, int P, const int32_t *send_cnt, const int64_t *send_off, const int32_t *recv_cnt,
                 const int64_t *recv_off, int nbuf, const void *const *send, void *const *recv,
                 const int64_t *row_bytes, cudaStream_t st) {
  ncclComm_t c = reinterpret_cast<ncclComm_t>(comm);
  if (ncclGroupStart() != ncclSuccess) return -1;
  bool ok = true;                       // the group is always closed, even after a failed call
  for (int p = 0; p < P && ok; ++p)
    for (int b = 0; b < nbuf && ok; ++b) {
      const char *sp = reinterpret_cast<const char *>(send[b]) + send_off[p] * row_bytes[b];
      char *rp = reinterpret_cast<char *>(recv[b]) + (int64_t)recv_off[p] * row_bytes[b];
      if (send_cnt[p]) ok = ncclSend(sp, (size_t)send_cnt[p] * row_bytes[b], ncclUint8, p, c, st) == ncclSuccess;
      if (ok && recv_cnt[p]) ok = ncclRecv(rp, (size_t)recv_cnt[p] * row_bytes[b], ncclUint8, p, c, st) == ncclSuccess;
    }
  const bool closed = ncclGroupEnd() == ncclSuccess;
  return ok && closed ? 0 : -1;
}

}  // namespace moe
