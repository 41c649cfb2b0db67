// elementwise.cu -- activation quantisation, row gather, weighted combine.
#include <algorithm>
#include "common.cuh"
#include "kernels.h"

namespace moe {

// ------------------------------------------------------------------ scatter
// Prefill: CTA per token -- quantise (FP8) / copy its row once into its k
// sorted rows and xq (shared expert).  Padding rows of the expert segments are
// left untouched: the GEMM rows they feed are never stored.
__global__ void __launch_bounds__(256) scatter_rows_kernel(const __nv_bfloat16 *__restrict__ x, int H, int k,
                                                           const int32_t *__restrict__ pos, ScatterDst d) {
  __shared__ int spos[32];
  const int t = blockIdx.x;
  if (threadIdx.x < k) spos[threadIdx.x] = pos[(int64_t)t * k + threadIdx.x];
  __syncthreads();
  scatter_token_row<256>(x + (size_t)t * H, H, t, k, spos, d);
}

cudaError_t launch_scatter_rows(const void *x, int T, int H, int k, const int32_t *pos, const ScatterDst &d,
                                cudaStream_t st) {
  if (T <= 0) return cudaSuccess;
  scatter_rows_kernel<<<T, 256, 0, st>>>(reinterpret_cast<const __nv_bfloat16 *>(x), H, k, pos, d);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ combine
// y[t]   = residual[t] + g_t * ys[t] + sum_{j < n_imm} w_tj * yperm[pos(t,j)] + deferred_in[t]
// dout[t] = sum_{j >= n_imm} w_tj * yperm[pos(t,j)]
// (PAPER.md L219 / L241; fp32 accumulation in slot order j = 0..k-1, one thread per 8 channels).
// KB > 0 (k <= KB): every operand row of the thread's 8 channels is loaded before any
// arithmetic, so each thread keeps up to KB + 3 16-byte loads in flight (HBM-bound kernel).
__device__ __forceinline__ uint4 ld_nc_v4(const void *p) {
  uint4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p));
  return v;
}

template <int KB>
__global__ void __launch_bounds__(128) combine_kernel(const __grid_constant__ CombineArgs a) {
  const int t = blockIdx.x;
  pdl_wait();
  __shared__ int32_t spos[32];
  __shared__ float sw[32];
  if (threadIdx.x < a.k) {
    spos[threadIdx.x] = a.pos[(int64_t)t * a.k + threadIdx.x];
    sw[threadIdx.x] = a.topk_w[(int64_t)t * a.k + threadIdx.x];
  }
  __syncthreads();
  const float g = a.sgate ? a.sgate[t] : 1.f;
  const int nvec = a.H / 8;
  const __nv_bfloat16 *yp = reinterpret_cast<const __nv_bfloat16 *>(a.yperm);
  for (int v = blockIdx.y * blockDim.x + threadIdx.x; v < nvec; v += gridDim.y * blockDim.x) {
    float acc[8], dacc[8], tmp[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) { acc[i] = 0.f; dacc[i] = 0.f; }
    const int64_t off = (int64_t)t * a.H + v * 8;
    const uint4 zero = make_uint4(0, 0, 0, 0);
    uint4 rres = zero, rsh = zero, rdin = zero;
    uint4 rows[KB > 0 ? KB : 1];
    if constexpr (KB > 0) {
#pragma unroll
      for (int j = 0; j < KB; ++j) {
        const int r = j < a.k ? spos[j] : -1;
        rows[j] = r >= 0 ? ld_nc_v4(yp + (int64_t)r * a.H + v * 8) : zero;
      }
    }
    if (a.residual) rres = ld_nc_v4(reinterpret_cast<const __nv_bfloat16 *>(a.residual) + off);
    if (a.ysh) rsh = ld_nc_v4(reinterpret_cast<const __nv_bfloat16 *>(a.ysh) + off);
    if (a.deferred_in) rdin = ld_nc_v4(reinterpret_cast<const __nv_bfloat16 *>(a.deferred_in) + off);
    if (a.residual) {
      bf16x8_to_f32(rres, tmp);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] += tmp[i];
    }
    if (a.ysh) {
      bf16x8_to_f32(rsh, tmp);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] = fmaf(g, tmp[i], acc[i]);
    }
    if constexpr (KB > 0) {
#pragma unroll
      for (int j = 0; j < KB; ++j) {
        if (j >= a.k || spos[j] < 0) continue;
        bf16x8_to_f32(rows[j], tmp);
        const float w = sw[j];
        if (j < a.n_imm) {
#pragma unroll
          for (int i = 0; i < 8; ++i) acc[i] = fmaf(w, tmp[i], acc[i]);
        } else {
#pragma unroll
          for (int i = 0; i < 8; ++i) dacc[i] = fmaf(w, tmp[i], dacc[i]);
        }
      }
    } else {
      for (int j = 0; j < a.k; ++j) {
        const int r = spos[j];
        if (r < 0) continue;
        bf16x8_to_f32(ld_nc_v4(yp + (int64_t)r * a.H + v * 8), tmp);
        const float w = sw[j];
        if (j < a.n_imm) {
#pragma unroll
          for (int i = 0; i < 8; ++i) acc[i] = fmaf(w, tmp[i], acc[i]);
        } else {
#pragma unroll
          for (int i = 0; i < 8; ++i) dacc[i] = fmaf(w, tmp[i], dacc[i]);
        }
      }
    }
    if (a.deferred_in) {
      bf16x8_to_f32(rdin, tmp);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] += tmp[i];
    }
    uint4 o;
    __nv_bfloat162 *op = reinterpret_cast<__nv_bfloat162 *>(&o);
#pragma unroll
    for (int i = 0; i < 4; ++i) op[i] = __floats2bfloat162_rn(acc[2 * i], acc[2 * i + 1]);
    *reinterpret_cast<uint4 *>(reinterpret_cast<__nv_bfloat16 *>(a.y) + off) = o;
    if (a.deferred_out) {
#pragma unroll
      for (int i = 0; i < 4; ++i) op[i] = __floats2bfloat162_rn(dacc[2 * i], dacc[2 * i + 1]);
      *reinterpret_cast<uint4 *>(reinterpret_cast<__nv_bfloat16 *>(a.deferred_out) + off) = o;
    }
  }
}

cudaError_t launch_combine(const CombineArgs &a, cudaStream_t st) {
  if (a.T <= 0) return cudaSuccess;
  // one CTA per (token, 1024 channels): enough CTAs to fill the GPU at T = 1
  const dim3 grid(a.T, (a.H / 8 + 127) / 128);
  if (a.k <= 8) return launch_pdl(combine_kernel<8>, grid, dim3(128), 0, st, a);
  return launch_pdl(combine_kernel<0>, grid, dim3(128), 0, st, a);
}

}  // namespace moe
