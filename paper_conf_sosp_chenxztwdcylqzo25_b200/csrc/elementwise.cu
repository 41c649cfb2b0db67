// elementwise.cu -- activation quantisation, row gather, weighted combine.
#include <algorithm>
#include "common.cuh"
#include "kernels.h"

namespace moe {

// ------------------------------------------------------------------ act quant
// Per token, per 128-channel block: s = UE8M0 ceil of amax/448, q = e4m3(x/s)
// (reading R10; north_star "128x128 block-scaled FP8" -- activations
// take the 1x128 granularity).  One warp per (row, block): 4 values per lane.
__global__ void __launch_bounds__(256) act_quant_kernel(const __nv_bfloat16 *__restrict__ x, int T, int H,
                                                        uint8_t *__restrict__ xq, float *__restrict__ xs,
                                                        uint8_t *__restrict__ img, int img_stride) {
  const int nb = H / 128;
  const int64_t total = (int64_t)T * nb;
  const int lane = threadIdx.x & 31;
  for (int64_t w = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5); w < total; w += (int64_t)gridDim.x * 8) {
    const int64_t row = w / nb, b = w % nb;
    const int64_t base = row * H + b * 128 + lane * 4;
    uint2 u = *reinterpret_cast<const uint2 *>(x + base);
    const __nv_bfloat162 *p = reinterpret_cast<const __nv_bfloat162 *>(&u);
    float2 v0 = __bfloat1622float2(p[0]), v1 = __bfloat1622float2(p[1]);
    float amax = fmaxf(fmaxf(fabsf(v0.x), fabsf(v0.y)), fmaxf(fabsf(v1.x), fabsf(v1.y)));
    amax = warp_max(amax);
    const int e = ue8m0_exponent(amax);
    const float inv = exp2i(-e);
    uint32_t q = (uint32_t)f32_to_e4m3(v0.x * inv) | ((uint32_t)f32_to_e4m3(v0.y * inv) << 8) |
                 ((uint32_t)f32_to_e4m3(v1.x * inv) << 16) | ((uint32_t)f32_to_e4m3(v1.y * inv) << 24);
    *reinterpret_cast<uint32_t *>(xq + base) = q;
    if (lane == 0) {
      xs[row * nb + b] = exp2i(e);
      if (img) img[sf_img_off(row, (int)b, img_stride)] = (uint8_t)(e + 127);
    }
  }
}

cudaError_t launch_act_quant(const void *x, int T, int H, void *xq, float *xs, uint8_t *img, int img_stride,
                             cudaStream_t st) {
  if (T <= 0) return cudaSuccess;
  const int64_t warps = (int64_t)T * (H / 128);
  const int grid = (int)std::min<int64_t>((warps + 7) / 8, 148 * 16);
  act_quant_kernel<<<grid, 256, 0, st>>>(reinterpret_cast<const __nv_bfloat16 *>(x), T, H,
                                         reinterpret_cast<uint8_t *>(xq), xs, img, img_stride);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ gather
// dst[r] = src[row_token[r]] for every padded row r < offs_pad[E]; pad rows zeroed.
__global__ void __launch_bounds__(256) gather_rows_kernel(const uint8_t *__restrict__ src,
                                                          const float *__restrict__ src_s, int row_bytes,
                                                          int nscale, const int32_t *__restrict__ row_token,
                                                          const int32_t *__restrict__ offs_pad, int E,
                                                          uint8_t *__restrict__ dst, float *__restrict__ dst_s,
                                                          uint8_t *__restrict__ dst_img, int img_stride) {
  const int64_t nrows = offs_pad[E];
  const int lane = threadIdx.x & 31;
  const int nvec = row_bytes / 16;
  for (int64_t r = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5); r < nrows; r += (int64_t)gridDim.x * 8) {
    const int t = row_token[r];
    uint4 *d = reinterpret_cast<uint4 *>(dst + r * row_bytes);
    if (t >= 0) {
      const uint4 *s = reinterpret_cast<const uint4 *>(src + (int64_t)t * row_bytes);
      for (int i = lane; i < nvec; i += 32) d[i] = __ldg(s + i);
      if (dst_s)
        for (int i = lane; i < nscale; i += 32) {
          const float s = src_s[(int64_t)t * nscale + i];
          dst_s[r * nscale + i] = s;
          if (dst_img) dst_img[sf_img_off(r, i, img_stride)] = (uint8_t)((__float_as_uint(s) >> 23) & 0xFF);
        }
    } else {
      for (int i = lane; i < nvec; i += 32) d[i] = make_uint4(0, 0, 0, 0);
      if (dst_s)
        for (int i = lane; i < nscale; i += 32) {
          dst_s[r * nscale + i] = 1.f;
          if (dst_img) dst_img[sf_img_off(r, i, img_stride)] = 127;
        }
    }
  }
}

cudaError_t launch_gather_rows(const void *src, const float *src_s, int H, int elem_bytes,
                               const int32_t *row_token, const int32_t *offs_pad, int E, int64_t R_bound,
                               void *dst, float *dst_s, uint8_t *dst_img, int img_stride, cudaStream_t st) {
  if (R_bound <= 0) return cudaSuccess;
  const int grid = (int)std::min<int64_t>((R_bound + 7) / 8, 148 * 8);
  gather_rows_kernel<<<grid, 256, 0, st>>>(reinterpret_cast<const uint8_t *>(src), src_s, H * elem_bytes,
                                           H / 128, row_token, offs_pad, E,
                                           reinterpret_cast<uint8_t *>(dst), dst_s, dst_img, img_stride);
  return cudaGetLastError();
}

// decode: FP8 quantisation + gather fused.  CTA per active expert slot: warp w
// quantises (or copies) token row w of the expert's segment into x_perm
// (rows >= count zeroed); the extra last CTA quantises all T tokens into xq for
// the shared expert.  Scale bytes go straight into the tcgen05 scale images.
// One warp quantises a row: all loads issued up front (lane l holds 8-element
// chunks c = 32 i + l), one 1x128 block = 16 lanes -> half-warp amax reduction.
__device__ __forceinline__ void quant_row_e4m3(const __nv_bfloat16 *__restrict__ src, uint8_t *__restrict__ dst,
                                               int H, int64_t row, uint8_t *img, int img_stride, float *xs_row,
                                               int lane) {
  constexpr int G = 16;                             // chunks per lane per batch (64 registers)
  const int nc = H / 8;
  for (int c0 = 0; c0 < nc; c0 += G * 32) {
  uint4 v[G];
#pragma unroll
  for (int i = 0; i < G; ++i) {
    const int c = c0 + i * 32 + lane;
    if (c < nc) v[i] = __ldg(reinterpret_cast<const uint4 *>(src) + c);
  }
#pragma unroll
  for (int i = 0; i < G; ++i) {
    if (c0 + i * 32 >= nc) break;
    const int c = c0 + i * 32 + lane;
    float f[8];
    bf16x8_to_f32(v[i], f);
    float am = 0.f;
#pragma unroll
    for (int j = 0; j < 8; ++j) am = fmaxf(am, fabsf(f[j]));
#pragma unroll
    for (int o = 8; o > 0; o >>= 1) am = fmaxf(am, __shfl_xor_sync(0xffffffffu, am, o));
    const int e = ue8m0_exponent(am);
    const float inv = exp2i(-e);
    uint2 q;
    q.x = (uint32_t)f32_to_e4m3(f[0] * inv) | ((uint32_t)f32_to_e4m3(f[1] * inv) << 8) |
          ((uint32_t)f32_to_e4m3(f[2] * inv) << 16) | ((uint32_t)f32_to_e4m3(f[3] * inv) << 24);
    q.y = (uint32_t)f32_to_e4m3(f[4] * inv) | ((uint32_t)f32_to_e4m3(f[5] * inv) << 8) |
          ((uint32_t)f32_to_e4m3(f[6] * inv) << 16) | ((uint32_t)f32_to_e4m3(f[7] * inv) << 24);
    if (c < nc) {
      *reinterpret_cast<uint2 *>(dst + c * 8) = q;
      if ((lane & 15) == 0) {
        const int b = c / 16;                       // 128-element block index
        if (img) img[sf_img_off(row, b, img_stride)] = (uint8_t)(e + 127);
        if (xs_row) xs_row[b] = exp2i(e);
      }
    }
  }
  }
}

__global__ void __launch_bounds__(512) quant_gather_decode_kernel(QuantGatherArgs a) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int H = a.H;
  const __nv_bfloat16 *x = reinterpret_cast<const __nv_bfloat16 *>(a.x);
  if ((int)blockIdx.x == a.max_slots) {            // shared expert: all tokens -> xq
    if (!a.xq) return;
    for (int t = warp; t < a.T; t += 16)
      quant_row_e4m3(x + (size_t)t * H, reinterpret_cast<uint8_t *>(a.xq) + (size_t)t * H, H, t, a.xq_img,
                     a.xq_img_stride, a.xs ? a.xs + (size_t)t * (H / 128) : nullptr, lane);
    return;
  }
  if ((int)blockIdx.x >= *a.n_active) return;
  const int e = a.act_list[blockIdx.x];
  const int64_t r = (int64_t)a.offs_pad[e] + warp;
  const int t = warp < a.counts[e] ? a.row_token[r] : -1;
  if (a.fp8) {
    uint8_t *d = reinterpret_cast<uint8_t *>(a.xperm) + r * H;
    if (t >= 0) {
      quant_row_e4m3(x + (size_t)t * H, d, H, r, a.xperm_img, a.xperm_img_stride, nullptr, lane);
    } else {
      for (int i = lane; i < H / 16; i += 32) reinterpret_cast<uint4 *>(d)[i] = make_uint4(0, 0, 0, 0);
      for (int b = lane; b < H / 128; b += 32) a.xperm_img[sf_img_off(r, b, a.xperm_img_stride)] = 127;
    }
  } else {
    uint4 *d = reinterpret_cast<uint4 *>(reinterpret_cast<__nv_bfloat16 *>(a.xperm) + r * H);
    const uint4 *sp = reinterpret_cast<const uint4 *>(x + (size_t)(t >= 0 ? t : 0) * H);
    for (int i = lane; i < H / 8; i += 32) d[i] = t >= 0 ? __ldg(sp + i) : make_uint4(0, 0, 0, 0);
  }
}

cudaError_t launch_quant_gather_decode(const QuantGatherArgs &a, cudaStream_t st) {
  if (a.T <= 0) return cudaSuccess;
  quant_gather_decode_kernel<<<a.max_slots + 1, 512, 0, st>>>(a);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ combine
// y[t]   = residual[t] + g_t * ys[t] + sum_{j < n_imm} w_tj * yperm[pos(t,j)] + deferred_in[t]
// dout[t] = sum_{j >= n_imm} w_tj * yperm[pos(t,j)]
// (PAPER.md L219 / L241; fp32 accumulation, one CTA per token, 8 channels per thread)
__global__ void __launch_bounds__(128) combine_kernel(CombineArgs a) {
  const int t = blockIdx.x;
  __shared__ int32_t spos[32];
  __shared__ float sw[32];
  if (threadIdx.x < a.k) {
    spos[threadIdx.x] = a.pos[(int64_t)t * a.k + threadIdx.x];
    sw[threadIdx.x] = a.topk_w[(int64_t)t * a.k + threadIdx.x];
  }
  __syncthreads();
  const float g = a.sgate ? a.sgate[t] : 1.f;
  const int nvec = a.H / 8;
  for (int v = blockIdx.y * blockDim.x + threadIdx.x; v < nvec; v += gridDim.y * blockDim.x) {
    float acc[8], dacc[8], tmp[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) { acc[i] = 0.f; dacc[i] = 0.f; }
    const int64_t off = (int64_t)t * a.H + v * 8;
    if (a.residual) {
      bf16x8_to_f32(*reinterpret_cast<const uint4 *>(reinterpret_cast<const __nv_bfloat16 *>(a.residual) + off), tmp);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] += tmp[i];
    }
    if (a.ysh) {
      bf16x8_to_f32(*reinterpret_cast<const uint4 *>(reinterpret_cast<const __nv_bfloat16 *>(a.ysh) + off), tmp);
#pragma unroll
      for (int i = 0; i < 8; ++i) acc[i] = fmaf(g, tmp[i], acc[i]);
    }
    for (int j = 0; j < a.k; ++j) {
      const int r = spos[j];
      if (r < 0) continue;
      bf16x8_to_f32(*reinterpret_cast<const uint4 *>(reinterpret_cast<const __nv_bfloat16 *>(a.yperm) +
                                                      (int64_t)r * a.H + v * 8), tmp);
      const float w = sw[j];
      if (j < a.n_imm) {
#pragma unroll
        for (int i = 0; i < 8; ++i) acc[i] = fmaf(w, tmp[i], acc[i]);
      } else {
#pragma unroll
        for (int i = 0; i < 8; ++i) dacc[i] = fmaf(w, tmp[i], dacc[i]);
      }
    }
    if (a.deferred_in) {
      bf16x8_to_f32(*reinterpret_cast<const uint4 *>(reinterpret_cast<const __nv_bfloat16 *>(a.deferred_in) + off), tmp);
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
  combine_kernel<<<dim3(a.T, (a.H / 8 + 127) / 128), 128, 0, st>>>(a);
  return cudaGetLastError();
}

}  // namespace moe
