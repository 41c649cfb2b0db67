// CUDA-core FP8 weight stream for T = 1 (evidence for the decode-TP next step,
// DESIGN.md §7.1): per-SM bytes/s of y = W x with W e4m3 [rows, K] row-major and
// x fp32 in shared memory, when only G CTAs (one per SM) stream.  The fused
// tensor-core decode stream is capped at ~55 GB/s per SM at N = 16 by the MMA
// issue rate; this measures what plain FMA code reaches per SM.
//   mode 0: e4m3x2 -> f16x2 (cvt), -> f32 (cvt), FFMA into fp32 accumulators
//   mode 1: e4m3x2 -> f16x2, HFMA2 against f16x2 x over 16 bytes, then f32 adds
// Each warp owns rows; lanes stride K in 16-byte loads, D = 4 / 14 loads in flight per lane.
#include <cuda_fp16.h>
#include <cuda_fp8.h>
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int K = 7168, THREADS = 512;

__device__ __forceinline__ __half2 e4m3x2_to_h2(uint16_t v) {
  uint32_t r;
  asm("cvt.rn.f16x2.e4m3x2 %0, %1;" : "=r"(r) : "h"(v));
  return *reinterpret_cast<__half2 *>(&r);
}

template <int MODE, int D>
__global__ void __launch_bounds__(THREADS, 1) gemv(const uint8_t *W, int rows_per_cta, float *y) {
  __shared__ float xs[K];
  __shared__ __half2 xh[K / 2];
  for (int i = threadIdx.x; i < K; i += THREADS) xs[i] = 1.0f / (1 + (i & 7));
  for (int i = threadIdx.x; i < K / 2; i += THREADS) xh[i] = __floats2half2_rn(xs[2 * i], xs[2 * i + 1]);
  __syncthreads();
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int r0 = blockIdx.x * rows_per_cta;
  for (int r = warp; r < rows_per_cta; r += THREADS / 32) {
    const uint4 *wr = reinterpret_cast<const uint4 *>(W + (size_t)(r0 + r) * K);
    float acc = 0.f;
#pragma unroll 1
    for (int c = lane; c < K / 16; c += 32 * D) {
      uint4 u[D];
#pragma unroll
      for (int j = 0; j < D; ++j) u[j] = (c + 32 * j < K / 16) ? __ldcs(wr + c + 32 * j) : make_uint4(0, 0, 0, 0);
#pragma unroll
      for (int j = 0; j < D; ++j) {
        const int k0 = (c + 32 * j) * 16;
        if (k0 >= K) break;
        const uint32_t w4[4] = {u[j].x, u[j].y, u[j].z, u[j].w};
        if (MODE == 0) {
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            float2 a = __half22float2(e4m3x2_to_h2((uint16_t)(w4[q] & 0xFFFF)));
            float2 b = __half22float2(e4m3x2_to_h2((uint16_t)(w4[q] >> 16)));
            acc = fmaf(a.x, xs[k0 + 4 * q], acc); acc = fmaf(a.y, xs[k0 + 4 * q + 1], acc);
            acc = fmaf(b.x, xs[k0 + 4 * q + 2], acc); acc = fmaf(b.y, xs[k0 + 4 * q + 3], acc);
          }
        } else {
          __half2 h = __float2half2_rn(0.f);
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            h = __hfma2(e4m3x2_to_h2((uint16_t)(w4[q] & 0xFFFF)), xh[k0 / 2 + 2 * q], h);
            h = __hfma2(e4m3x2_to_h2((uint16_t)(w4[q] >> 16)), xh[k0 / 2 + 2 * q + 1], h);
          }
          float2 f = __half22float2(h);
          acc += f.x + f.y;
        }
      }
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffff, acc, o);
    if (lane == 0) y[r0 + r] = acc;
  }
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const size_t bytes = (size_t)2 << 30;
  const int rows_total = (int)(bytes / K);
  uint8_t *W;
  float *y;
  cudaMalloc(&W, bytes);
  cudaMemset(W, 0x38, bytes);   // e4m3 1.0
  cudaMalloc(&y, rows_total * sizeof(float));
  uint8_t *fl;
  cudaMalloc(&fl, 256 << 20);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  printf("mode (0/1: D=4, 2/3: D=14, even FFMA, odd HFMA2) grid rows_per_cta MB_per_cta us GB/s_total GB/s_per_SM\n");
  for (int mode = 0; mode < 4; ++mode) {
    for (int grid : {18, 37, 74, sms}) {
      for (int rpc : {128, 256, 512}) {
        if ((size_t)grid * rpc > (size_t)rows_total) continue;
        float best = 1e30f;
        for (int it = 0; it < 5; ++it) {
          cudaMemset(fl, it, 256 << 20);   // flush L2
          cudaEventRecord(e0);
          if (mode == 0) gemv<0, 4><<<grid, THREADS>>>(W, rpc, y);
          else if (mode == 1) gemv<1, 4><<<grid, THREADS>>>(W, rpc, y);
          else if (mode == 2) gemv<0, 14><<<grid, THREADS>>>(W, rpc, y);
          else gemv<1, 14><<<grid, THREADS>>>(W, rpc, y);
          cudaEventRecord(e1);
          cudaEventSynchronize(e1);
          float ms;
          cudaEventElapsedTime(&ms, e0, e1);
          if (it > 0 && ms < best) best = ms;
        }
        const double b = (double)grid * rpc * K;
        printf("%d %4d %4d %6.2f %8.1f %8.1f %7.1f\n", mode, grid, rpc, rpc * (double)K / 1e6, best * 1e3,
               b / (best * 1e-3) / 1e9, b / (best * 1e-3) / 1e9 / grid);
      }
    }
  }
  cudaError_t e = cudaGetLastError();
  printf("status %s\n", cudaGetErrorString(e));
  return 0;
}
