// tcgen05 MMA issue rate, single CTA (cta_group::1), kind::f8f6f4 (unscaled FP8), M x N x 32
// back to back on fixed shared-memory operands, one CTA per SM (which
// orientation streams decode weights faster per SM -- weights as the M operand with the
// <= 16 tokens as N (the shipped swap-AB stream), or weights as the N operand with the
// tokens padded to M = 64 / 128).  Prints ns and cycles per MMA and the weight bytes per
// cycle of each orientation.
#include <cstdio>
#include <cuda.h>
#include <cuda_runtime.h>
#include "../../paper_conf_sosp_chenxztwdcylqzo25_b200/csrc/sm100.cuh"
using namespace moe::sm100;

__device__ __forceinline__ void mma_f8(uint32_t d, uint64_t a, uint64_t b, uint32_t id) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, 1, 0;\n\t"
               "tcgen05.mma.cta_group::1.kind::f8f6f4 [%0], %1, %2, %3, p;\n\t}" ::"r"(d), "l"(a), "l"(b), "r"(id)
               : "memory");
}
__host__ __device__ constexpr uint32_t idesc_f8(int M, int N) {
  return (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

template <int M, int N>
__global__ void __launch_bounds__(128, 1) mma_loop(int iters, unsigned long long *out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t *s = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(sm) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_barrier_init(); }
  if (warp == 0) tmem_alloc(&tbase, 256);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tbase;
  if (warp == 1 && lane == 0) {
    const uint32_t a0 = smem_u32(s), b0 = smem_u32(s + 16384);
    unsigned long long t0, t1;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    uint32_t ph = 0;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
      for (int k = 0; k < 4; ++k)
        mma_f8(tmem, sw128_kmajor_desc(a0 + k * 32), sw128_kmajor_desc(b0 + k * 32), idesc_f8(M, N));
      if ((it & 7) == 7) {
        mma_commit(&bar);
        mbar_wait(&bar, ph);
        ph ^= 1;
      }
    }
    mma_commit(&bar);
    mbar_wait(&bar, ph);
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
    out[blockIdx.x] = t1 - t0;
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tmem, 256);
}

template <int M, int N>
void run(int sms, int clock_khz) {
  const int iters = 20000;
  unsigned long long *out;
  cudaMalloc(&out, sms * 8);
  auto k = mma_loop<M, N>;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
  k<<<sms, 128, 64 * 1024>>>(100, out);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  k<<<sms, 128, 64 * 1024>>>(iters, out);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  const double n_mma = 4.0 * iters, ns = ms * 1e6 / n_mma, cyc = ns * clock_khz * 1e-6;
  printf("M=%3d N=%3d: %6.1f ns = %5.0f cycles per MMA; weights as M: %5.1f B/cycle, as N: %5.1f B/cycle  %s\n",
         M, N, ns, cyc, M * 32 / cyc, N * 32 / cyc, cudaGetErrorString(cudaGetLastError()));
  cudaFree(out);
}

int main() {
  int sms, clk;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("SMs %d, clock %d kHz (cycles use this clock)\n", sms, clk);
  for (int rep = 0; rep < 2; ++rep) {
    run<128, 16>(sms, clk);
    run<128, 32>(sms, clk);
    run<128, 64>(sms, clk);
    run<128, 128>(sms, clk);
    run<128, 256>(sms, clk);
    run<64, 16>(sms, clk);
    run<64, 64>(sms, clk);
    run<64, 128>(sms, clk);
    run<64, 256>(sms, clk);
  }
  return 0;
}
