// tcgen05 MMA issue cost on CTA pairs without pipeline drains: 4 MMAs (one 128-byte
// k-block) per iteration, a commit per iteration into an R-deep barrier ring, and a wait
// only on the commit of R-1 iterations ago (the GEMM's stage-release cadence).  Reports
// SM cycles per MMA (clock64) and the SM clock (clock64 / globaltimer) per variant.
#include <cstdio>
#include <cuda.h>
#include <cuda_runtime.h>
#include "../../paper_conf_sosp_chenxztwdcylqzo25_b200/csrc/sm100.cuh"
using namespace moe::sm100;

__device__ __forceinline__ void mma_f8_pair(uint32_t d, uint64_t a, uint64_t b, uint32_t id, uint32_t acc) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
               "tcgen05.mma.cta_group::2.kind::f8f6f4 [%0], %1, %2, %3, p;\n\t}" ::"r"(d), "l"(a), "l"(b), "r"(id), "r"(acc)
               : "memory");
}
__device__ __forceinline__ void mma_f8_1(uint32_t d, uint64_t a, uint64_t b, uint32_t id, uint32_t acc) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
               "tcgen05.mma.cta_group::1.kind::f8f6f4 [%0], %1, %2, %3, p;\n\t}" ::"r"(d), "l"(a), "l"(b), "r"(id), "r"(acc)
               : "memory");
}
__host__ __device__ constexpr uint32_t idesc_f8(int M, int N) {
  return (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
constexpr int R = 6;

template <int KIND, int CP, int G, int CE = 1, int RR = R>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1) mma_loop(int iters, int N, int M, unsigned long long *out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t *s = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(sm) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t ring[RR];
  __shared__ uint32_t tbase;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t crank = cluster_rank();
  if (threadIdx.x == 0) { for (int i = 0; i < RR; ++i) mbar_init(&ring[i], 1); fence_barrier_init(); }
  if (warp == 0) { if (G == 2) tmem_alloc_pair(&tbase, 512); else tmem_alloc(&tbase, 512); }
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  const uint32_t tmem = tbase;
  if ((G == 1 || crank == 0) && warp == 1 && lane == 0) {
    const uint32_t a0 = smem_u32(s), b0 = smem_u32(s + 16384);
    unsigned long long g0, g1;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g0));
    const long long c0 = clock64();
    uint32_t ph[RR] = {};
    for (int it = 0; it < iters; ++it) {
      const int ci = it / CE, r = ci % RR;                          // commit index of this iteration
      if (it % CE == 0 && ci >= RR) { mbar_wait(&ring[r], ph[r]); ph[r] ^= 1; }   // the commit RR commits ago
      const uint32_t set = ((it >> 2) & 1) * 16;
      if (CP && (it & 3) == 0 && G == 1) {
        tmem_cp_32x128b_x4(tmem + 256 + set, sf_desc(smem_u32(s + 49152)));
        tmem_cp_32x128b_x4(tmem + 264 + set, sf_desc(smem_u32(s + 49152 + 512)));
        tmem_cp_32x128b_x4(tmem + 268 + set, sf_desc(smem_u32(s + 49152 + 1024)));
      } else if (CP && (it & 3) == 0) {
        tmem_cp_32x128b_x4_pair(tmem + 256 + set, sf_desc(smem_u32(s + 49152)));
        tmem_cp_32x128b_x4_pair(tmem + 264 + set, sf_desc(smem_u32(s + 49152 + 512)));
        tmem_cp_32x128b_x4_pair(tmem + 268 + set, sf_desc(smem_u32(s + 49152 + 1024)));
      }
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const uint64_t ad = sw128_kmajor_desc(a0 + k * 32), bd = sw128_kmajor_desc(b0 + k * 32);
        if (G == 2) {
          if (KIND == 0) mma_mxf8_pair(tmem, ad, bd, idesc_mxf8(M, N, it & 3, it & 3), 1, tmem + 256 + set, tmem + 264 + set);
          else mma_f8_pair(tmem, ad, bd, idesc_f8(M, N), 1);
        } else {
          if (KIND == 0) mma_mxf8(tmem, ad, bd, idesc_mxf8(M, N, it & 3, it & 3), 1, tmem + 256 + set, tmem + 264 + set);
          else mma_f8_1(tmem, ad, bd, idesc_f8(M, N), 1);
        }
      }
      if (it % CE == CE - 1) { if (G == 2) mma_commit_pair(&ring[r]); else mma_commit(&ring[r]); }
    }
    {
      const int nc = iters / CE;
      for (int c = nc - RR; c < nc; ++c) { const int r = c % RR; mbar_wait(&ring[r], ph[r]); ph[r] ^= 1; }
    }
    const long long c1 = clock64();
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g1));
    out[2 * blockIdx.x] = c1 - c0;
    out[2 * blockIdx.x + 1] = g1 - g0;
  }
  tc_fence_before();
  cluster_sync();
  if (warp == 0) { if (G == 2) tmem_dealloc_pair(tmem, 512); else tmem_dealloc(tmem, 512); }
}

template <int KIND, int CP, int G, int CE = 1, int RR = R>
void run(const char *name, int N, int M, int grid) {
  const int iters = 20000;
  unsigned long long *out; cudaMalloc(&out, grid * 16); cudaMemset(out, 0, grid * 16);
  auto k = mma_loop<KIND, CP, G, CE, RR>;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
  k<<<grid, 128, 64 * 1024>>>(100, N, M, out);
  cudaDeviceSynchronize();
  k<<<grid, 128, 64 * 1024>>>(iters, N, M, out);
  cudaDeviceSynchronize();
  unsigned long long h[2 * 148];
  cudaMemcpy(h, out, grid * 16, cudaMemcpyDeviceToHost);
  double cyc = 0, ns = 0; int n = 0;
  for (int i = 0; i < grid; i += (G == 2 ? 2 : 1)) { cyc += h[2 * i]; ns += h[2 * i + 1]; ++n; }
  cyc /= n; ns /= n;
  const double macs_sm = (double)M / G * N * 32;      // per SM per MMA
  printf("%-10s CE=%d R=%2d G=%d M=%3d N=%3d: %6.1f cyc/MMA  %6.0f MAC/cyc/SM  clock %4.0f MHz  %s\n", name, CE, RR, G, M, N,
         cyc / (4.0 * iters), macs_sm / (cyc / (4.0 * iters)), cyc / ns * 1e3, cudaGetErrorString(cudaGetLastError()));
  cudaFree(out);
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int g = sms & ~1;
  const int Ns[] = {64, 128, 192, 256};
  for (int N : Ns) run<0, 1, 2, 1, 6>("mxf8", N, 256, g);
  for (int N : Ns) run<0, 1, 2, 1, 12>("mxf8", N, 256, g);
  for (int N : Ns) run<0, 1, 2, 2, 6>("mxf8", N, 256, g);
  for (int N : Ns) run<0, 1, 2, 4, 4>("mxf8", N, 256, g);
  for (int N : Ns) run<0, 0, 2, 4, 4>("mxf8-nocp", N, 256, g);
  for (int N : Ns) run<1, 0, 2, 1, 12>("f8f6f4", N, 256, g);
  for (int N : Ns) run<1, 0, 2, 4, 4>("f8f6f4", N, 256, g);
  for (int N : Ns) run<1, 0, 1, 4, 4>("f8f6f4", N, 128, g);
  for (int N : Ns) run<0, 1, 1, 4, 4>("mxf8", N, 128, g);
  return 0;
}
