// simt_gemm.cu -- CUDA-core tiled grouped expert GEMM: the path for the F32
// toy weights and hidden sizes that are not a multiple of 256 (the router
// logits of those layers run in gemv.cu's router_gemv / umma_gemm.cu).
//
//   C[m, n] = sum_k A[m, k] * B_e[n, k]        (fp32 accumulate)
//
// Modes:
//   SWIGLU : A = x_perm / x (bf16 or e4m3 + 1x128 scales), B = W13 of expert e
//            (rows interleaved per 128: W1 block b then W3 block b), epilogue
//            h = silu(g) * u  (fused gate+up batch), optional
//            e4m3 requantisation of h from fp32 (reading R11)
//   PLAIN  : A = h, B = W2 of expert e -> bf16 y rows ("down")
#include "common.cuh"
#include "kernels.h"

namespace moe {

constexpr int SG_BM = 64, SG_BK = 32, SG_THREADS = 256;

template <int MODE>
struct SgCfg {
  static constexpr int BN = (MODE == GEMM_SWIGLU) ? 256 : 128;  // B rows per CTA
  static constexpr int NJ = BN / 16;                             // cols per thread
};

__device__ __forceinline__ void load8_B(const void *B, int btype, int64_t elem_off, float scale,
                                        float *out) {
  if (btype == WT_BF16) {
    uint4 u = __ldg(reinterpret_cast<const uint4 *>(reinterpret_cast<const __nv_bfloat16 *>(B) + elem_off));
    bf16x8_to_f32(u, out);
  } else if (btype == WT_FP8) {
    uint2 u = __ldg(reinterpret_cast<const uint2 *>(reinterpret_cast<const uint8_t *>(B) + elem_off));
    fp8x8_to_f32(u, out);
#pragma unroll
    for (int i = 0; i < 8; ++i) out[i] *= scale;
  } else {
    const float4 *p = reinterpret_cast<const float4 *>(reinterpret_cast<const float *>(B) + elem_off);
    float4 a = __ldg(p), b = __ldg(p + 1);
    out[0] = a.x; out[1] = a.y; out[2] = a.z; out[3] = a.w;
    out[4] = b.x; out[5] = b.y; out[6] = b.z; out[7] = b.w;
  }
}

template <int MODE>
__global__ void __launch_bounds__(SG_THREADS)
simt_gemm_kernel(const __grid_constant__ SimtGemmArgs a) {
  constexpr int BN = SgCfg<MODE>::BN;
  constexpr int NJ = SgCfg<MODE>::NJ;
  __shared__ __align__(16) float As[SG_BK][SG_BM];
  __shared__ __align__(16) float Bs[SG_BK][BN];

  const int tid = threadIdx.x;
  const int tx = tid & 15, ty = tid >> 4;

  // ---- which rows / which expert ----
  int expert = 0, row0, row_end;
  if (a.tiles) {
    const int t = blockIdx.x >> 1;
    if (t >= *a.n_tiles) return;
    int4 tl = a.tiles[t];
    expert = tl.x;
    row0 = tl.y + (blockIdx.x & 1) * SG_BM;
    row_end = tl.z;
    if (row0 >= row_end) return;
  } else {
    row0 = blockIdx.x * SG_BM;
    row_end = a.M;
    if (row0 >= row_end) return;
  }
  const int n0 = blockIdx.y * BN;
  const void *B = a.B;
  const float *Bsc = a.Bs;
  if (a.b_type == WT_FP8) Bsc += (int64_t)expert * a.bs_stride;
  const int64_t b_base = (int64_t)expert * a.b_stride;
  const int K = a.K;
  const int kblocks = K / 128;

  float acc[4][NJ];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < NJ; ++j) acc[i][j] = 0.f;

  for (int k0 = 0; k0 < K; k0 += SG_BK) {
    // ---- stage A: 64 rows x 32 k, 8 elements per thread ----
    {
      const int r = tid >> 2, kk = (tid & 3) * 8;
      const int row = row0 + r;
      float v[8];
      if (row < row_end) {
        const int64_t off = (int64_t)row * a.lda + k0 + kk;
        if (a.a_fp8) {
          uint2 u = __ldg(reinterpret_cast<const uint2 *>(reinterpret_cast<const uint8_t *>(a.A) + off));
          fp8x8_to_f32(u, v);
          const float s = a.As[(int64_t)row * (K / 128) + (k0 + kk) / 128];
#pragma unroll
          for (int i = 0; i < 8; ++i) v[i] *= s;
        } else {
          uint4 u = __ldg(reinterpret_cast<const uint4 *>(reinterpret_cast<const __nv_bfloat16 *>(a.A) + off));
          bf16x8_to_f32(u, v);
        }
      } else {
#pragma unroll
        for (int i = 0; i < 8; ++i) v[i] = 0.f;
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) As[kk + i][r] = v[i];
    }
    // ---- stage B: BN rows x 32 k ----
#pragma unroll
    for (int it = 0; it < BN / 64; ++it) {
      const int idx = tid + it * SG_THREADS;
      const int r = idx >> 2, kk = (idx & 3) * 8;
      const int n = n0 + r;
      float v[8];
      if (n < a.N) {
        float sc = 1.f;
        if (a.b_type == WT_FP8) sc = Bsc[(int64_t)(n / 128) * kblocks + (k0 + kk) / 128];
        load8_B(B, a.b_type, b_base + (int64_t)n * K + k0 + kk, sc, v);
      } else {
#pragma unroll
        for (int i = 0; i < 8; ++i) v[i] = 0.f;
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) Bs[kk + i][r] = v[i];
    }
    __syncthreads();
#pragma unroll 8
    for (int kk = 0; kk < SG_BK; ++kk) {
      float4 av = *reinterpret_cast<const float4 *>(&As[kk][ty * 4]);
      float ar[4] = {av.x, av.y, av.z, av.w};
      float br[NJ];
#pragma unroll
      for (int j = 0; j < NJ; ++j) br[j] = Bs[kk][tx + 16 * j];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < NJ; ++j) acc[i][j] = fmaf(ar[i], br[j], acc[i][j]);
    }
    __syncthreads();
  }

  // ---- epilogues ----
  if constexpr (MODE == GEMM_PLAIN) {
    __nv_bfloat16 *C = reinterpret_cast<__nv_bfloat16 *>(a.C);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int row = row0 + ty * 4 + i;
      if (row >= row_end) continue;
#pragma unroll
      for (int j = 0; j < NJ; ++j) {
        const int n = n0 + tx + 16 * j;
        if (n < a.N) C[(int64_t)row * a.ldc + n] = __float2bfloat16_rn(acc[i][j]);
      }
    }
  } else {  // SWIGLU: gate at j < 8 (cols 0..127 of the 256-row block), up at j + 8
    const int f0 = blockIdx.y * 128;
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int row = row0 + ty * 4 + i;
      float h[8];
      float amax = 0.f;
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        h[j] = silu_f(acc[i][j]) * acc[i][j + 8];
        amax = fmaxf(amax, fabsf(h[j]));
      }
      if (a.out_fp8) {
        // amax over the row's 128 h values: the 16 lanes sharing ty
#pragma unroll
        for (int o = 8; o > 0; o >>= 1) amax = fmaxf(amax, __shfl_xor_sync(0xffffffffu, amax, o));
        const int e = ue8m0_exponent(amax);
        const float inv = exp2i(-e);
        if (row < row_end) {
          uint8_t *C = reinterpret_cast<uint8_t *>(a.C);
#pragma unroll
          for (int j = 0; j < 8; ++j) C[(int64_t)row * a.ldc + f0 + tx + 16 * j] = f32_to_e4m3(h[j] * inv);
          if (tx == 0) a.Cs[(int64_t)row * (a.ldc / 128) + f0 / 128] = exp2i(e);
        }
      } else if (row < row_end) {
        __nv_bfloat16 *C = reinterpret_cast<__nv_bfloat16 *>(a.C);
#pragma unroll
        for (int j = 0; j < 8; ++j) C[(int64_t)row * a.ldc + f0 + tx + 16 * j] = __float2bfloat16_rn(h[j]);
      }
    }
  }
}

cudaError_t launch_simt_gemm(int mode, const SimtGemmArgs &a, int grid_x, cudaStream_t st) {
  if (grid_x <= 0) return cudaSuccess;
  if (mode == GEMM_PLAIN) {
    dim3 g(grid_x, (a.N + 127) / 128);
    simt_gemm_kernel<GEMM_PLAIN><<<g, SG_THREADS, 0, st>>>(a);
  } else {
    dim3 g(grid_x, a.N / 256);
    simt_gemm_kernel<GEMM_SWIGLU><<<g, SG_THREADS, 0, st>>>(a);
  }
  return cudaGetLastError();
}

}  // namespace moe
