// gemv.cu -- decode path: weight-streaming kernels for few tokens per expert.
//
// PAPER.md L170 (§3.2): AMX "incurs excessive overhead by processing full
// tiles" when an expert sees <= 4 tokens, so KTransformers switches to a
// lighter AVX-512 kernel "fully compatible with the AMX memory layout".  The
// B200 analog: for T <= gemv_max_tokens the expert FFNs bypass the tcgen05
// tiles and stream each active expert's weights exactly once with coalesced
// 16-byte loads, dotting them with the expert's (<= 8) token rows held in
// shared memory.  Decode is HBM-bound (L415): the roofline is the bytes of the
// experts hit.  Same numerics as the GEMM path (fp32 accumulation; FP8
// activations quantised per 1x128 block before each GEMM).
#include "common.cuh"
#include "kernels.h"

namespace moe {

constexpr int GV_THREADS = 512, GV_WARPS = GV_THREADS / 32;

// 16 weight values (bf16: 2 x uint4, fp8: 1 x uint4) -> fp32
template <bool FP8>
__device__ __forceinline__ void load16(const uint8_t *p, float *w) {
  if (FP8) {
    uint4 u = __ldg(reinterpret_cast<const uint4 *>(p));
    fp8x8_to_f32(make_uint2(u.x, u.y), w);
    fp8x8_to_f32(make_uint2(u.z, u.w), w + 8);
  } else {
    const uint4 *q = reinterpret_cast<const uint4 *>(p);
    bf16x8_to_f32(__ldg(q), w);
    bf16x8_to_f32(__ldg(q + 1), w + 8);
  }
}

// Which rows does this CTA serve?  slot < n_active: routed expert act_list[slot]
// (its tokens are the rows [offs_pad[e], offs_pad[e] + counts[e]) of the sorted
// order); slot == shared_slot: the shared expert on tokens 0..T-1.
struct GvSlot {
  int valid, expert, n, row0;  // row0: first sorted row (routed) or -1 (shared)
};
__device__ __forceinline__ GvSlot gv_slot(const GemvArgs &a) {
  GvSlot s{};
  const int slot = blockIdx.x;
  if (slot < *a.n_active) {
    const int e = a.act_list[slot];
    s.valid = 1; s.expert = e; s.n = a.counts[e]; s.row0 = a.offs_pad[e];
  } else if (a.has_shared && slot == gridDim.x - 1) {
    s.valid = 1; s.expert = -1; s.n = a.T; s.row0 = -1;
  }
  return s;
}

// ------------------------------------------------------------------ GEMV1: W13 + SwiGLU
// CTA = (slot, 256-row block of the interleaved W13 = 128 gate + 128 up rows)
// -> 128 h values per token.  FP8: h quantised per token over those 128 values.
template <bool FP8, int NT>
__global__ void __launch_bounds__(GV_THREADS) gemv13_kernel(const __grid_constant__ GemvArgs a) {
  extern __shared__ __align__(16) uint8_t gsm[];
  const GvSlot s = gv_slot(a);
  if (!s.valid) return;
  const int H = a.H, nb = blockIdx.y;
  const bool shared = s.expert < 0;
  const int Fo = shared ? a.Fs : a.F;
  if (nb * 128 >= Fo) return;
  __nv_bfloat16 *xs = reinterpret_cast<__nv_bfloat16 *>(gsm);         // [n][H] activations (dequantised)
  float *wsc = reinterpret_cast<float *>(gsm + (size_t)a.T * H * 2);  // [2][H/128] weight scales
  float *hbuf = wsc + 2 * (H / 128);                                  // [n][128]
  const int n = s.n;
  // ---- activations of this slot's tokens -> smem (bf16; exact for e4m3 x 2^e) ----
  for (int idx = threadIdx.x; idx < n * (H / 8); idx += GV_THREADS) {
    const int i = idx / (H / 8), c = idx % (H / 8);
    const int t = shared ? i : a.row_token[s.row0 + i];
    uint4 v;
    if (FP8) {
      uint2 q = *reinterpret_cast<const uint2 *>(reinterpret_cast<const uint8_t *>(a.xq) + (size_t)t * H + c * 8);
      float f[8];
      fp8x8_to_f32(q, f);
      const float sc = a.xs[(size_t)t * (H / 128) + (c * 8) / 128];
      __nv_bfloat162 *o = reinterpret_cast<__nv_bfloat162 *>(&v);
#pragma unroll
      for (int j = 0; j < 4; ++j) o[j] = __floats2bfloat162_rn(f[2 * j] * sc, f[2 * j + 1] * sc);
    } else {
      v = *reinterpret_cast<const uint4 *>(reinterpret_cast<const __nv_bfloat16 *>(a.x) + (size_t)t * H + c * 8);
    }
    *reinterpret_cast<uint4 *>(xs + (size_t)i * H + c * 8) = v;
  }
  const uint8_t *W = reinterpret_cast<const uint8_t *>(shared ? a.ws13 : a.w13);
  const int es = FP8 ? 1 : 2;
  const size_t row_bytes = (size_t)H * es;
  if (!shared) W += (size_t)s.expert * 2 * a.F * row_bytes;
  const float *Ws = shared ? a.ws13_s : a.w13_s;
  if (FP8) {
    if (!shared) Ws += (size_t)s.expert * (2 * a.F / 128) * (H / 128);
    for (int i = threadIdx.x; i < 2 * (H / 128); i += GV_THREADS) {
      const int half = i / (H / 128), kb = i % (H / 128);
      wsc[i] = Ws[(size_t)(2 * nb + half) * (H / 128) + kb];
    }
  }
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // each warp: 8 (gate, up) row pairs, P pairs at a time so 2P 16-byte weight
  // loads per lane are in flight (memory-level parallelism for HBM streaming)
  constexpr int P = NT <= 2 ? 4 : 2;
  constexpr int EPL = FP8 ? 16 : 8;             // weight elements per 16-byte load
  for (int p0 = 0; p0 < 128 / GV_WARPS; p0 += P) {
    const int i0 = warp * (128 / GV_WARPS) + p0;
    float ag[P][NT], au[P][NT];
#pragma unroll
    for (int q = 0; q < P; ++q)
#pragma unroll
      for (int t = 0; t < NT; ++t) { ag[q][t] = 0.f; au[q][t] = 0.f; }
    for (int k0 = lane * EPL; k0 < H; k0 += 32 * EPL) {
      uint4 wgv[P], wuv[P];
#pragma unroll
      for (int q = 0; q < P; ++q) {
        wgv[q] = __ldg(reinterpret_cast<const uint4 *>(W + (size_t)(256 * nb + i0 + q) * row_bytes + (size_t)k0 * es));
        wuv[q] = __ldg(reinterpret_cast<const uint4 *>(W + (size_t)(256 * nb + 128 + i0 + q) * row_bytes + (size_t)k0 * es));
      }
      float sg = 1.f, su = 1.f;
      if (FP8) { sg = wsc[k0 / 128]; su = wsc[H / 128 + k0 / 128]; }
#pragma unroll
      for (int t = 0; t < NT; ++t) {
        if (t < n) {
          float xv[EPL];
          const uint4 *xp = reinterpret_cast<const uint4 *>(xs + (size_t)t * H + k0);
          bf16x8_to_f32(xp[0], xv);
          if (FP8) bf16x8_to_f32(xp[1], xv + 8);
#pragma unroll
          for (int q = 0; q < P; ++q) {
            float wv[EPL], uv[EPL];
            if (FP8) {
              fp8x8_to_f32(make_uint2(wgv[q].x, wgv[q].y), wv); fp8x8_to_f32(make_uint2(wgv[q].z, wgv[q].w), wv + 8);
              fp8x8_to_f32(make_uint2(wuv[q].x, wuv[q].y), uv); fp8x8_to_f32(make_uint2(wuv[q].z, wuv[q].w), uv + 8);
            } else {
              bf16x8_to_f32(wgv[q], wv);
              bf16x8_to_f32(wuv[q], uv);
            }
            float pg = 0.f, pu = 0.f;
#pragma unroll
            for (int j = 0; j < EPL; ++j) { pg = fmaf(wv[j], xv[j], pg); pu = fmaf(uv[j], xv[j], pu); }
            ag[q][t] = fmaf(pg, sg, ag[q][t]);
            au[q][t] = fmaf(pu, su, au[q][t]);
          }
        }
      }
    }
#pragma unroll
    for (int q = 0; q < P; ++q)
#pragma unroll
      for (int t = 0; t < NT; ++t) {
        if (t < n) {
          const float g = warp_sum(ag[q][t]), u = warp_sum(au[q][t]);
          if (lane == 0) hbuf[t * 128 + i0 + q] = silu_f(g) * u;
        }
      }
  }
  __syncthreads();
  // ---- write h (FP8: per-token 1x128 UE8M0 quantisation) ----
  for (int t = warp; t < n; t += GV_WARPS) {
    float v[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) v[j] = hbuf[t * 128 + lane * 4 + j];
    const int64_t row = shared ? t : (int64_t)s.row0 + t;
    if (FP8) {
      float am = fmaxf(fmaxf(fabsf(v[0]), fabsf(v[1])), fmaxf(fabsf(v[2]), fabsf(v[3])));
      am = warp_max(am);
      const int e = ue8m0_exponent(am);
      const float inv = exp2i(-e);
      uint32_t q = (uint32_t)f32_to_e4m3(v[0] * inv) | ((uint32_t)f32_to_e4m3(v[1] * inv) << 8) |
                   ((uint32_t)f32_to_e4m3(v[2] * inv) << 16) | ((uint32_t)f32_to_e4m3(v[3] * inv) << 24);
      uint8_t *hp = reinterpret_cast<uint8_t *>(shared ? a.hsh : a.h);
      *reinterpret_cast<uint32_t *>(hp + row * Fo + nb * 128 + lane * 4) = q;
      if (lane == 0) (shared ? a.hsh_s : a.h_s)[row * (Fo / 128) + nb] = exp2i(e);
    } else {
      __nv_bfloat16 *hp = reinterpret_cast<__nv_bfloat16 *>(shared ? a.hsh : a.h);
      __nv_bfloat162 *o = reinterpret_cast<__nv_bfloat162 *>(hp + row * Fo + nb * 128 + lane * 4);
      o[0] = __floats2bfloat162_rn(v[0], v[1]);
      o[1] = __floats2bfloat162_rn(v[2], v[3]);
    }
  }
}

// ------------------------------------------------------------------ GEMV2: W2
// CTA = (slot, 128-row block of W2) -> 128 output channels per token.
template <bool FP8, int NT>
__global__ void __launch_bounds__(GV_THREADS) gemv2_kernel(const __grid_constant__ GemvArgs a) {
  extern __shared__ __align__(16) uint8_t gsm[];
  const GvSlot s = gv_slot(a);
  if (!s.valid) return;
  const int H = a.H, rb = blockIdx.y;
  const bool shared = s.expert < 0;
  const int K = shared ? a.Fs : a.F;
  __nv_bfloat16 *hs = reinterpret_cast<__nv_bfloat16 *>(gsm);                 // [n][K]
  float *wsc = reinterpret_cast<float *>(gsm + (size_t)a.T * K * 2);         // [K/128]
  const int n = s.n;
  for (int idx = threadIdx.x; idx < n * (K / 8); idx += GV_THREADS) {
    const int i = idx / (K / 8), c = idx % (K / 8);
    const int64_t row = shared ? i : (int64_t)s.row0 + i;
    uint4 v;
    if (FP8) {
      const uint8_t *hp = reinterpret_cast<const uint8_t *>(shared ? a.hsh : a.h);
      uint2 q = *reinterpret_cast<const uint2 *>(hp + row * K + c * 8);
      float f[8];
      fp8x8_to_f32(q, f);
      const float sc = (shared ? a.hsh_s : a.h_s)[row * (K / 128) + (c * 8) / 128];
      __nv_bfloat162 *o = reinterpret_cast<__nv_bfloat162 *>(&v);
#pragma unroll
      for (int j = 0; j < 4; ++j) o[j] = __floats2bfloat162_rn(f[2 * j] * sc, f[2 * j + 1] * sc);
    } else {
      const __nv_bfloat16 *hp = reinterpret_cast<const __nv_bfloat16 *>(shared ? a.hsh : a.h);
      v = *reinterpret_cast<const uint4 *>(hp + row * K + c * 8);
    }
    *reinterpret_cast<uint4 *>(hs + (size_t)i * K + c * 8) = v;
  }
  const uint8_t *W = reinterpret_cast<const uint8_t *>(shared ? a.ws2 : a.w2);
  const int es = FP8 ? 1 : 2;
  const size_t row_bytes = (size_t)K * es;
  if (!shared) W += (size_t)s.expert * H * row_bytes;
  if (FP8) {
    const float *Ws = shared ? a.ws2_s : a.w2_s + (size_t)s.expert * (H / 128) * (K / 128);
    for (int i = threadIdx.x; i < K / 128; i += GV_THREADS) wsc[i] = Ws[(size_t)rb * (K / 128) + i];
  }
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  constexpr int R = NT <= 2 ? 8 : 4;            // rows per warp pass (R loads in flight)
  constexpr int EPL = FP8 ? 16 : 8;
  for (int p0 = 0; p0 < 128 / GV_WARPS; p0 += R) {
    const int r0 = rb * 128 + warp * (128 / GV_WARPS) + p0;
    float acc[R][NT];
#pragma unroll
    for (int q = 0; q < R; ++q)
#pragma unroll
      for (int t = 0; t < NT; ++t) acc[q][t] = 0.f;
    for (int k0 = lane * EPL; k0 < K; k0 += 32 * EPL) {
      uint4 wv4[R];
#pragma unroll
      for (int q = 0; q < R; ++q)
        wv4[q] = __ldg(reinterpret_cast<const uint4 *>(W + (size_t)(r0 + q) * row_bytes + (size_t)k0 * es));
      const float sw = FP8 ? wsc[k0 / 128] : 1.f;
#pragma unroll
      for (int t = 0; t < NT; ++t) {
        if (t < n) {
          float hv[EPL];
          const uint4 *hp = reinterpret_cast<const uint4 *>(hs + (size_t)t * K + k0);
          bf16x8_to_f32(hp[0], hv);
          if (FP8) bf16x8_to_f32(hp[1], hv + 8);
#pragma unroll
          for (int q = 0; q < R; ++q) {
            float wv[EPL];
            if (FP8) {
              fp8x8_to_f32(make_uint2(wv4[q].x, wv4[q].y), wv); fp8x8_to_f32(make_uint2(wv4[q].z, wv4[q].w), wv + 8);
            } else {
              bf16x8_to_f32(wv4[q], wv);
            }
            float pp = 0.f;
#pragma unroll
            for (int j = 0; j < EPL; ++j) pp = fmaf(wv[j], hv[j], pp);
            acc[q][t] = fmaf(pp, sw, acc[q][t]);
          }
        }
      }
    }
#pragma unroll
    for (int q = 0; q < R; ++q)
#pragma unroll
      for (int t = 0; t < NT; ++t) {
        if (t < n) {
          const float v = warp_sum(acc[q][t]);
          if (lane == 0) {
            const int64_t row = shared ? t : (int64_t)s.row0 + t;
            __nv_bfloat16 *out = shared ? a.ysh : a.yperm;
            out[row * H + r0 + q] = __float2bfloat16_rn(v);
          }
        }
      }
  }
}

// ------------------------------------------------------------------ router GEMV
// logits[t, e] = x[t] . Wg[e] for T <= GV_MAXTOK: one warp per router row.
template <int NT>
__global__ void __launch_bounds__(128) router_gemv_kernel(const __nv_bfloat16 *__restrict__ x, int T, int H,
                                                          const __nv_bfloat16 *__restrict__ wg, int rows,
                                                          float *__restrict__ logits) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int e = blockIdx.x * 4 + warp;
  if (e >= rows) return;
  float acc[NT];
#pragma unroll
  for (int t = 0; t < NT; ++t) acc[t] = 0.f;
  const __nv_bfloat16 *wr = wg + (size_t)e * H;
  constexpr int U = 4;
  for (int kb = lane * 8; kb < H; kb += 256 * U) {
    uint4 w4[U];
#pragma unroll
    for (int u = 0; u < U; ++u)
      w4[u] = (kb + u * 256 < H) ? __ldg(reinterpret_cast<const uint4 *>(wr + kb + u * 256)) : make_uint4(0, 0, 0, 0);
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int k0 = kb + u * 256;
      if (k0 >= H) break;
      float w8[8];
      bf16x8_to_f32(w4[u], w8);
#pragma unroll
      for (int t = 0; t < NT; ++t) {
        if (t < T) {
          float x8[8];
          bf16x8_to_f32(__ldg(reinterpret_cast<const uint4 *>(x + (size_t)t * H + k0)), x8);
#pragma unroll
          for (int j = 0; j < 8; ++j) acc[t] = fmaf(w8[j], x8[j], acc[t]);
        }
      }
    }
  }
#pragma unroll
  for (int t = 0; t < NT; ++t) {
    if (t < T) {
      const float v = warp_sum(acc[t]);
      if (lane == 0) logits[(size_t)t * rows + e] = v;
    }
  }
}

cudaError_t launch_router_gemv(const void *x, int T, int H, const void *wg, int rows, float *logits,
                               cudaStream_t st) {
  if (T <= 0) return cudaSuccess;
  const dim3 g((rows + 3) / 4);
  auto xb = reinterpret_cast<const __nv_bfloat16 *>(x);
  auto wb = reinterpret_cast<const __nv_bfloat16 *>(wg);
  if (T <= 1) router_gemv_kernel<1><<<g, 128, 0, st>>>(xb, T, H, wb, rows, logits);
  else if (T <= 2) router_gemv_kernel<2><<<g, 128, 0, st>>>(xb, T, H, wb, rows, logits);
  else if (T <= 4) router_gemv_kernel<4><<<g, 128, 0, st>>>(xb, T, H, wb, rows, logits);
  else router_gemv_kernel<8><<<g, 128, 0, st>>>(xb, T, H, wb, rows, logits);
  return cudaGetLastError();
}

template <class K>
static cudaError_t set_smem(K kern, size_t bytes) {
  if (bytes <= 48 * 1024) return cudaSuccess;
  return set_kernel_attr((const void *)kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
}

size_t gemv_smem_bytes(int T, int H, int F, int Fs) {
  const int Fmax = Fs > F ? Fs : F;
  const size_t sm1 = (size_t)T * H * 2 + 2 * (H / 128) * 4 + (size_t)T * 128 * 4;
  const size_t sm2 = (size_t)T * Fmax * 2 + (Fmax / 128) * 4;
  return sm1 > sm2 ? sm1 : sm2;
}

template <bool FP8, int NT>
static cudaError_t launch_gemv_t(const GemvArgs &a, int which, int max_slots, cudaStream_t st) {
  const int Fmax = a.Fs > a.F ? a.Fs : a.F;
  const size_t sm1 = (size_t)a.T * a.H * 2 + 2 * (a.H / 128) * 4 + (size_t)a.T * 128 * 4;
  const size_t sm2 = (size_t)a.T * Fmax * 2 + (Fmax / 128) * 4;
  cudaError_t e;
  if (which == 1) {
    if ((e = set_smem(gemv13_kernel<FP8, NT>, sm1)) != cudaSuccess) return e;
    gemv13_kernel<FP8, NT><<<dim3(max_slots, Fmax / 128), GV_THREADS, sm1, st>>>(a);
  } else {
    if ((e = set_smem(gemv2_kernel<FP8, NT>, sm2)) != cudaSuccess) return e;
    gemv2_kernel<FP8, NT><<<dim3(max_slots, a.H / 128), GV_THREADS, sm2, st>>>(a);
  }
  return cudaGetLastError();
}

template <bool FP8>
static cudaError_t launch_gemv_nt(const GemvArgs &a, int which, int max_slots, cudaStream_t st) {
  if (a.T <= 1) return launch_gemv_t<FP8, 1>(a, which, max_slots, st);
  if (a.T <= 2) return launch_gemv_t<FP8, 2>(a, which, max_slots, st);
  if (a.T <= 4) return launch_gemv_t<FP8, 4>(a, which, max_slots, st);
  return launch_gemv_t<FP8, 8>(a, which, max_slots, st);
}

cudaError_t launch_gemv(const GemvArgs &a, int which, int max_slots, cudaStream_t st) {
  if (max_slots <= 0 || a.T <= 0) return cudaSuccess;
  return a.fp8 ? launch_gemv_nt<true>(a, which, max_slots, st) : launch_gemv_nt<false>(a, which, max_slots, st);
}

}  // namespace moe
