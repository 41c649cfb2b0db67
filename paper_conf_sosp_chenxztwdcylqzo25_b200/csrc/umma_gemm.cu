// umma_gemm.cu -- prefill router logits on the 5th-gen tensor cores, the
// load-time weight tiling, and the host helpers (tensor maps, per-device
// kernel attributes, experiment knobs).
//
//   logits[t, e] = x[t, :] . Wg[e, :]   (bf16 x bf16, fp32 accumulate in TMEM;
//                                        DESIGN.md reading R9)
//
// Work units = (128-token m-tile, 256-wide block of router rows) claimed from a
// device counter.  Roles per CTA (320 threads, one CTA per SM):
//   warp 0     TMA producer (x and router-row tiles) into a 4-stage ring
//   warp 1     TMEM allocator + single-thread tcgen05.mma issuer
//   warps 2-9  epilogue: tcgen05.ld -> registers (TMEM released) -> fp32 rows
// (The expert GEMMs run in umma_swap.cu.)
#include <cuda.h>
#include <mutex>
#include <set>
#include <tuple>

#include "common.cuh"
#include "kernels.h"
#include "sm100.cuh"

namespace moe {
using namespace sm100;

constexpr int UG_BM = 128, UG_BN = 256, UG_STAGES = 4, UG_THREADS = 320;
constexpr int UG_A_BYTES = UG_BM * 128;        // 16 KB (128 rows x 128 B)
constexpr int UG_B_BYTES = UG_BN * 128;        // 32 KB
constexpr uint32_t UG_TMEM_COLS = 256;
constexpr int UG_UQ = 4;                       // depth of the in-CTA work-unit queue
constexpr size_t UG_SMEM = 1024 + (size_t)UG_STAGES * (UG_A_BYTES + UG_B_BYTES) + 512;

__global__ void __launch_bounds__(UG_THREADS, 1) umma_logits_kernel(const __grid_constant__ LogitsParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t *sA = smem;
  uint8_t *sB = sA + UG_STAGES * UG_A_BYTES;
  uint64_t *full = reinterpret_cast<uint64_t *>(sB + UG_STAGES * UG_B_BYTES);
  uint64_t *empty = full + UG_STAGES;
  uint64_t *tmem_full = empty + UG_STAGES;
  uint64_t *tmem_empty = tmem_full + 1;
  uint64_t *uq_full = tmem_empty + 1;
  uint64_t *uq_empty = uq_full + UG_UQ;
  uint32_t *tmem_base_smem = reinterpret_cast<uint32_t *>(uq_empty + UG_UQ);
  int *unit_q = reinterpret_cast<int *>(tmem_base_smem + 4);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int mt = (p.T + UG_BM - 1) / UG_BM;
  const int n_units = mt * p.nb;

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&p.a_map);
    prefetch_tmap(&p.b_map);
    for (int s = 0; s < UG_STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    mbar_init(tmem_full, 1);
    mbar_init(tmem_empty, 8);
    for (int i = 0; i < UG_UQ; ++i) { mbar_init(&uq_full[i], 1); mbar_init(&uq_empty[i], 9); }
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc(tmem_base_smem, UG_TMEM_COLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_base_smem;

  if (warp == 0) {
    // ============================ TMA producer ============================
    if (lane == 0) {
      int stage = 0; uint32_t phase = 0;
      int qs = 0; uint32_t qph = 0;
      for (;;) {
        const int u = atomicAdd(p.sched, 1);
        mbar_wait(&uq_empty[qs], qph ^ 1);
        unit_q[qs] = u;
        mbar_arrive(&uq_full[qs]);
        if (++qs == UG_UQ) { qs = 0; qph ^= 1; }
        if (u >= n_units) break;
        const int row0 = (u % mt) * UG_BM, nb = u / mt;
        for (int kb = 0; kb < p.kblocks; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          mbar_expect_tx(&full[stage], UG_A_BYTES + UG_B_BYTES);
          tma_load_2d(sA + stage * UG_A_BYTES, &p.a_map, &full[stage], kb * 64, row0);
          tma_load_2d(sB + stage * UG_B_BYTES, &p.b_map, &full[stage], kb * 64, nb * UG_BN);
          if (++stage == UG_STAGES) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ============================ MMA issuer ============================
    int stage = 0; uint32_t phase = 0; uint32_t acc_phase = 0;
    int qs = 0; uint32_t qph = 0;
    for (;;) {
      mbar_wait(&uq_full[qs], qph);
      const int u = unit_q[qs];
      __syncwarp();
      if (lane == 0) mbar_arrive(&uq_empty[qs]);
      if (++qs == UG_UQ) { qs = 0; qph ^= 1; }
      if (u >= n_units) break;
      mbar_wait(tmem_empty, acc_phase ^ 1);
      tc_fence_after();
      for (int kb = 0; kb < p.kblocks; ++kb) {
        mbar_wait(&full[stage], phase);
        tc_fence_after();
        if (lane == 0) {
          const uint32_t a0 = smem_u32(sA + stage * UG_A_BYTES);
          const uint32_t b0 = smem_u32(sB + stage * UG_B_BYTES);
#pragma unroll
          for (int k = 0; k < 4; ++k)
            mma_bf16(tmem, sw128_kmajor_desc(a0 + k * 32), sw128_kmajor_desc(b0 + k * 32), idesc_bf16(UG_BM, UG_BN),
                     (kb | k) != 0);
          mma_commit(&empty[stage]);
          if (kb == p.kblocks - 1) mma_commit(tmem_full);
        }
        __syncwarp();
        if (++stage == UG_STAGES) { stage = 0; phase ^= 1; }
      }
      acc_phase ^= 1;
    }
  } else {
    // ============================ epilogue ============================
    // 8 warps: two per TMEM lane quadrant (= 32 token rows), each owning 128 of
    // the 256 router-row columns; registers first, TMEM released, then stores.
    const int ew = warp - 2;
    const int q = warp & 3;
    const int half = ew >> 2;
    const uint32_t lane_base = (uint32_t)(q * 32) << 16;
    uint32_t acc_phase = 0;
    int qs = 0; uint32_t qph = 0;
    for (;;) {
      mbar_wait(&uq_full[qs], qph);
      const int u = unit_q[qs];
      __syncwarp();
      if (lane == 0) mbar_arrive(&uq_empty[qs]);
      if (++qs == UG_UQ) { qs = 0; qph ^= 1; }
      if (u >= n_units) break;
      const int row = (u % mt) * UG_BM + q * 32 + lane, nb = u / mt;
      mbar_wait(tmem_full, acc_phase);
      tc_fence_after();
      uint32_t r[128];
#pragma unroll
      for (int c = 0; c < 4; ++c)
        tmem_ld_32x32b_x32(tmem + lane_base + half * 128 + c * 32, *reinterpret_cast<uint32_t(*)[32]>(r + 32 * c));
      tmem_ld_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(tmem_empty);
      const int n0 = nb * UG_BN + half * 128;
      if (row < p.T) {
        float *crow = p.out + (size_t)row * p.ldc;
        if ((p.ldc & 3) == 0 && n0 + 128 <= p.n_valid) {
          // 16-byte stores (4-byte stores put 32 rows x 4 B in every warp store)
          float4 *c4 = reinterpret_cast<float4 *>(crow + n0);
#pragma unroll
          for (int i = 0; i < 32; ++i)
            c4[i] = make_float4(__uint_as_float(r[4 * i]), __uint_as_float(r[4 * i + 1]),
                                __uint_as_float(r[4 * i + 2]), __uint_as_float(r[4 * i + 3]));
        } else {
#pragma unroll
          for (int i = 0; i < 128; ++i)
            if (n0 + i < p.n_valid) crow[n0 + i] = __uint_as_float(r[i]);
        }
      }
      acc_phase ^= 1;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc(tmem, UG_TMEM_COLS);
}

cudaError_t launch_umma_logits(const LogitsParams &p, int grid, cudaStream_t st) {
  if (grid <= 0) return cudaSuccess;
  cudaError_t e = set_kernel_attr((const void *)umma_logits_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  (int)UG_SMEM);
  if (e != cudaSuccess) return e;
  umma_logits_kernel<<<grid, UG_THREADS, UG_SMEM, st>>>(p);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ host helpers
cudaError_t set_kernel_attr(const void *kernel, cudaFuncAttribute attr, int value) {
  static std::mutex mu;
  static std::set<std::tuple<const void *, int, int, int>> done;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  const auto key = std::make_tuple(kernel, dev, (int)attr, value);
  std::lock_guard<std::mutex> lock(mu);
  if (done.count(key)) return cudaSuccess;
  e = cudaFuncSetAttribute(kernel, attr, value);
  if (e == cudaSuccess) done.insert(key);
  return e;
}

int experiment_knob(const char *env) {
#ifdef MOE_EXPERIMENTS
  const char *v = getenv(env);
  return v ? atoi(v) : 0;
#else
  (void)env;
  return 0;
#endif
}

// ------------------------------------------------------------------ weight tiling
// one thread per 16-byte chunk of the destination
__global__ void tile_weights_kernel(const uint8_t *__restrict__ src, uint8_t *__restrict__ dst, int nexp, int rows,
                                    int kbytes, int interleave_f, int es) {
  const int nt = rows / 256, kbn = kbytes / 128;
  const int64_t per_exp = (int64_t)rows * kbytes / 16;
  const int64_t total = per_exp * nexp;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < total; c += (int64_t)gridDim.x * blockDim.x) {
    const int64_t e = c / per_exp;
    int64_t rem = c % per_exp;
    const int64_t tile = rem / (256 * 8);          // 2048 chunks of 16 B per tile
    const int in = (int)(rem % (256 * 8));
    const int r = in >> 3, j = in & 7;              // tile row, 16-byte chunk slot (swizzled)
    const int nb = (int)(tile / kbn), kb = (int)(tile % kbn);
    const int jsrc = j ^ (r & 7);                    // chunk j of row r holds source chunk j ^ (r % 8)
    int srow;
    if (interleave_f > 0) {
      // W13 tile nb = h block nb (128 h columns); 128-row half c holds, per
      // 32-row lane quadrant q, [gate | up | gate | up] of columns
      // 128 nb + 64 c + 32 (q >> 1) + i  (umma_swap.cu / umma_decode.cu epilogues)
      const int c = r >> 7, q = (r >> 5) & 3, i = r & 31;
      const int f = nb * 128 + c * 64 + (q >> 1) * 32 + i;
      srow = (q & 1) ? interleave_f + f : f;
    } else {
      srow = nb * 256 + r;
    }
    const uint4 v = *reinterpret_cast<const uint4 *>(src + ((int64_t)e * rows + srow) * kbytes + (int64_t)kb * 128 +
                                                     jsrc * 16);
    *reinterpret_cast<uint4 *>(dst + c * 16) = v;
  }
  (void)nt; (void)es;
}

cudaError_t launch_tile_weights(const void *src, void *dst, int nexp, int rows, int kbytes, int interleave_f,
                                cudaStream_t st) {
  tile_weights_kernel<<<148 * 8, 256, 0, st>>>(reinterpret_cast<const uint8_t *>(src),
                                              reinterpret_cast<uint8_t *>(dst), nexp, rows, kbytes, interleave_f, 1);
  return cudaGetLastError();
}

// ------------------------------------------------------------------ tensor maps
static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    void *ptr = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(ptr);
  }
  return fn;
}

// plain 2-D view of a pre-tiled / scale-image buffer: rows of row_elems
// elements (uint8 or uint32), box = (row_elems, box_rows), no swizzle
bool make_rows_map(CUtensorMap *m, const void *base, bool u32, int64_t rows, int row_elems, int box_rows) {
  auto enc = get_encode();
  if (!enc) return false;
  const int es = u32 ? 4 : 1;
  cuuint64_t dims[2] = {(cuuint64_t)row_elems, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)row_elems * es};
  cuuint32_t box[2] = {(cuuint32_t)row_elems, (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(m, u32 ? CU_TENSOR_MAP_DATA_TYPE_UINT32 : CU_TENSOR_MAP_DATA_TYPE_UINT8, 2,
                   const_cast<void *>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

// contiguous buffer viewed as rows of row_bytes (8-byte elements), box = box_rows
// whole rows: few, long TMA rows for pre-tiled (already swizzled) operands
bool make_blocks_map(CUtensorMap *m, const void *base, int64_t total_bytes, int row_bytes, int box_rows) {
  auto enc = get_encode();
  if (!enc) return false;
  cuuint64_t dims[2] = {(cuuint64_t)(row_bytes / 8), (cuuint64_t)(total_bytes / row_bytes)};
  cuuint64_t strides[1] = {(cuuint64_t)row_bytes};
  cuuint32_t box[2] = {(cuuint32_t)(row_bytes / 8), (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_UINT64, 2, const_cast<void *>(base), dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

bool make_fp4_map(CUtensorMap *m, const void *base, int64_t rows, int64_t cols, int box_rows) {
  auto enc = get_encode();
  if (!enc) return false;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)(cols / 2)};
  cuuint32_t box[2] = {128, (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_16U4_ALIGN16B, 2, const_cast<void *>(base), dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

// e2m1 code -> e4m3 byte: magnitudes 0, .5, 1, 1.5, 2, 3, 4, 6 are e4m3 values exactly
__global__ void fp4_to_e4m3_kernel(const uint8_t *__restrict__ in, uint16_t *__restrict__ out, int64_t n) {
  const uint8_t lut[8] = {0x00, 0x30, 0x38, 0x3C, 0x40, 0x44, 0x48, 0x4C};
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const uint8_t b = in[i];
    const uint8_t lo = b & 0xF, hi = b >> 4;
    const uint16_t e0 = lut[lo & 7] | ((lo & 8) << 4), e1 = lut[hi & 7] | ((hi & 8) << 4);
    out[i] = (uint16_t)(e0 | (e1 << 8));          // element 2i (low nibble) first
  }
}

cudaError_t launch_fp4_to_e4m3(const void *packed, void *out, int64_t n_bytes_in, cudaStream_t st) {
  if (n_bytes_in <= 0) return cudaSuccess;
  fp4_to_e4m3_kernel<<<148 * 8, 256, 0, st>>>(reinterpret_cast<const uint8_t *>(packed),
                                             reinterpret_cast<uint16_t *>(out), n_bytes_in);
  return cudaGetLastError();
}

// dst row (e, nb, r) <- src row of W1 / W3 with the swap-AB tile interleave (tile_weights_kernel)
__global__ void permute_w13_rows_kernel(const uint8_t *__restrict__ src, uint8_t *__restrict__ dst, int nexp, int F,
                                        int row_bytes) {
  const int64_t chunks = (int64_t)row_bytes / 16, total = (int64_t)nexp * 2 * F * chunks;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < total; c += (int64_t)gridDim.x * blockDim.x) {
    const int64_t row = c / chunks, j = c % chunks;
    const int64_t e = row / (2 * F);
    const int rr = (int)(row % (2 * F)), nb = rr / 256, r = rr % 256;
    const int h = r >> 7, q = (r >> 5) & 3, i = r & 31;
    const int f = nb * 128 + h * 64 + (q >> 1) * 32 + i;
    const int64_t srow = e * 2 * F + ((q & 1) ? F + f : f);
    reinterpret_cast<uint4 *>(dst + row * row_bytes)[j] = reinterpret_cast<const uint4 *>(src + srow * row_bytes)[j];
  }
}

cudaError_t launch_permute_w13_rows(const void *src, void *dst, int nexp, int F, int row_bytes, cudaStream_t st) {
  permute_w13_rows_kernel<<<148 * 8, 256, 0, st>>>(reinterpret_cast<const uint8_t *>(src), reinterpret_cast<uint8_t *>(dst),
                                                  nexp, F, row_bytes);
  return cudaGetLastError();
}

// 2-D row-major [rows, cols] K-major operand, box = (128 bytes of K, box_rows), 128B swizzle
bool make_kmajor_map(CUtensorMap *m, const void *base, bool fp8, int64_t rows, int64_t cols, int box_rows) {
  auto enc = get_encode();
  if (!enc) return false;
  const int es = fp8 ? 1 : 2;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)(cols * es)};
  cuuint32_t box[2] = {(cuuint32_t)(128 / es), (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = enc(m, fp8 ? CU_TENSOR_MAP_DATA_TYPE_UINT8 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2,
                   const_cast<void *>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

}  // namespace moe
