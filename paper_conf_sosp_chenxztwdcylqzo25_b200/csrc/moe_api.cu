// moe_api.cu -- the C ABI of include/moe.h: create (validate, allocate,
// repack weights), forward (enqueue the kernels, no host sync), destroy.
#include <cmath>
#include <cstdarg>
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "common.cuh"
#include "kernels.h"

using namespace moe;

namespace {
// NVTX range for the host-side enqueue of a call (nsys / ncu --nvtx); header-only
// NVTX v3, a no-op unless a tool is attached
struct NvtxRange {
  explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

thread_local std::string g_err;

moe_status fail(moe_status s, const char *fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return s;
}

#define CUDA_TRY(expr)                                                                        \
  do {                                                                                        \
    cudaError_t _e = (expr);                                                                  \
    if (_e != cudaSuccess)                                                                    \
      return fail(_e == cudaErrorMemoryAllocation ? MOE_ERR_OOM : MOE_ERR_CUDA, "%s: %s (%s:%d)", \
                  #expr, cudaGetErrorString(_e), __FILE__, __LINE__);                         \
  } while (0)

// a kernel launch of the forward: checked and counted (moe_layer_info reports the
// launches of the last prefill / decode forward)
#define KL_TRY(expr)         \
  do {                       \
    CUDA_TRY(expr);          \
    ++L->n_launch;           \
  } while (0)

template <class T>
cudaError_t dalloc(moe_layer *L, T **p, size_t bytes, bool weight) {
  if (bytes == 0) { *p = nullptr; return cudaSuccess; }
  cudaError_t e = cudaMalloc(reinterpret_cast<void **>(p), bytes);
  if (e == cudaSuccess) (weight ? L->weight_bytes : L->workspace_bytes) += (int64_t)bytes;
  return e;
}

void free_all(moe_layer *L) {
  void *ptrs[] = {L->gate_w, L->gate_bias, L->w13, L->w13_s, L->w2, L->w2_s, L->ws13, L->ws13_s, L->ws2,
                  L->ws2_s, L->logits, L->topk_idx, L->topk_w, L->sgate, L->chunk_cnt, L->chunk_base,
                  L->counts, L->offs, L->offs_pad, L->tiles, L->n_tiles, L->act_list, L->n_active,
                  L->row_token, L->pos, L->sched, L->pairs, L->n_pairs, L->xq, L->xs, L->xperm, L->xperm_s, L->hbuf, L->h_s, L->yperm,
                  L->hsh, L->hsh_s, L->ysh, L->w13_img, L->w2_img, L->ws13_img, L->ws2_img,
                  L->xperm_img, L->h_img, L->xq_img, L->hsh_img, L->dacc, L->trace, L->imm_list, L->def_list,
                  L->n_lists, L->xcopy, L->cl_scratch, L->zero_i32, L->w13_f4, L->w2_f4, L->ws13_f4, L->ws2_f4};
  for (void *p : ptrs)
    if (p) cudaFree(p);
  void *eps[] = {L->ep.send_x, L->ep.send_idx, L->ep.send_w, L->ep.sendpos, L->ep.cnt_dev, L->ep.recv_x,
                 L->ep.partial, L->ep.partial_def, L->ep.back, L->ep.back_def};
  for (void *p : eps)
    if (p) cudaFree(p);
  if (L->ep.cnt_host) cudaFreeHost(L->ep.cnt_host);
  ep_nccl_destroy(L->ep.comm);
  L->ep.comm = nullptr;
  ep_nccl_destroy(L->tp_comm);
  L->tp_comm = nullptr;
}

// Expert-parallel buffers (+ the NCCL communicator when a unique id is given;
// without one the layer belongs to an in-process group, moe_ep_group_forward).
moe_status ep_create(moe_layer *L, const moe_layer_config *cfg) {
  const int P = cfg->ep_size, H = L->H, k = L->k;
  const size_t Tm = std::max(1, cfg->max_tokens);
  L->ep.P = P;
  L->ep.rank = cfg->ep_rank;
  L->ep.fixed = cfg->ep_fixed_capacity != 0;
  const size_t rows = (size_t)P * Tm;
  // dispatched token rows: bf16 (2H bytes) or, FP8 layers, [H e4m3 codes | H/128 UE8M0 bytes]
  L->ep.row_bytes = L->fp8 ? ((H + H / 128 + 15) / 16) * 16 : 2 * H;
  CUDA_TRY(dalloc(L, &L->ep.send_x, rows * L->ep.row_bytes, false));
  CUDA_TRY(dalloc(L, &L->ep.send_idx, rows * k * 4, false));
  CUDA_TRY(dalloc(L, &L->ep.send_w, rows * k * 4, false));
  CUDA_TRY(dalloc(L, &L->ep.sendpos, Tm * P * 4, false));
  CUDA_TRY(dalloc(L, &L->ep.cnt_dev, 2 * P * 4, false));
  CUDA_TRY(dalloc(L, &L->ep.recv_x, rows * L->ep.row_bytes, false));
  CUDA_TRY(dalloc(L, &L->ep.partial, rows * H * 2, false));
  CUDA_TRY(dalloc(L, &L->ep.partial_def, rows * H * 2, false));
  CUDA_TRY(dalloc(L, &L->ep.back, rows * H * 2, false));
  CUDA_TRY(dalloc(L, &L->ep.back_def, rows * H * 2, false));
  CUDA_TRY(cudaMallocHost(reinterpret_cast<void **>(&L->ep.cnt_host), 2 * P * 4));
  if (cfg->nccl_unique_id && ep_nccl_init(&L->ep.comm, P, cfg->ep_rank, cfg->nccl_unique_id) != 0)
    return fail(MOE_ERR_NCCL, "ncclCommInitRank(P=%d, rank=%d) failed", P, cfg->ep_rank);
  return MOE_OK;
}

bool is_pow2(float v) {
  if (!(v > 0.f) || !std::isfinite(v)) return false;
  int e;
  float m = std::frexp(v, &e);
  return m == 0.5f;
}

// Repack [rows = 2F, cols] W13 into 128-row interleave: block 2b = W1 rows
// [128b, 128b+128), block 2b+1 = W3 rows [F + 128b, ...).  One 256-row GEMM N
// tile then holds matching gate/up columns (fused gate+up).
cudaError_t interleave_w13(const void *src, void *dst, int nexp, int F, int H, int es) {
  const size_t blk = (size_t)128 * H * es;
  for (int e = 0; e < nexp; ++e) {
    const char *s = reinterpret_cast<const char *>(src) + (size_t)e * 2 * F * H * es;
    char *d = reinterpret_cast<char *>(dst) + (size_t)e * 2 * F * H * es;
    cudaError_t r = cudaMemcpy2D(d, 2 * blk, s, blk, blk, F / 128, cudaMemcpyDeviceToDevice);
    if (r != cudaSuccess) return r;
    r = cudaMemcpy2D(d + blk, 2 * blk, s + (size_t)F * H * es, blk, blk, F / 128, cudaMemcpyDeviceToDevice);
    if (r != cudaSuccess) return r;
  }
  return cudaSuccess;
}

// scales: copy to host, check them (positive, finite; note any that is not a power of
// two -- the prefill GEMMs take UE8M0 scales only), optionally interleave like W13
moe_status load_scales(const float *src, float **dst, moe_layer *L, int nexp, int rows, int cols, bool inter,
                       const char *name, std::vector<float> *host_out = nullptr) {
  const int rb = rows / 128, cb = cols / 128;
  const size_t n = (size_t)nexp * rb * cb;
  std::vector<float> h(n), o(n);
  CUDA_TRY(cudaMemcpy(h.data(), src, n * sizeof(float), cudaMemcpyDeviceToHost));
  for (size_t i = 0; i < n; ++i) {
    if (!(h[i] > 0.f) || !std::isfinite(h[i]))
      return fail(MOE_ERR_INVALID_ARG, "%s[%zu] = %g is not a positive finite scale", name, i, (double)h[i]);
    if (!is_pow2(h[i]) && !L->scale_nonpow2) {
      L->scale_nonpow2 = true;
      snprintf(L->nonpow2_what, sizeof L->nonpow2_what, "%s[%zu] = %g", name, i, (double)h[i]);
    }
  }
  if (inter) {
    const int half = rb / 2;
    for (int e = 0; e < nexp; ++e)
      for (int b = 0; b < half; ++b)
        for (int c = 0; c < cb; ++c) {
          o[((size_t)e * rb + 2 * b) * cb + c] = h[((size_t)e * rb + b) * cb + c];
          o[((size_t)e * rb + 2 * b + 1) * cb + c] = h[((size_t)e * rb + half + b) * cb + c];
        }
  } else {
    o = h;
  }
  CUDA_TRY(dalloc(L, dst, n * sizeof(float), true));
  CUDA_TRY(cudaMemcpy(*dst, o.data(), n * sizeof(float), cudaMemcpyHostToDevice));
  if (host_out) *host_out = std::move(o);
  return MOE_OK;
}

// Scale image of a weight tensor for the tcgen05 block-scaled MMA: for every
// expert, group of 4 K-blocks and 128-row block, 128 identical 32-bit words
// holding the UE8M0 bytes of the 4 K-blocks (the tcgen05.cp source layout;
// every row of a 128x128 block shares the block's scale, R10).
moe_status build_weight_image(const std::vector<float> &s, int nexp, int rows, int cols, uint8_t **dst,
                              moe_layer *L, int64_t *expert_stride) {
  const int rb = rows / 128, kbn = cols / 128, G = (kbn + 3) / 4;
  const size_t per_exp = (size_t)G * rb * 512;
  std::vector<uint8_t> img((size_t)nexp * per_exp);
  for (int e = 0; e < nexp; ++e)
    for (int g = 0; g < G; ++g)
      for (int r = 0; r < rb; ++r) {
        uint8_t b[4];
        for (int j = 0; j < 4; ++j) {
          const int kb = 4 * g + j;
          uint32_t bits = 127u << 23;
          if (kb < kbn) {
            float v = s[((size_t)e * rb + r) * kbn + kb];
            memcpy(&bits, &v, 4);
          }
          b[j] = (uint8_t)((bits >> 23) & 0xFF);
        }
        uint8_t *d = img.data() + e * per_exp + ((size_t)g * rb + r) * 512;
        for (int w = 0; w < 128; ++w) memcpy(d + 4 * w, b, 4);
      }
  CUDA_TRY(dalloc(L, dst, img.size(), true));
  CUDA_TRY(cudaMemcpy(*dst, img.data(), img.size(), cudaMemcpyHostToDevice));
  *expert_stride = (int64_t)per_exp;
  return MOE_OK;
}

// W13 scale image for the swap-AB layout (umma_swap.cu / umma_decode.cu): one
// 512-byte image per (expert, group of 4 k-blocks, 128-column h block nb).  A
// 128-row CTA half of tile nb holds, per lane quadrant, [gate | up | gate | up]
// rows of block nb, so TMEM word w (= quadrant) of every lane takes the gate
// (w even) or up (w odd) block scale.  s = interleaved block scales from
// load_scales: [(e * 2F/128 + 2 nb (+1 up)) * H/128 + kb].
moe_status build_w13_swap_image(const std::vector<float> &s, int nexp, int F, int H, uint8_t **dst, moe_layer *L,
                                int64_t *expert_stride) {
  const int nbn = F / 128, rb = 2 * nbn, kbn = H / 128, G = (kbn + 3) / 4;
  const size_t per_exp = (size_t)G * nbn * 512;
  std::vector<uint8_t> img((size_t)nexp * per_exp);
  for (int e = 0; e < nexp; ++e)
    for (int g = 0; g < G; ++g)
      for (int nb = 0; nb < nbn; ++nb) {
        uint8_t b[2][4];
        for (int u = 0; u < 2; ++u)
          for (int j = 0; j < 4; ++j) {
            const int kb = 4 * g + j;
            uint32_t bits = 127u << 23;
            if (kb < kbn) {
              const float v = s[((size_t)e * rb + 2 * nb + u) * kbn + kb];
              memcpy(&bits, &v, 4);
            }
            b[u][j] = (uint8_t)((bits >> 23) & 0xFF);
          }
        uint8_t *d = img.data() + e * per_exp + ((size_t)g * nbn + nb) * 512;
        for (int l = 0; l < 32; ++l)
          for (int w = 0; w < 4; ++w) memcpy(d + 16 * l + 4 * w, b[w & 1], 4);
      }
  CUDA_TRY(dalloc(L, dst, img.size(), true));
  CUDA_TRY(cudaMemcpy(*dst, img.data(), img.size(), cudaMemcpyHostToDevice));
  *expert_stride = (int64_t)per_exp;
  return MOE_OK;
}

moe_status validate(const moe_layer_config *c, const moe_layer_weights *w) {
  if (!c || !w) return fail(MOE_ERR_INVALID_ARG, "null config or weights");
  if (c->hidden <= 0 || c->hidden % 128 || c->hidden > 8192)
    return fail(MOE_ERR_UNSUPPORTED, "hidden %d must be a positive multiple of 128, at most 8192", c->hidden);
  if (c->ffn <= 0 || c->ffn % 128) return fail(MOE_ERR_UNSUPPORTED, "ffn %d must be a positive multiple of 128", c->ffn);
  if (c->shared_ffn < 0 || c->shared_ffn % 128) return fail(MOE_ERR_UNSUPPORTED, "shared_ffn %d must be a multiple of 128", c->shared_ffn);
  if (c->n_experts <= 0 || c->n_experts > 1024) return fail(MOE_ERR_UNSUPPORTED, "n_experts %d not in [1, 1024]", c->n_experts);
  if (c->top_k <= 0 || c->top_k > 32 || c->top_k > c->n_experts) return fail(MOE_ERR_INVALID_ARG, "top_k %d invalid", c->top_k);
  if (c->n_group <= 0 || c->n_group > 32 || c->n_experts % c->n_group)
    return fail(MOE_ERR_INVALID_ARG, "n_group %d must divide n_experts and be <= 32", c->n_group);
  if (c->topk_group <= 0 || c->topk_group > c->n_group) return fail(MOE_ERR_INVALID_ARG, "topk_group %d invalid", c->topk_group);
  if (c->n_group > 1 && c->topk_group * (c->n_experts / c->n_group) < c->top_k)
    return fail(MOE_ERR_INVALID_ARG, "kept groups hold fewer than top_k experts");
  if (c->n_group > 1 && c->group_score == MOE_GROUP_TOP2_SUM && c->n_experts / c->n_group < 2)
    return fail(MOE_ERR_INVALID_ARG, "top-2 group score needs >= 2 experts per group");
  if (c->score_fn != MOE_SCORE_SOFTMAX && c->score_fn != MOE_SCORE_SIGMOID) return fail(MOE_ERR_INVALID_ARG, "score_fn");
  if (c->group_score != MOE_GROUP_MAX && c->group_score != MOE_GROUP_TOP2_SUM) return fail(MOE_ERR_INVALID_ARG, "group_score");
  if (c->wtype != MOE_W_BF16 && c->wtype != MOE_W_FP8_BLOCK128 && c->wtype != MOE_W_F32 && c->wtype != MOE_W_FP4_BLOCK128)
    return fail(MOE_ERR_INVALID_ARG, "wtype");
  if (c->wtype == MOE_W_FP4_BLOCK128 && c->hidden % 256)
    return fail(MOE_ERR_UNSUPPORTED, "FP4 weights need hidden %% 256 == 0 (the tensor-core paths)");
  if (c->max_tokens < 0) return fail(MOE_ERR_INVALID_ARG, "max_tokens");
  if (c->ep_size < 1 || c->ep_size > 32 || c->n_experts % c->ep_size)
    return fail(MOE_ERR_INVALID_ARG, "ep_size %d must be in [1, 32] and divide n_experts", c->ep_size);
  if (c->ep_rank < 0 || c->ep_rank >= c->ep_size) return fail(MOE_ERR_INVALID_ARG, "ep_rank %d", c->ep_rank);
  if (c->ep_fixed_capacity != 0 && c->ep_fixed_capacity != 1)
    return fail(MOE_ERR_INVALID_ARG, "ep_fixed_capacity %d (0 or 1)", c->ep_fixed_capacity);
  if (c->tp_size < 0 || c->tp_size > 32 || c->tp_rank < 0 || (c->tp_size > 1 && c->tp_rank >= c->tp_size))
    return fail(MOE_ERR_INVALID_ARG, "tp rank %d / size %d", c->tp_rank, c->tp_size);
  if (c->tp_size > 1) {
    if (c->ep_size > 1) return fail(MOE_ERR_UNSUPPORTED, "expert parallelism and expert TP together");
    if (c->ffn / 128 < c->tp_size || (c->shared_ffn > 0 && c->shared_ffn / 128 < c->tp_size))
      return fail(MOE_ERR_INVALID_ARG, "tp_size %d > 128-column chunks (ffn/128 = %d, shared_ffn/128 = %d)",
                  c->tp_size, c->ffn / 128, c->shared_ffn / 128);
    if (c->wtype == MOE_W_F32 || c->hidden % 256)
      return fail(MOE_ERR_UNSUPPORTED, "expert TP needs the tensor-core decode stream (bf16/fp8, hidden %% 256 == 0)");
  }
  if (!w->gate_w || !w->w13 || !w->w2) return fail(MOE_ERR_INVALID_ARG, "gate_w / w13 / w2 must be non-null");
  if ((c->wtype == MOE_W_FP8_BLOCK128 || c->wtype == MOE_W_FP4_BLOCK128) && (!w->w13_scale || !w->w2_scale))
    return fail(MOE_ERR_INVALID_ARG, "FP8 weights need w13_scale and w2_scale");
  if (c->shared_ffn > 0 && (!w->ws13 || !w->ws2)) return fail(MOE_ERR_INVALID_ARG, "shared_ffn > 0 needs ws13 / ws2");
  if (c->shared_ffn > 0 && (c->wtype == MOE_W_FP8_BLOCK128 || c->wtype == MOE_W_FP4_BLOCK128) &&
      (!w->ws13_scale || !w->ws2_scale))
    return fail(MOE_ERR_INVALID_ARG, "FP8 shared expert needs scales");
  if (c->shared_gated && (!w->shared_gate_w || c->shared_ffn == 0))
    return fail(MOE_ERR_INVALID_ARG, "shared_gated needs shared_gate_w and a shared expert");
  return MOE_OK;
}
}  // namespace

extern "C" {

const char *moe_status_string(moe_status s) {
  switch (s) {
    case MOE_OK: return "MOE_OK";
    case MOE_ERR_INVALID_ARG: return "MOE_ERR_INVALID_ARG";
    case MOE_ERR_UNSUPPORTED: return "MOE_ERR_UNSUPPORTED";
    case MOE_ERR_OOM: return "MOE_ERR_OOM";
    case MOE_ERR_CUDA: return "MOE_ERR_CUDA";
    case MOE_ERR_NCCL: return "MOE_ERR_NCCL";
    case MOE_ERR_CAPACITY: return "MOE_ERR_CAPACITY";
  }
  return "MOE_ERR_UNKNOWN";
}

const char *moe_last_error(void) { return g_err.c_str(); }

moe_status moe_get_unique_id(void *out128) {
  if (!out128) return fail(MOE_ERR_INVALID_ARG, "null out");
  if (ep_nccl_get_unique_id(out128) != 0) return fail(MOE_ERR_NCCL, "ncclGetUniqueId failed");
  return MOE_OK;
}

moe_status moe_layer_create(const moe_layer_config *cfg, const moe_layer_weights *w, moe_layer **out) {
  NvtxRange nvtx("moe_layer_create");
  if (!out) return fail(MOE_ERR_INVALID_ARG, "null out");
  *out = nullptr;
  moe_status st = validate(cfg, w);
  if (st != MOE_OK) return st;
  CUDA_TRY(cudaSetDevice(cfg->device));

  moe_layer *L = new moe_layer();
  L->cfg = *cfg;
  L->cfg.nccl_unique_id = nullptr;
  L->E_glob = cfg->n_experts;
  L->E = cfg->n_experts / cfg->ep_size;
  L->e0 = cfg->ep_rank * L->E;
  L->k = cfg->top_k;
  L->H = cfg->hidden;
  L->F_full = cfg->ffn;
  L->Fs_full = cfg->shared_ffn;
  L->tp_size = cfg->tp_size > 1 ? cfg->tp_size : 1;
  L->tp_rank = L->tp_size > 1 ? cfg->tp_rank : 0;
  {
    // TP: rank r holds chunks [r n / P, (r+1) n / P) of the n 128-column chunks
    auto slice = [&](int full) {
      const int n = full / 128, P = L->tp_size, r = L->tp_rank;
      return ((r + 1) * n / P - r * n / P) * 128;
    };
    L->F = slice(cfg->ffn);
    L->Fs = cfg->shared_ffn > 0 ? slice(cfg->shared_ffn) : 0;
  }
  L->fp4 = cfg->wtype == MOE_W_FP4_BLOCK128;
  L->fp8 = cfg->wtype == MOE_W_FP8_BLOCK128 || L->fp4;   // FP4: e4m3 activations, e4m3-expanded prefill weights
  L->f32w = cfg->wtype == MOE_W_F32;
  L->act_bytes = L->fp8 ? 1 : 2;
  L->max_tokens = cfg->max_tokens;
  const int H = L->H, F = L->F, Fs = L->Fs, E = L->E, k = L->k;
  const int wes = L->fp8 ? 1 : (L->f32w ? 4 : 2);
  auto cleanup = [&](moe_status s) { free_all(L); delete L; return s; };
#define C_TRY(expr)                                                                            \
  do {                                                                                         \
    cudaError_t _e = (expr);                                                                   \
    if (_e != cudaSuccess)                                                                     \
      return cleanup(fail(_e == cudaErrorMemoryAllocation ? MOE_ERR_OOM : MOE_ERR_CUDA, "%s: %s", #expr, \
                          cudaGetErrorString(_e)));                                            \
  } while (0)
#define S_TRY(expr)                      \
  do {                                   \
    moe_status _s = (expr);              \
    if (_s != MOE_OK) return cleanup(_s); \
  } while (0)

  // ---- router weights (+ Qwen2 shared gate as one extra row) ----
  L->gate_rows = L->E_glob + (cfg->shared_gated ? 1 : 0);
  C_TRY(dalloc(L, &L->gate_w, (size_t)L->gate_rows * H * 2, true));
  C_TRY(cudaMemcpy(L->gate_w, w->gate_w, (size_t)L->E_glob * H * 2, cudaMemcpyDeviceToDevice));
  if (cfg->shared_gated)
    C_TRY(cudaMemcpy(reinterpret_cast<char *>(L->gate_w) + (size_t)L->E_glob * H * 2, w->shared_gate_w,
                     (size_t)H * 2, cudaMemcpyDeviceToDevice));
  if (w->gate_bias) {
    C_TRY(dalloc(L, &L->gate_bias, (size_t)L->E_glob * 4, true));
    C_TRY(cudaMemcpy(L->gate_bias, w->gate_bias, (size_t)L->E_glob * 4, cudaMemcpyDeviceToDevice));
  }
  // ---- routed experts ----
  // FP4 (e2m1, 2 per byte): the decode stream reads the packed codes (W13 rows in its tile
  // order) through 16U4_ALIGN16B tensor maps; the prefill GEMMs run on the exact e4m3
  // expansion of the same codes (e2m1 is a subset of e4m3; same power-of-two block scales)
  struct Expand {
    void *buf = nullptr;
    ~Expand() { if (buf) cudaFree(buf); }
  } ex13, ex2, exs13, exs2;
  const void *src13 = w->w13, *src2 = w->w2, *srcs13 = w->ws13, *srcs2 = w->ws2;
  if (L->fp4) {
    C_TRY(dalloc(L, &L->w13_f4, (size_t)E * 2 * F * H / 2, true));
    C_TRY(launch_permute_w13_rows(w->w13, L->w13_f4, E, F, H / 2, 0));
    C_TRY(dalloc(L, &L->w2_f4, (size_t)E * H * F / 2, true));
    C_TRY(cudaMemcpy(L->w2_f4, w->w2, (size_t)E * H * F / 2, cudaMemcpyDeviceToDevice));
    C_TRY(cudaMalloc(&ex13.buf, (size_t)E * 2 * F * H));
    C_TRY(launch_fp4_to_e4m3(w->w13, ex13.buf, (int64_t)E * 2 * F * H / 2, 0));
    C_TRY(cudaMalloc(&ex2.buf, (size_t)E * H * F));
    C_TRY(launch_fp4_to_e4m3(w->w2, ex2.buf, (int64_t)E * H * F / 2, 0));
    src13 = ex13.buf; src2 = ex2.buf;
    if (Fs > 0) {
      C_TRY(dalloc(L, &L->ws13_f4, (size_t)2 * Fs * H / 2, true));
      C_TRY(launch_permute_w13_rows(w->ws13, L->ws13_f4, 1, Fs, H / 2, 0));
      C_TRY(dalloc(L, &L->ws2_f4, (size_t)H * Fs / 2, true));
      C_TRY(cudaMemcpy(L->ws2_f4, w->ws2, (size_t)H * Fs / 2, cudaMemcpyDeviceToDevice));
      C_TRY(cudaMalloc(&exs13.buf, (size_t)2 * Fs * H));
      C_TRY(launch_fp4_to_e4m3(w->ws13, exs13.buf, (int64_t)Fs * H, 0));
      C_TRY(cudaMalloc(&exs2.buf, (size_t)H * Fs));
      C_TRY(launch_fp4_to_e4m3(w->ws2, exs2.buf, (int64_t)H * Fs / 2, 0));
      srcs13 = exs13.buf; srcs2 = exs2.buf;
    }
    bool ok = make_fp4_map(&L->fmap_w13, L->w13_f4, (int64_t)E * 2 * F, H, 256) &&
              make_fp4_map(&L->fmap_w2, L->w2_f4, (int64_t)E * H, F, 256);
    if (Fs > 0)
      ok = ok && make_fp4_map(&L->fmap_ws13, L->ws13_f4, 2 * Fs, H, 256) && make_fp4_map(&L->fmap_ws2, L->ws2_f4, H, Fs, 256);
    if (!ok) return cleanup(fail(MOE_ERR_CUDA, "cuTensorMapEncodeTiled failed for the FP4 weights"));
  }
  C_TRY(dalloc(L, &L->w13, (size_t)E * 2 * F * H * wes, true));
  L->umma = !L->f32w && (H % 256 == 0);
  // tcgen05 path: weights repacked into 256-row x 128-byte SW128 tiles (one
  // contiguous 32 KB read per k-block); CUDA-core path: row-major, W13 interleaved
  if (L->umma) C_TRY(launch_tile_weights(src13, L->w13, E, 2 * F, H * wes, F, 0));
  else C_TRY(interleave_w13(src13, L->w13, E, F, H, wes));
  C_TRY(dalloc(L, &L->w2, (size_t)E * H * F * wes, true));
  if (L->umma) C_TRY(launch_tile_weights(src2, L->w2, E, H, F * wes, 0, 0));
  else C_TRY(cudaMemcpy(L->w2, src2, (size_t)E * H * F * wes, cudaMemcpyDeviceToDevice));
  std::vector<float> hs13, hs2, hss13, hss2;
  if (L->fp8) {
    if (!L->umma) return cleanup(fail(MOE_ERR_UNSUPPORTED, "FP8 weights need hidden %% 256 == 0"));
    S_TRY(load_scales(w->w13_scale, &L->w13_s, L, E, 2 * F, H, true, "w13_scale", &hs13));
    S_TRY(load_scales(w->w2_scale, &L->w2_s, L, E, H, F, false, "w2_scale", &hs2));
  }
  if (Fs > 0) {
    C_TRY(dalloc(L, &L->ws13, (size_t)2 * Fs * H * wes, true));
    if (L->umma) C_TRY(launch_tile_weights(srcs13, L->ws13, 1, 2 * Fs, H * wes, Fs, 0));
    else C_TRY(interleave_w13(srcs13, L->ws13, 1, Fs, H, wes));
    C_TRY(dalloc(L, &L->ws2, (size_t)H * Fs * wes, true));
    if (L->umma) C_TRY(launch_tile_weights(srcs2, L->ws2, 1, H, Fs * wes, 0, 0));
    else C_TRY(cudaMemcpy(L->ws2, srcs2, (size_t)H * Fs * wes, cudaMemcpyDeviceToDevice));
    if (L->fp8) {
      S_TRY(load_scales(w->ws13_scale, &L->ws13_s, L, 1, 2 * Fs, H, true, "ws13_scale", &hss13));
      S_TRY(load_scales(w->ws2_scale, &L->ws2_s, L, 1, H, Fs, false, "ws2_scale", &hss2));
    }
  }

  // ---- workspace, sized for max_tokens ----
  const int64_t Tm = std::max(1, cfg->max_tokens);
  // expert-parallel: the expert side processes the rows every rank sends here,
  // at most ep_size * max_tokens (each rank sends a token to a rank at most once)
  const int64_t Tr = Tm * cfg->ep_size;
  L->max_rows = (int)Tr;
  const int64_t pairs = Tr * k;
  L->R_max = pairs + (int64_t)E * kPadM;
  L->max_tiles = (int)(L->R_max / kPadM);
  L->nchunk_max = (int)((Tr + kChunkTokens - 1) / kChunkTokens);
  const int ab = L->act_bytes;
  C_TRY(dalloc(L, &L->logits, (size_t)Tm * L->gate_rows * 4, false));
  C_TRY(cudaMemset(L->logits, 0, (size_t)Tm * L->gate_rows * 4));   // finite for the router's warm-up pass
  if (cfg->ep_size > 1 || (cfg->nccl_unique_id && L->tp_size == 1)) S_TRY(ep_create(L, cfg));
  C_TRY(dalloc(L, &L->topk_idx, (size_t)pairs * 4, false));
  C_TRY(dalloc(L, &L->topk_w, (size_t)pairs * 4, false));
  C_TRY(dalloc(L, &L->sgate, (size_t)Tm * 4, false));
  C_TRY(dalloc(L, &L->chunk_cnt, (size_t)L->nchunk_max * E * 4, false));
  C_TRY(dalloc(L, &L->chunk_base, (size_t)L->nchunk_max * E * 4, false));
  C_TRY(dalloc(L, &L->counts, (size_t)E * 4, false));
  C_TRY(dalloc(L, &L->offs, (size_t)(E + 1) * 4, false));
  C_TRY(dalloc(L, &L->offs_pad, (size_t)(E + 1) * 4, false));
  C_TRY(dalloc(L, &L->tiles, (size_t)L->max_tiles * sizeof(int4), false));
  C_TRY(dalloc(L, &L->n_tiles, 4, false));
  C_TRY(dalloc(L, &L->act_list, (size_t)E * 4, false));
  C_TRY(dalloc(L, &L->n_active, 4, false));
  C_TRY(dalloc(L, &L->imm_list, (size_t)E * 4, false));
  C_TRY(dalloc(L, &L->def_list, (size_t)E * 4, false));
  C_TRY(dalloc(L, &L->n_lists, 8, false));
  C_TRY(cudaMemset(L->n_lists, 0, 8));
  C_TRY(dalloc(L, &L->sched, 32, false));
  C_TRY(cudaMemset(L->sched, 0, 32));
  C_TRY(dalloc(L, &L->pairs, (size_t)L->max_tiles * sizeof(int4), false));
  C_TRY(dalloc(L, &L->n_pairs, 4, false));
  C_TRY(dalloc(L, &L->row_token, (size_t)L->R_max * 4, false));
  C_TRY(dalloc(L, &L->pos, (size_t)pairs * 4, false));
  if (L->fp8) {
    C_TRY(dalloc(L, &L->xq, (size_t)Tm * H, false));
    C_TRY(dalloc(L, &L->xs, (size_t)Tm * (H / 128) * 4, false));
    C_TRY(dalloc(L, &L->xperm_s, (size_t)L->R_max * (H / 128) * 4, false));
    C_TRY(dalloc(L, &L->h_s, (size_t)L->R_max * (F / 128) * 4, false));
    if (Fs) C_TRY(dalloc(L, &L->hsh_s, (size_t)Tm * (Fs / 128) * 4, false));
  }
  C_TRY(dalloc(L, &L->xperm, (size_t)L->R_max * H * ab, false));
  C_TRY(dalloc(L, &L->hbuf, (size_t)L->R_max * F * ab, false));
  C_TRY(dalloc(L, &L->yperm, (size_t)L->R_max * H * 2, false));
  if (Fs) {
    C_TRY(dalloc(L, &L->hsh, (size_t)Tm * Fs * ab, false));
    C_TRY(dalloc(L, &L->ysh, (size_t)Tm * H * 2, false));
  }
  C_TRY(cudaMemset(L->row_token, 0xff, (size_t)L->R_max * 4));
  // padding rows of the sorted activations are read by the GEMM tiles but never
  // written by the scatter: start them at zero (finite) once
  C_TRY(cudaMemset(L->xperm, 0, (size_t)L->R_max * H * ab));

  // ---- tcgen05 path: scale images and tensor maps ----
  C_TRY(cudaDeviceGetAttribute(&L->num_sms, cudaDevAttrMultiProcessorCount, cfg->device));
  if (L->umma) L->swap_clusters4 = umma_swap_max_clusters4(L->fp8);
  if (!make_kmajor_map(&L->map_gate, L->gate_w, false, L->gate_rows, H, 256))
    return cleanup(fail(MOE_ERR_CUDA, "cuTensorMapEncodeTiled failed for the router weights"));
  {
    // decode switch (the L170 analog): weight streaming for T <= gemv_max_tokens
    // tensor-core decode (swap-AB, N = 16 tokens) when the tcgen05 path is
    // available, else the CUDA-core GEMV for up to 8 tokens
    const bool tc = !L->f32w && (H % 256 == 0);
    int g = cfg->gemv_max_tokens > 0 ? cfg->gemv_max_tokens : (tc ? 16 : 4);
    g = std::min(g, tc ? 16 : kGemvMaxTokens);
    if (!tc)
      while (g > 0 && gemv_smem_bytes(g, H, F, Fs) > 200 * 1024) --g;
    L->gemv_max_tokens = L->f32w ? 0 : g;
    L->gemv_ok = L->gemv_max_tokens > 0;
  }
  if (L->umma) {
    const bool f8 = L->fp8;
    L->img_tiles_sh = (int)((Tm + 127) / 128);
    if (f8) {
      int64_t st;
      S_TRY(build_w13_swap_image(hs13, E, F, H, &L->w13_img, L, &st)); L->w13_img_stride = st;
      S_TRY(build_weight_image(hs2, E, H, F, &L->w2_img, L, &st)); L->w2_img_stride = st;
      if (Fs) {
        S_TRY(build_w13_swap_image(hss13, 1, Fs, H, &L->ws13_img, L, &st));
        S_TRY(build_weight_image(hss2, 1, H, Fs, &L->ws2_img, L, &st));
      }
      const size_t g1 = (H / 128 + 3) / 4, g2 = (F / 128 + 3) / 4, gs = (Fs / 128 + 3) / 4;
      C_TRY(dalloc(L, &L->xperm_img, g1 * L->max_tiles * 512, false));
      C_TRY(dalloc(L, &L->h_img, g2 * L->max_tiles * 512, false));
      C_TRY(dalloc(L, &L->xq_img, g1 * L->img_tiles_sh * 512, false));
      C_TRY(cudaMemset(L->xperm_img, 127, g1 * L->max_tiles * 512));
      C_TRY(cudaMemset(L->h_img, 127, g2 * L->max_tiles * 512));
      C_TRY(cudaMemset(L->xq_img, 127, g1 * L->img_tiles_sh * 512));
      if (Fs) {
        C_TRY(dalloc(L, &L->hsh_img, gs * L->img_tiles_sh * 512, false));
        C_TRY(cudaMemset(L->hsh_img, 127, gs * L->img_tiles_sh * 512));
      }
    }
    bool ok = make_kmajor_map(&L->map_xperm, L->xperm, f8, L->R_max, H, 128) &&
              make_kmajor_map(&L->map_h, L->hbuf, f8, L->R_max, F, 128);
    if (Fs) {
      ok = ok && make_kmajor_map(&L->map_hsh, L->hsh, f8, Tm, Fs, 128);
      if (f8) ok = ok && make_kmajor_map(&L->map_xq, L->xq, true, Tm, H, 128);
    }
    ok = ok && make_kmajor_map(&L->dmap_xperm, L->xperm, f8, L->R_max, H, 16) &&
         make_kmajor_map(&L->dmap_h, L->hbuf, f8, L->R_max, F, 16);
    if (Fs) ok = ok && make_kmajor_map(&L->dmap_hsh, L->hsh, f8, Tm, Fs, 16);
    if (f8) ok = ok && make_kmajor_map(&L->dmap_xq, L->xq, true, Tm, H, 16);   // fused decode + shared expert
    // swap-AB pair GEMM maps: tiled weights as 128-byte rows, token rows (box 32),
    // scale images as 512-byte rows (weights: box 1 per CTA; tokens: box 2 = 256 rows)
    {
      const int64_t es = f8 ? 1 : 2;
      // weights: 2 KB TMA rows (a CTA's 16 KB half tile = 8 rows)
      ok = ok && make_blocks_map(&L->tmap_w13, L->w13, (int64_t)E * 2 * F * H * es, 2048, 8) &&
           make_blocks_map(&L->tmap_w2, L->w2, (int64_t)E * H * F * es, 2048, 8) &&
           make_kmajor_map(&L->xmap_xperm, L->xperm, f8, L->R_max, H, 32) &&
           make_kmajor_map(&L->xmap_h, L->hbuf, f8, L->R_max, F, 32) &&
           make_kmajor_map(&L->x64map_xperm, L->xperm, f8, L->R_max, H, 64) &&
           make_kmajor_map(&L->x64map_h, L->hbuf, f8, L->R_max, F, 64);
      if (Fs) {
        ok = ok && make_blocks_map(&L->tmap_ws13, L->ws13, (int64_t)2 * Fs * H * es, 2048, 8) &&
             make_blocks_map(&L->tmap_ws2, L->ws2, (int64_t)H * Fs * es, 2048, 8) &&
             make_kmajor_map(&L->xmap_hsh, L->hsh, f8, Tm, Fs, 32) &&
             make_kmajor_map(&L->x64map_hsh, L->hsh, f8, Tm, Fs, 64);
        if (f8) ok = ok && make_kmajor_map(&L->xmap_xq, L->xq, true, Tm, H, 32) &&
                     make_kmajor_map(&L->x64map_xq, L->xq, true, Tm, H, 64);
      }
      if (f8) {
        const int64_t g1 = (H / 128 + 3) / 4, g2 = (F / 128 + 3) / 4, gs = (Fs / 128 + 3) / 4;
        ok = ok && make_rows_map(&L->smap_w13, L->w13_img, true, E * g1 * (F / 128), 128, 1) &&
             make_rows_map(&L->smap_w2, L->w2_img, true, E * g2 * (H / 128), 128, 1) &&
             make_rows_map(&L->smap_xperm, L->xperm_img, true, g1 * L->max_tiles, 128, 2) &&
             make_rows_map(&L->smap_h, L->h_img, true, g2 * L->max_tiles, 128, 2) &&
             make_rows_map(&L->smap_xq, L->xq_img, true, g1 * L->img_tiles_sh, 128, 2);
        if (Fs)
          ok = ok && make_rows_map(&L->smap_ws13, L->ws13_img, true, g1 * (Fs / 128), 128, 1) &&
               make_rows_map(&L->smap_ws2, L->ws2_img, true, gs * (H / 128), 128, 1) &&
               make_rows_map(&L->smap_hsh, L->hsh_img, true, gs * L->img_tiles_sh, 128, 2);
      }
    }
    if (!ok) return cleanup(fail(MOE_ERR_CUDA, "cuTensorMapEncodeTiled failed (driver entry point unavailable?)"));
    if (getenv("MOE_DEBUG_TRACE")) {               // timing experiments: device timeline buffer
      C_TRY(dalloc(L, &L->trace, 4096 * 8, false));
      C_TRY(cudaMemset(L->trace, 0, 4096 * 8));
    }
    L->fused_decode = L->gemv_ok;            // decode (T <= 16): the fused stream of umma_decode_fused.cu
    if (L->fused_decode) {
      const size_t n = (size_t)2 * L->gemv_max_tokens * H * 4;
      C_TRY(dalloc(L, &L->dacc, n, false));
      C_TRY(cudaMemset(L->dacc, 0, n));
      C_TRY(dalloc(L, &L->zero_i32, 16, false));   // [0] = 0, [1..2] a second stream work counter
      C_TRY(cudaMemset(L->zero_i32, 0, 16));
      // cluster split of the stream (few units): how many clusters of 2 / 4 / 8 fit, and the
      // L2 scratch the peers hand their fp32 partials to the leader through
      for (int c = 2; c <= 8; c *= 2) L->fd_max_clusters[c] = fused_decode_max_clusters(f8, c);
      const int ncl = std::max(L->fd_max_clusters[2], 1);
      C_TRY(dalloc(L, &L->cl_scratch, (size_t)ncl * 7 * 128 * 32 * 4, false));
      if (!f8) {
        C_TRY(dalloc(L, &L->xcopy, (size_t)L->gemv_max_tokens * H * 2, false));
        C_TRY(cudaMemset(L->xcopy, 0, (size_t)L->gemv_max_tokens * H * 2));
        if (!make_kmajor_map(&L->dmap_xc, L->xcopy, false, L->gemv_max_tokens, H, 16))
          return cleanup(fail(MOE_ERR_CUDA, "cuTensorMapEncodeTiled failed for the decode x copy"));
      }
    }
  }
  if (L->scale_nonpow2) {
    // arbitrary fp32 block scales (e.g. the released DeepSeek-V3/V2.5 FP8 checkpoints' weight_scale_inv):
    // the decode stream applies the weight scales in its epilogues (any fp32 value is exact there);
    // the prefill GEMMs' block-scaled MMAs take UE8M0 (power-of-two) scales only
    if (!(L->fused_decode && L->E_glob <= 256 && cfg->ep_size == 1 && cfg->max_tokens <= L->gemv_max_tokens))
      return cleanup(fail(MOE_ERR_UNSUPPORTED,
                          "%s is not a power of two: non-UE8M0 block scales are served by the decode stream only "
                          "(max_tokens <= %d, no expert parallelism); the prefill GEMMs need UE8M0 scales "
                          "(DESIGN.md R10)", L->nonpow2_what, L->gemv_max_tokens));
  }
  if (L->tp_size > 1) {
    if (!L->fused_decode) return cleanup(fail(MOE_ERR_UNSUPPORTED, "expert TP needs the fused decode stream"));
    if (cfg->nccl_unique_id && ep_nccl_init(&L->tp_comm, L->tp_size, L->tp_rank, cfg->nccl_unique_id) != 0)
      return cleanup(fail(MOE_ERR_NCCL, "ncclCommInitRank(P=%d, rank=%d) failed (TP)", L->tp_size, L->tp_rank));
  }
  C_TRY(cudaDeviceSynchronize());
#undef C_TRY
#undef S_TRY
  *out = L;
  return MOE_OK;
}

static const char *kStageNames[moe_layer::kStages] = {
    "router_logits", "router_select", "permute", "act_quant", "quant_scatter", "gemm1_swiglu", "gemm2",
    "shared_gemm1", "shared_gemm2", "combine"};
enum { ST_LOGITS = 0, ST_SELECT, ST_PERMUTE, ST_QUANT, ST_GATHER, ST_GEMM1, ST_GEMM2, ST_SH1, ST_SH2, ST_COMBINE };

static inline void mark(moe_layer *L, int stage, cudaStream_t st) {
  nvtxMarkA(kStageNames[stage]);
  if (!L->prof) return;
  cudaEventRecord(L->ev[stage + 1], st);
  L->ev_hit[stage + 1] = true;
}

// Prefill-shaped expert GEMMs: routed experts over the sorted rows described by
// L->tiles (built by the permutation) and the shared expert over T_shared token
// rows (FP8: L->xq, quantised by the scatter; BF16: x_shared).
// CTA pairs per cluster of the swap GEMM: 2 (token boxes multicast to two pairs that take
// adjacent weight blocks) when both groups' weight-block counts are even and enough clusters
// of 4 fit, else 1.  MOE_SWAP_NP1 / MOE_SWAP_NP2 = 1 or 2 choose per GEMM (A/B experiments).
static int swap_np(const moe_layer *L, int gemm, int nb_r, int nb_s, int dbg_mode) {
  // default: pairs for both GEMMs.  Clusters of 4 fit only 33 times on a B200 (132 of 148 SMs):
  // per unit 7 % faster, per launch 2-5 % slower (interleaved A/B, profiles/r02/swap_np.txt)
  static const int force1 = getenv("MOE_SWAP_NP1") ? atoi(getenv("MOE_SWAP_NP1")) : 1;
  static const int force2 = getenv("MOE_SWAP_NP2") ? atoi(getenv("MOE_SWAP_NP2")) : 1;
  if ((gemm == 1 ? force1 : force2) == 1 || dbg_mode != 0) return 1;
  if ((nb_r & 1) || (nb_s & 1) || 4 * L->swap_clusters4 < L->num_sms * 3 / 4) return 1;
  return 2;
}

static moe_status run_expert_gemms(moe_layer *L, int tile_bound, const void *x_shared, int T_shared,
                                   cudaStream_t st) {
  const int H = L->H, F = L->F, Fs = T_shared > 0 ? L->Fs : 0;
  const int T = T_shared;
  const void *x = x_shared;
  const void *xa = L->fp8 ? L->xq : x_shared;
  const float *xa_s = L->fp8 ? L->xs : nullptr;
  const int btype = L->fp8 ? WT_FP8 : (L->f32w ? WT_F32 : WT_BF16);
  if (L->umma) {
    // 5+6. routed experts and the shared expert in one persistent swap-AB CTA-pair
    // tcgen05 launch per GEMM (umma_swap.cu)
    const bool f8 = L->fp8;
    const int kdiv = f8 ? 128 : 64;
    static const int dbg_mode = experiment_knob("MOE_DEBUG_GEMM");   // timing experiments (MOE_EXPERIMENTS builds)
    SwapParams p1{};
    {
      SwapGroup &g = p1.g[0];
      g.w_map = L->tmap_w13; g.x_map = L->xmap_xperm; g.x_map128 = L->map_xperm; g.x_map64 = L->x64map_xperm; g.x_map16 = L->dmap_xperm;
      g.sfw_map = L->smap_w13; g.sfx_map = L->smap_xperm;
      g.w_nblk = F / 128; g.kblocks = H / kdiv; g.sfw_per_cta = 0; g.sfx_tile_stride = L->max_tiles;
      g.out = L->hbuf; g.ldc = F; g.out_sf = L->h_img; g.out_sf_tile_stride = L->max_tiles;
    }
    if (Fs > 0) {
      SwapGroup &g = p1.g[1];
      g.w_map = L->tmap_ws13; g.sfw_map = L->smap_ws13; g.sfx_map = L->smap_xq;
      if (f8) {
        g.x_map = L->xmap_xq; g.x_map128 = L->map_xq; g.x_map64 = L->x64map_xq; g.x_map16 = L->dmap_xq;
      } else if (!make_kmajor_map(&g.x_map, x, false, T, H, 32) || !make_kmajor_map(&g.x_map128, x, false, T, H, 128) ||
                 !make_kmajor_map(&g.x_map64, x, false, T, H, 64) || !make_kmajor_map(&g.x_map16, x, false, T, H, 16)) {
        return fail(MOE_ERR_CUDA, "cuTensorMapEncodeTiled failed for x");
      }
      g.w_nblk = Fs / 128; g.kblocks = H / kdiv; g.sfw_per_cta = 0; g.sfx_tile_stride = L->img_tiles_sh;
      g.out = L->hsh; g.ldc = Fs; g.out_sf = L->hsh_img; g.out_sf_tile_stride = L->img_tiles_sh;
    } else {
      p1.g[1] = p1.g[0];
    }
    // clusters of 2 CTA pairs (adjacent weight blocks, token boxes multicast to both pairs)
    // when every operand group has an even number of weight blocks
    const int np1 = swap_np(L, 1, F / 128, Fs / 128, dbg_mode), np2 = swap_np(L, 2, H / 256, Fs > 0 ? H / 256 : 0, dbg_mode);
    p1.tiles = L->pairs; p1.n_tiles = L->n_pairs; p1.nb_r = F / 128 / np1;
    p1.T_shared = Fs > 0 ? T : 0; p1.nb_s = Fs / 128 / np1; p1.sched = L->sched; p1.debug_mode = dbg_mode; p1.trace = L->trace;
    KL_TRY(launch_umma_swap_gemm(f8, GEMM_SWIGLU, p1, np1 == 2 ? L->swap_clusters4 : L->num_sms, np1, st));
    mark(L, ST_GEMM1, st);
    SwapParams p2{};
    {
      SwapGroup &g = p2.g[0];
      g.w_map = L->tmap_w2; g.x_map = L->xmap_h; g.x_map128 = L->map_h; g.x_map64 = L->x64map_h; g.x_map16 = L->dmap_h;
      g.sfw_map = L->smap_w2; g.sfx_map = L->smap_h;
      g.w_nblk = H / 256; g.kblocks = F / kdiv; g.sfw_per_cta = 1; g.sfx_tile_stride = L->max_tiles;
      g.out = L->yperm; g.ldc = H;
    }
    if (Fs > 0) {
      SwapGroup &g = p2.g[1];
      g.w_map = L->tmap_ws2; g.x_map = L->xmap_hsh; g.x_map128 = L->map_hsh; g.x_map64 = L->x64map_hsh; g.x_map16 = L->dmap_hsh;
      g.sfw_map = L->smap_ws2; g.sfx_map = L->smap_hsh;
      g.w_nblk = H / 256; g.kblocks = Fs / kdiv; g.sfw_per_cta = 1; g.sfx_tile_stride = L->img_tiles_sh;
      g.out = L->ysh; g.ldc = H;
    } else {
      p2.g[1] = p2.g[0];
    }
    p2.tiles = L->pairs; p2.n_tiles = L->n_pairs; p2.nb_r = H / 256 / np2;
    p2.T_shared = Fs > 0 ? T : 0; p2.nb_s = H / 256 / np2; p2.sched = L->sched + 1; p2.debug_mode = dbg_mode; p2.trace = L->trace ? L->trace + 2048 : nullptr;
    KL_TRY(launch_umma_swap_gemm(f8, GEMM_PLAIN, p2, np2 == 2 ? L->swap_clusters4 : L->num_sms, np2, st));
    mark(L, ST_GEMM2, st);
  } else {
    // 5. routed experts: GEMM1 + SwiGLU, GEMM2 (CUDA-core path: F32 weights, H % 256 != 0)
    SimtGemmArgs a{};
    a.A = L->xperm; a.As = L->xperm_s; a.lda = H; a.a_fp8 = L->fp8;
    a.B = L->w13; a.Bs = L->w13_s; a.b_stride = (int64_t)2 * F * H; a.bs_stride = (int64_t)(2 * F / 128) * (H / 128);
    a.b_type = btype; a.N = 2 * F; a.K = H;
    a.tiles = L->tiles; a.n_tiles = L->n_tiles;
    a.C = L->hbuf; a.Cs = L->h_s; a.ldc = F; a.out_fp8 = L->fp8;
    KL_TRY(launch_simt_gemm(GEMM_SWIGLU, a, 2 * tile_bound, st));
    mark(L, ST_GEMM1, st);
    SimtGemmArgs b{};
    b.A = L->hbuf; b.As = L->h_s; b.lda = F; b.a_fp8 = L->fp8;
    b.B = L->w2; b.Bs = L->w2_s; b.b_stride = (int64_t)H * F; b.bs_stride = (int64_t)(H / 128) * (F / 128);
    b.b_type = btype; b.N = H; b.K = F;
    b.tiles = L->tiles; b.n_tiles = L->n_tiles;
    b.C = L->yperm; b.ldc = H;
    KL_TRY(launch_simt_gemm(GEMM_PLAIN, b, 2 * tile_bound, st));
    mark(L, ST_GEMM2, st);
    // 6. shared expert on every token
    if (Fs > 0) {
      SimtGemmArgs a{};
      a.A = xa; a.As = xa_s; a.lda = H; a.a_fp8 = L->fp8;
      a.B = L->ws13; a.Bs = L->ws13_s; a.b_type = btype; a.N = 2 * Fs; a.K = H;
      a.M = T; a.C = L->hsh; a.Cs = L->hsh_s; a.ldc = Fs; a.out_fp8 = L->fp8;
      KL_TRY(launch_simt_gemm(GEMM_SWIGLU, a, (T + 63) / 64, st));
      mark(L, ST_SH1, st);
      SimtGemmArgs b{};
      b.A = L->hsh; b.As = L->hsh_s; b.lda = Fs; b.a_fp8 = L->fp8;
      b.B = L->ws2; b.Bs = L->ws2_s; b.b_type = btype; b.N = H; b.K = Fs;
      b.M = T; b.C = L->ysh; b.ldc = H;
      KL_TRY(launch_simt_gemm(GEMM_PLAIN, b, (T + 63) / 64, st));
      mark(L, ST_SH2, st);
    }
  }
  return MOE_OK;
}


// ======================================================================
// Expert parallelism: rank r owns experts [e0, e0 + E_loc).
//   A  route own tokens, plan + pack one row per (token, destination rank)
//   -- exchange counts, rows + (masked expert ids, weights) --
//   C  expert side: permute the received rows by local expert, FP8-quantise,
//      grouped GEMMs (+ the shared expert on the own tokens), weighted partial
//      sums per received row (immediate / deferred)
//   -- return the partial rows to their origin --
//   D  origin: y = residual + shared + sum of partials (+ deferred_in)
// ======================================================================
// router logits of T > 8 tokens: tcgen05 BF16 GEMM (umma_gemm.cu), fp32 out (reading R9)
static moe_status launch_logits(moe_layer *L, const void *x, int T, cudaStream_t st) {
  LogitsParams p{};
  if (!make_kmajor_map(&p.a_map, x, false, T, L->H, 128)) return fail(MOE_ERR_CUDA, "tensor map for x failed");
  p.b_map = L->map_gate;
  p.kblocks = L->H / 64; p.out = L->logits; p.ldc = L->gate_rows; p.n_valid = L->gate_rows;
  p.T = T; p.nb = (L->gate_rows + 255) / 256; p.sched = L->sched + 2;
  const int units = ((T + 127) / 128) * p.nb;
  KL_TRY(launch_umma_logits(p, std::min(units, L->num_sms), st));
  return MOE_OK;
}

static moe_status run_router_full(moe_layer *L, const void *x, int T, cudaStream_t st) {
  if (T <= 0) return MOE_OK;
  const int H = L->H;
  if (T <= kGemvMaxTokens) {
    KL_TRY(launch_router_gemv(x, T, H, L->gate_w, L->gate_rows, L->logits, st));
  } else {
    moe_status s = launch_logits(L, x, T, st);
    if (s != MOE_OK) return s;
  }
  RouterArgs r{};
  r.logits = L->logits; r.ldl = L->gate_rows; r.bias = L->gate_bias;
  r.T = T; r.E = L->E_glob; r.k = L->k; r.n_group = L->cfg.n_group; r.topk_group = L->cfg.topk_group;
  r.group_score = L->cfg.group_score; r.score_fn = L->cfg.score_fn; r.norm_topk = L->cfg.norm_topk;
  r.routed_scale = L->cfg.routed_scale; r.shared_gated = L->cfg.shared_gated;
  r.topk_idx = L->topk_idx; r.topk_w = L->topk_w; r.sgate = L->sgate;
  KL_TRY(launch_router_select(r, st));
  return MOE_OK;
}

static moe_status ep_phase_a(moe_layer *L, const void *x, int T, cudaStream_t st) {
  CUDA_TRY(cudaMemsetAsync(L->sched, 0, 32, st));
  moe_status s = run_router_full(L, x, T, st);
  if (s != MOE_OK) return s;
  const int P = L->ep.P, Tm = std::max(1, L->max_tokens);
  KL_TRY(launch_ep_plan(L->topk_idx, T, L->k, L->E, P, L->ep.sendpos, L->ep.cnt_dev, st));
  // fixed-capacity exchange: every [P][Tm] send block travels whole, so the rows past a
  // destination's count must carry no expert ids (-1: the expert side skips them)
  if (L->ep.fixed) CUDA_TRY(cudaMemsetAsync(L->ep.send_idx, 0xff, (size_t)P * Tm * L->k * 4, st));
  if (L->fp8) {
    // quantise the own tokens once (1x128 UE8M0 + e4m3, reading R10): the dispatched rows and
    // the shared expert's input (xq) -- half the bytes of a bf16 row on the wire
    ScatterDst q{};
    q.fp8 = 1; q.xq = L->xq; q.xs = L->xs; q.xq_img = L->xq_img; q.xq_img_stride = L->img_tiles_sh;
    KL_TRY(launch_scatter_rows(x, T, L->H, 0, L->pos, q, st));
    KL_TRY(launch_ep_pack_fp8(L->xq, L->xs, T, L->H, L->k, L->topk_idx, L->topk_w, L->E, P, Tm, L->ep.row_bytes,
                              L->ep.sendpos, L->ep.send_x, L->ep.send_idx, L->ep.send_w, st));
  } else {
    KL_TRY(launch_ep_pack(x, T, L->H, L->k, L->topk_idx, L->topk_w, L->E, P, Tm, L->ep.sendpos, L->ep.send_x,
                          L->ep.send_idx, L->ep.send_w, st));
  }
  return MOE_OK;
}

// fixed-capacity exchange: source p's rows land in block [p Tm, (p+1) Tm) whatever its count
static void ep_fixed_layout(moe_layer *L) {
  const int P = L->ep.P, Tm = std::max(1, L->max_tokens);
  for (int p = 0; p <= P; ++p) L->ep.roff[p] = p * Tm;
  L->ep.R = P * Tm;
}

// send counts (cnt_dev[0:P]) and received counts (cnt_dev[P:2P]) -> host
static moe_status ep_counts_to_host(moe_layer *L, cudaStream_t st) {
  const int P = L->ep.P;
  CUDA_TRY(cudaMemcpyAsync(L->ep.cnt_host, L->ep.cnt_dev, 2 * P * 4, cudaMemcpyDeviceToHost, st));
  CUDA_TRY(cudaStreamSynchronize(st));
  int off = 0;
  for (int p = 0; p < P; ++p) {
    L->ep.roff[p] = off;
    off += L->ep.cnt_host[P + p];
  }
  L->ep.roff[P] = off;
  L->ep.R = off;
  if (off > L->max_rows) return fail(MOE_ERR_CAPACITY, "received %d rows > %d", off, L->max_rows);
  return MOE_OK;
}

static int fd_cluster_size(const moe_layer *L, int units, int k_used, int T, bool with_shared, int *ncl_out);

// Expert side at decode sizes (R received rows and T_own own tokens <= gemv_max_tokens): the
// fused decode stream instead of the prefill grouped GEMMs -- (A) the routed experts over the
// received rows (arrival order, expert ids masked to this rank) -> fp32 sums -> the bf16 partial
// rows returned to the origins; (B) the shared expert over the own tokens -> ysh (ungated: the
// origin's final combine applies the Qwen2 gate).  Two stream launches + finalizes, in order.
static moe_status ep_decode_stream(moe_layer *L, const void *x_own, int T_own, int n_def, bool want_def,
                                   cudaStream_t st) {
  const int R = L->ep.R, k = L->k, H = L->H, Fs = L->Fs;
  const bool f8 = L->fp8;
  float *acc_imm = L->dacc, *acc_def = L->dacc + (size_t)L->gemv_max_tokens * H;
  // (B may launch while A's last CTAs still run -- finalize A triggers it through PDL -- so
  // the two launches take units from separate work counters)
  auto launch = [&](FusedDecodeParams &fp, int T, int units, int k_used, bool shared, int *ctr) -> moe_status {
    fp.H = H; fp.T = T; fp.has_shared = shared; fp.has_prev = 0; fp.sgate = nullptr;
    fp.acc_imm = acc_imm; fp.acc_def = acc_def;
    fp.sched = ctr; fp.done = ctr + 1;
    fp.cl_scratch = L->cl_scratch;
    int ncl = 0;
    const int csize = fd_cluster_size(L, units, k_used, T, shared, &ncl);
    const int grid = csize > 1 ? std::min(units, ncl) * csize : std::min(L->num_sms, units);
    KL_TRY(launch_umma_decode_fused(f8, L->fp4, fp, grid, csize, st));
    return MOE_OK;
  };
  if (R > 0) {
    // (A) routed experts over the received rows
    FusedDecodeParams fp{};
    FdGroup &g = fp.g[0];
    if (f8) {
      KL_TRY(launch_ep_unpack_fp8(L->ep.recv_x, R, H, L->ep.row_bytes, L->xperm, L->xperm_s, st));
      g.x_map = L->dmap_xperm;
      g.xs = L->xperm_s;
    } else if (!make_kmajor_map(&g.x_map, L->ep.recv_x, false, (int64_t)L->ep.P * std::max(1, L->max_tokens), H, 16)) {
      return fail(MOE_ERR_CUDA, "cuTensorMapEncodeTiled failed for the received rows");
    }
    if (L->fp4) { g.w13_map4 = L->fmap_w13; g.w2_map4 = L->fmap_w2; }
    g.w13 = (const uint8_t *)L->w13; g.w13_s = L->w13_s;
    g.w2 = (const uint8_t *)L->w2; g.w2_s = L->w2_s; g.nch = L->F / 128;
    g.list = L->act_list; g.n_list = L->n_active; g.topk_idx = L->topk_idx; g.topk_w = L->topk_w;
    g.k = k; g.e0 = L->e0;
    g.a0 = 0; g.a1 = want_def ? k - n_def : k; g.a2 = k;
    fp.g[1] = fp.g[2] = g;
    const int units = (int)std::min<int64_t>(L->E, (int64_t)R * k) * (L->F / 128);
    moe_status s = launch(fp, R, units, k, false, L->sched + 5);
    if (s != MOE_OK) return s;
    DecodeFinalizeArgs fa{};
    fa.T = R; fa.H = H; fa.use_def = want_def; fa.acc_imm = acc_imm; fa.acc_def = acc_def;
    fa.y = L->ep.partial; fa.deferred_out = want_def ? L->ep.partial_def : nullptr;
    KL_TRY(launch_decode_finalize(fa, st));
  }
  if (Fs > 0 && T_own > 0) {
    // (B) the shared expert over the own tokens (FP8: xq / xs quantised in phase A)
    FusedDecodeParams fp{};
    FdGroup &g = fp.g[1];
    if (!f8) CUDA_TRY(cudaMemcpyAsync(L->xcopy, x_own, (size_t)T_own * H * 2, cudaMemcpyDeviceToDevice, st));
    g.x_map = f8 ? L->dmap_xq : L->dmap_xc;
    if (L->fp4) { g.w13_map4 = L->fmap_ws13; g.w2_map4 = L->fmap_ws2; }
    g.w13 = (const uint8_t *)L->ws13; g.w13_s = L->ws13_s; g.xs = L->xs;
    g.w2 = (const uint8_t *)L->ws2; g.w2_s = L->ws2_s; g.nch = Fs / 128;
    fp.g[0] = g;
    fp.g[0].list = L->act_list; fp.g[0].n_list = L->zero_i32;   // no routed units
    fp.g[0].nch = L->F / 128;
    fp.g[2] = fp.g[0];
    moe_status s = launch(fp, T_own, Fs / 128, 0, true, L->zero_i32 + 1);
    if (s != MOE_OK) return s;
    DecodeFinalizeArgs fa{};
    fa.T = T_own; fa.H = H; fa.use_def = 0; fa.acc_imm = acc_imm; fa.acc_def = acc_def; fa.y = L->ysh;
    KL_TRY(launch_decode_finalize(fa, st));
  }
  return MOE_OK;
}

static moe_status ep_phase_c(moe_layer *L, const void *x_own, int T_own, int n_def, bool want_def,
                             cudaStream_t st) {
  const int R = L->ep.R, k = L->k, H = L->H, Fs = L->Fs, E = L->E;
  // routing of the received rows (global ids, -1 = not ours) is in topk_idx/topk_w
  PermuteArgs pa{};
  pa.topk_idx = L->topk_idx; pa.T = R; pa.k = k; pa.E = E; pa.e0 = L->e0;
  pa.chunk_cnt = L->chunk_cnt; pa.chunk_base = L->chunk_base; pa.counts = L->counts; pa.offs = L->offs;
  pa.offs_pad = L->offs_pad; pa.tiles = L->tiles; pa.n_tiles = L->n_tiles; pa.act_list = L->act_list;
  pa.n_active = L->n_active; pa.row_token = L->row_token; pa.R_max = L->R_max; pa.pos = L->pos;
  pa.pairs = L->pairs; pa.n_pairs = L->n_pairs;
  if (R > 0) {
    KL_TRY(launch_permute(pa, st));
    L->n_launch += 2;                            // count + scan + assign kernels
  } else {
    CUDA_TRY(cudaMemsetAsync(L->n_tiles, 0, 4, st));
    CUDA_TRY(cudaMemsetAsync(L->n_pairs, 0, 4, st));
  }
  static const bool ep_gemm = getenv("MOE_EP_DECODE_GEMM") && atoi(getenv("MOE_EP_DECODE_GEMM")) == 1;  // A/B
  if (!ep_gemm && L->fused_decode && L->umma && R <= L->gemv_max_tokens && T_own <= L->gemv_max_tokens)
    return ep_decode_stream(L, x_own, T_own, n_def, want_def, st);
  if (L->fp8) {
    // received e4m3 rows + exponents -> the expert-sorted rows and their scale images (the
    // own tokens' xq for the shared expert was quantised in phase A)
    KL_TRY(launch_ep_scatter_fp8(L->ep.recv_x, R, H, k, L->ep.row_bytes, L->pos, L->xperm, L->xperm_img,
                                 L->max_tiles, st));
  } else {
    ScatterDst d{};
    d.fp8 = 0; d.xperm = L->xperm;
    KL_TRY(launch_scatter_rows(L->ep.recv_x, R, H, k, L->pos, d, st));
  }
  const int64_t pairs = (int64_t)R * k;
  const int64_t R_bound = std::min<int64_t>(L->R_max, pairs + (int64_t)std::min<int64_t>(E, pairs) * kPadM);
  moe_status gs = run_expert_gemms(L, (int)(R_bound / kPadM), x_own, Fs > 0 ? T_own : 0, st);
  if (gs != MOE_OK) return gs;
  if (R > 0) {
    CombineArgs c{};
    c.T = R; c.H = H; c.k = k; c.n_imm = want_def ? k - n_def : k;
    c.pos = L->pos; c.topk_w = L->topk_w; c.yperm = L->yperm;
    c.y = L->ep.partial; c.deferred_out = want_def ? L->ep.partial_def : nullptr;
    KL_TRY(launch_combine(c, st));
  }
  return MOE_OK;
}

static moe_status ep_phase_d(moe_layer *L, const void *residual, int T, const void *din, void *y, void *dout,
                             cudaStream_t st) {
  EpCombineArgs c{};
  c.T = T; c.H = L->H; c.P = L->ep.P; c.Tm = std::max(1, L->max_tokens);
  c.sendpos = L->ep.sendpos; c.back = L->ep.back; c.back_def = dout ? L->ep.back_def : nullptr;
  c.ysh = L->Fs > 0 ? L->ysh : nullptr; c.sgate = L->cfg.shared_gated ? L->sgate : nullptr;
  c.residual = reinterpret_cast<const __nv_bfloat16 *>(residual);
  c.deferred_in = reinterpret_cast<const __nv_bfloat16 *>(din);
  c.y = reinterpret_cast<__nv_bfloat16 *>(y); c.deferred_out = reinterpret_cast<__nv_bfloat16 *>(dout);
  KL_TRY(launch_ep_final_combine(c, st));
  return MOE_OK;
}

#define NCCL_TRY(expr)                                                                                 \
  do {                                                                                                 \
    if ((expr) != 0) return fail(MOE_ERR_NCCL, "%s failed %s", #expr, ep_nccl_error(L->ep.comm));    \
  } while (0)

// one rank of an NCCL expert-parallel group (collective over the group)
static moe_status ep_forward_nccl(moe_layer *L, const void *x, const void *residual, int T, int n_def,
                                  const void *din, void *y, void *dout, cudaStream_t st) {
  const int P = L->ep.P, k = L->k, H = L->H;
  const int64_t Tm = std::max(1, L->max_tokens);
  moe_status s = ep_phase_a(L, x, T, st);
  if (s != MOE_OK) return s;
  int32_t full_cnt[32];
  const int32_t *scnt = L->ep.cnt_host, *rcnt = L->ep.cnt_host + P;
  if (L->ep.fixed) {
    // no host synchronisation (CUDA-Graph capturable): whole Tm-row blocks both ways
    ep_fixed_layout(L);
    for (int p = 0; p < P; ++p) full_cnt[p] = (int32_t)Tm;
    scnt = rcnt = full_cnt;
  } else {
    NCCL_TRY(ep_nccl_counts(L->ep.comm, L->ep.cnt_dev, L->ep.cnt_dev + P, P, st));
    if ((s = ep_counts_to_host(L, st)) != MOE_OK) return s;
  }
  int64_t soff[32], roff[32];
  for (int p = 0; p < P; ++p) { soff[p] = p * Tm; roff[p] = L->ep.roff[p]; }
  {
    const void *snd[3] = {L->ep.send_x, L->ep.send_idx, L->ep.send_w};
    void *rcv[3] = {L->ep.recv_x, L->topk_idx, L->topk_w};
    const int64_t rb[3] = {(int64_t)L->ep.row_bytes, (int64_t)k * 4, (int64_t)k * 4};
    NCCL_TRY(ep_nccl_rows(L->ep.comm, P, scnt, soff, rcnt, roff, 3, snd, rcv, rb, st));
  }
  const bool want_def = dout != nullptr && n_def > 0;
  if ((s = ep_phase_c(L, x, T, n_def, want_def, st)) != MOE_OK) return s;
  {
    const void *snd[2] = {L->ep.partial, L->ep.partial_def};
    void *rcv[2] = {L->ep.back, L->ep.back_def};
    const int64_t rb[2] = {(int64_t)H * 2, (int64_t)H * 2};
    NCCL_TRY(ep_nccl_rows(L->ep.comm, P, rcnt, roff, scnt, soff, want_def ? 2 : 1, snd, rcv, rb, st));
  }
  return ep_phase_d(L, residual, T, din, y, want_def ? dout : nullptr, st);
}

// Cluster size of the fused decode stream for `units` queued units (k_used slots per token of T
// tokens routed here, with / without the shared expert's units after the router).
static int fd_cluster_size(const moe_layer *L, int units, int k_used, int T, bool with_shared, int *ncl_out) {
  const int H = L->H, E = L->E;
  const bool f8 = L->fp8;
  // Cluster split: each unit over C = 1/2/4/8 CTAs (C <= the W13 k-blocks and W2 tiles).
  // (1) Few units (expert TP, small layers): the largest C whose clusters all fit in one wave.
  // (2) Otherwise C = 2 when a cost model of the part after the router says so -- this
  //     layer's routed + shared units (a chained layer's group-2 units run beside the router):
  //     rounds x (unit time / C + split overhead), rounds = ceil(units / resident clusters),
  //     unit time = its weight bytes at ~56 GB/s per SM, overhead 1.5 us, and >= 2 % cheaper
  //     than C = 1.  Routed units use the expected number of distinct experts of T tokens.
  //     (Fitted to profiles/r02/decode_csize.txt: C = 2 wins when the post-router units fit
  //     one round of pairs -- V2-Lite / V2.5 chained deferral -- or leave a ragged third round
  //     at C = 1 -- Qwen2, 320 units; C = 4 / 8 beyond one wave lost everywhere.)
  // Clusters take units from the device queue.  MOE_FD_CSIZE forces C (A/B experiments).
  static const int force_c = getenv("MOE_FD_CSIZE") ? atoi(getenv("MOE_FD_CSIZE")) : 0;
  const int KA = H / (f8 ? 128 : 64), NT = H / 256;
  auto c_ok = [&](int c) { return c == 1 || (c <= KA && c <= NT && L->fd_max_clusters[c] >= 1); };
  auto n_cl = [&](int c) { return c == 1 ? L->num_sms : L->fd_max_clusters[c]; };
  int csize = 1;
  for (int c = 8; c >= 2; c /= 2)
    if (c_ok(c) && units <= n_cl(c) && units * c <= L->num_sms) { csize = c; break; }
  if (csize == 1 && c_ok(2)) {
    const double wb = L->fp4 ? 0.5 : (f8 ? 1.0 : 2.0);
    const double unit_us = (256.0 * H + 128.0 * H) * wb / 56e3;
    const int k_now = k_used;
    const double e_exp = T <= 1 ? (double)k_now
                                : std::min((double)E, std::ceil(E * (1.0 - std::pow(1.0 - (double)k_now / E, T))));
    const int post = (with_shared ? L->Fs / 128 : 0) + (int)e_exp * (L->F / 128);
    const double c1 = (double)((post + n_cl(1) - 1) / n_cl(1)) * unit_us;
    const double c2 = (double)((post + n_cl(2) - 1) / n_cl(2)) * (unit_us / 2 + 1.5);
    if (c2 < 0.98 * c1) csize = 2;
  }
  if (force_c == 1 || ((force_c == 2 || force_c == 4 || force_c == 8) && c_ok(force_c))) csize = force_c;
  *ncl_out = n_cl(csize);
  return csize;
}

// One forward.  Modes: plain / split deferral (moe_layer_forward[_deferred]:
// deferred slots -> deferred_out) and chained deferral (moe_layer_forward_chained:
// deferred slots left for the next layer, `prev`'s deferred slots computed here).
// skip_finalize: leave the fp32 partial sums in L->dacc (in-process TP group).
struct FwdArgs {
  const void *x, *residual;
  int32_t T, n_def;
  const void *deferred_in;
  void *y, *deferred_out;
  moe_routing_out *dbg;
  bool chained;
  moe_layer *prev;
  bool skip_finalize;
};

static moe_status forward_impl(moe_layer *L, const FwdArgs &A, void *stream) {
  if (!L) return fail(MOE_ERR_INVALID_ARG, "null layer");
  const void *x = A.x, *residual = A.residual, *deferred_in = A.deferred_in;
  void *y = A.y, *deferred_out = A.deferred_out;
  const int32_t T = A.T, n_def = A.n_def;
  moe_routing_out *dbg = A.dbg;
  NvtxRange nvtx(T <= L->gemv_max_tokens ? "moe_layer_forward/decode" : "moe_layer_forward/prefill");
  if (T < 0) return fail(MOE_ERR_INVALID_ARG, "T = %d < 0", T);
  if (T > L->max_tokens) return fail(MOE_ERR_CAPACITY, "T = %d > max_tokens = %d", T, L->max_tokens);
  if (n_def < 0 || n_def > L->k - 1) return fail(MOE_ERR_INVALID_ARG, "n_deferred = %d not in [0, k-1]", n_def);
  if (T > 0 && (!x || !y)) return fail(MOE_ERR_INVALID_ARG, "x and y must be non-null");
  if (x && x == y) return fail(MOE_ERR_INVALID_ARG, "y must not alias x");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  moe_layer *prev = A.prev;
  if (A.chained) {
    if (L->ep.P > 1 || L->ep.comm) return fail(MOE_ERR_UNSUPPORTED, "chained deferral on an expert-parallel layer");
    if (!(L->fused_decode && T >= 1 && T <= L->gemv_max_tokens && L->E_glob <= 256))
      return fail(MOE_ERR_UNSUPPORTED, "chained deferral runs on the decode stream: T = %d must be in [1, %d]", T,
                  L->gemv_max_tokens);
    if (prev) {
      if (prev == L) return fail(MOE_ERR_INVALID_ARG, "prev is this layer");
      if (prev->H != L->H || prev->fp8 != L->fp8 || prev->fp4 != L->fp4 || prev->cfg.device != L->cfg.device ||
          prev->tp_size != L->tp_size || prev->tp_rank != L->tp_rank || !prev->fused_decode || prev->ep.P > 1)
        return fail(MOE_ERR_INVALID_ARG, "prev has another shape / dtype / device / TP split");
      if (prev->chain_T != T || prev->chain_ndef <= 0)
        return fail(MOE_ERR_INVALID_ARG, "prev's last call was not a chained forward with n_deferred > 0 on %d tokens", T);
    }
  } else if (prev) {
    return fail(MOE_ERR_INVALID_ARG, "prev is for chained forwards only");
  }
  if (L->tp_size > 1 && !L->tp_comm && !A.skip_finalize)
    return fail(MOE_ERR_INVALID_ARG, "layer is a rank of an in-process TP group: use moe_tp_group_forward");
  if (L->ep.P > 1 || L->ep.comm) {
    if (!L->ep.comm)
      return fail(MOE_ERR_INVALID_ARG, "layer belongs to an in-process EP group: use moe_ep_group_forward");
    if (dbg) return fail(MOE_ERR_UNSUPPORTED, "routing debug outputs are single-GPU only");
    return ep_forward_nccl(L, x, residual, T, n_def, deferred_in, y, deferred_out, st);  // T == 0 participates
  }
  if (T == 0) return MOE_OK;
  L->n_launch = 0;
  if (L->prof) {
    for (int i = 0; i <= moe_layer::kStages; ++i) L->ev_hit[i] = false;
    cudaEventRecord(L->ev[0], st);
    L->ev_hit[0] = true;
  }
  const int H = L->H, F = L->F, Fs = L->Fs, E = L->E, k = L->k;
  const bool decode = L->gemv_ok && T <= L->gemv_max_tokens;
  const bool tc_decode = decode && L->umma && L->E_glob <= 256 && L->E <= 256;  // T <= 16: small-T route + swap-AB kernels
  const bool fused = tc_decode && L->fused_decode;  // route -> fused W13/W2 stream -> finalize (self-re-arming counters)
  if (L->tp_size > 1 && !fused)
    return fail(MOE_ERR_UNSUPPORTED, "expert TP (tp_size = %d) needs the fused decode stream: T = %d must be <= %d",
                L->tp_size, T, L->gemv_max_tokens);
  if (!fused) CUDA_TRY(cudaMemsetAsync(L->sched, 0, 32, st));
  RouterArgs r{};
  r.logits = L->logits; r.ldl = L->gate_rows; r.bias = L->gate_bias;
  r.T = T; r.E = L->E_glob; r.k = k; r.n_group = L->cfg.n_group; r.topk_group = L->cfg.topk_group;
  r.group_score = L->cfg.group_score; r.score_fn = L->cfg.score_fn; r.norm_topk = L->cfg.norm_topk;
  r.routed_scale = L->cfg.routed_scale; r.shared_gated = L->cfg.shared_gated;
  r.topk_idx = L->topk_idx; r.topk_w = L->topk_w; r.sgate = L->sgate;
  PermuteArgs pa{};
  pa.topk_idx = L->topk_idx; pa.T = T; pa.k = k; pa.E = E; pa.e0 = L->e0;
  pa.chunk_cnt = L->chunk_cnt; pa.chunk_base = L->chunk_base; pa.counts = L->counts; pa.offs = L->offs;
  pa.offs_pad = L->offs_pad; pa.tiles = L->tiles; pa.n_tiles = L->n_tiles; pa.act_list = L->act_list;
  pa.n_active = L->n_active; pa.row_token = L->row_token; pa.R_max = L->R_max; pa.pos = L->pos;
  pa.pairs = L->pairs; pa.n_pairs = L->n_pairs;
  pa.dbg_perm = dbg ? dbg->perm : nullptr;
  pa.dbg_counts = dbg ? dbg->expert_counts : nullptr;
  if (tc_decode) {
    // 1-3 (decode). logits + select + count/scan/assign in one launch
    RouteSmallArgs rs{};
    rs.r = r; rs.p = pa; rs.x = x; rs.wg = L->gate_w; rs.H = H; rs.rows = L->gate_rows; rs.done = L->sched + 7;
    static const int dbg_route = experiment_knob("MOE_DEBUG_ROUTE");   // timing experiments (MOE_EXPERIMENTS builds)
    rs.debug = dbg_route;
    rs.trace = L->trace;
    rs.fp8 = L->fp8;
    if (L->fp8) { rs.xq = L->xq; rs.xs = L->xs; }
    else rs.xcopy = L->xcopy;
    rs.n_imm = A.chained ? k - n_def : k;
    static const int early_knob = experiment_knob("MOE_ROUTE_EARLY");   // A/B (MOE_EXPERIMENTS builds)
    rs.early_trigger = prev != nullptr || early_knob == 1;
    rs.imm_list = L->imm_list; rs.def_list = L->def_list; rs.n_imm_list = L->n_lists; rs.n_def_list = L->n_lists + 1;
    KL_TRY(launch_route_small(rs, st));
    mark(L, ST_PERMUTE, st);
  } else {
    // 1. router logits (bf16 x . bf16 Wg, fp32 accumulate; reading R9)
    if (T <= kGemvMaxTokens) {
      KL_TRY(launch_router_gemv(x, T, H, L->gate_w, L->gate_rows, L->logits, st));
    } else {
      moe_status s = launch_logits(L, x, T, st);
      if (s != MOE_OK) return s;
    }
    mark(L, ST_LOGITS, st);
    // 2. scores + group-limited top-k + weights
    KL_TRY(launch_router_select(r, st));
    mark(L, ST_SELECT, st);
    // 3. count / scan / permute
    KL_TRY(launch_permute(pa, st));
    L->n_launch += 2;                            // count + scan + assign kernels
    mark(L, ST_PERMUTE, st);
  }
  const int64_t pairs = (int64_t)T * k;
  const int64_t R_bound = std::min<int64_t>(L->R_max, pairs + (int64_t)std::min<int64_t>(E, pairs) * kPadM);
  const int tile_bound = (int)(R_bound / kPadM);
  // 4. activation quantisation (FP8) and gather into expert order
  if (!tc_decode) {
    // each token's row -> its k sorted rows (+ xq): FP8 quantisation fused with the gather
    ScatterDst d{};
    d.fp8 = L->fp8; d.xperm = L->xperm;
    if (L->fp8) {
      d.xperm_img = L->umma ? L->xperm_img : nullptr; d.xperm_img_stride = L->max_tiles;
      d.xperm_s = L->umma ? nullptr : L->xperm_s;
      d.xq = L->xq; d.xs = L->xs; d.xq_img = L->umma ? L->xq_img : nullptr; d.xq_img_stride = L->img_tiles_sh;
    }
    KL_TRY(launch_scatter_rows(x, T, H, k, L->pos, d, st));
    mark(L, ST_GATHER, st);
  }
  if (fused) {
    // 5+6+7 (decode). one weight stream per (expert, 128-column chunk): W13 -> SwiGLU -> h in smem ->
    // W2 -> weighted fp32 sums (umma_decode_fused.cu), then residual / deferral / bf16 in finalize
    const bool f8 = L->fp8;
    FusedDecodeParams fp{};
    auto routed = [&](FdGroup &g, const moe_layer *S, const int32_t *list, const int32_t *n_list, int a0, int a1,
                      int a2) {
      g.x_map = S->fp8 ? S->dmap_xq : S->dmap_xc;
      if (S->fp4) { g.w13_map4 = S->fmap_w13; g.w2_map4 = S->fmap_w2; }
      g.w13 = (const uint8_t *)S->w13; g.w13_s = S->w13_s; g.xs = S->xs;
      g.w2 = (const uint8_t *)S->w2; g.w2_s = S->w2_s; g.nch = S->F / 128;
      g.list = list; g.n_list = n_list; g.topk_idx = S->topk_idx; g.topk_w = S->topk_w; g.k = S->k; g.e0 = S->e0;
      g.a0 = a0; g.a1 = a1; g.a2 = a2;
    };
    const bool want_def = !A.chained && deferred_out != nullptr && n_def > 0;
    if (A.chained && n_def > 0)      // this layer's deferred slots are the next layer's work (Eq. L241)
      routed(fp.g[0], L, L->imm_list, L->n_lists, 0, k - n_def, k - n_def);
    else                             // split deferral: [k - n_def, k) -> deferred_out
      routed(fp.g[0], L, L->act_list, L->n_active, 0, want_def ? k - n_def : k, k);
    if (Fs > 0) {
      FdGroup &g = fp.g[1];
      g.x_map = f8 ? L->dmap_xq : L->dmap_xc;
      if (L->fp4) { g.w13_map4 = L->fmap_ws13; g.w2_map4 = L->fmap_ws2; }
      g.w13 = (const uint8_t *)L->ws13; g.w13_s = L->ws13_s; g.xs = L->xs;
      g.w2 = (const uint8_t *)L->ws2; g.w2_s = L->ws2_s; g.nch = Fs / 128;
    } else {
      fp.g[1] = fp.g[0];
    }
    int prev_units = 0;
    if (prev) {                      // R^def_{k-1}(I_{k-1}) joins this layer's output (acc_imm)
      routed(fp.g[2], prev, prev->def_list, prev->n_lists + 1, prev->k - prev->chain_ndef, prev->k, prev->k);
      prev_units = (int)std::min<int64_t>(prev->E, (int64_t)T * prev->chain_ndef) * (prev->F / 128);
      prev->chain_T = -1;            // consumed
    } else {
      fp.g[2] = fp.g[0];
    }
    fp.H = H; fp.T = T; fp.has_shared = Fs > 0; fp.has_prev = prev != nullptr;
    fp.sgate = L->cfg.shared_gated ? L->sgate : nullptr;
    float *acc_imm = L->dacc, *acc_def = L->dacc + (size_t)L->gemv_max_tokens * H;
    fp.acc_imm = acc_imm; fp.acc_def = acc_def;
    fp.sched = L->sched + 5; fp.done = L->sched + 6;
    fp.trace = L->trace;
    static const int dbg_fd = experiment_knob("MOE_DEBUG_FD");   // timing experiments (MOE_EXPERIMENTS builds)
    fp.debug = dbg_fd;
    const int units = prev_units + Fs / 128 + (int)std::min<int64_t>(E, pairs) * (F / 128);
    int ncl = 0;
    const int csize = fd_cluster_size(L, units, (A.chained && n_def > 0) ? k - n_def : k, T, Fs > 0, &ncl);
    fp.cl_scratch = L->cl_scratch;
    const int grid = csize > 1 ? std::min(units, ncl) * csize : std::min(L->num_sms, units);
    KL_TRY(launch_umma_decode_fused(f8, L->fp4, fp, grid, csize, st));
    mark(L, ST_GEMM1, st);
    if (A.chained) { L->chain_T = n_def > 0 ? T : -1; L->chain_ndef = n_def; }
    else L->chain_T = -1;
    if (L->tp_size > 1 && L->tp_comm) {
      // TP: sum the P ranks' fp32 partials (immediate and deferred sums) -- PAPER.md L197
      if (ep_nccl_allreduce_f32(L->tp_comm, acc_imm, (size_t)T * H, st) != 0 ||
          (want_def && ep_nccl_allreduce_f32(L->tp_comm, acc_def, (size_t)T * H, st) != 0))
        return fail(MOE_ERR_NCCL, "ncclAllReduce of the TP partials failed %s", ep_nccl_error(L->tp_comm));
    }
    if (A.skip_finalize) {
      L->pending_use_def = want_def;
      (decode ? L->launches_decode : L->launches_prefill) = L->n_launch;
      return MOE_OK;
    }
    DecodeFinalizeArgs fa{};
    fa.T = T; fa.H = H; fa.use_def = want_def;
    fa.acc_imm = acc_imm; fa.acc_def = acc_def;
    fa.residual = residual; fa.deferred_in = A.chained ? nullptr : deferred_in; fa.y = y;
    fa.deferred_out = A.chained ? nullptr : deferred_out;
    fa.trace = L->trace;
    KL_TRY(launch_decode_finalize(fa, st));
    mark(L, ST_COMBINE, st);
  } else if (decode) {
    // 5+6 (decode, CUDA-core path). weight-streaming GEMVs over the active experts + shared expert
    GemvArgs g{};
    g.T = T; g.H = H; g.F = F; g.Fs = Fs; g.fp8 = L->fp8; g.has_shared = Fs > 0;
    g.act_list = L->act_list; g.n_active = L->n_active; g.counts = L->counts; g.offs_pad = L->offs_pad;
    g.row_token = L->row_token; g.x = x; g.xq = L->xq; g.xs = L->xs;
    g.w13 = L->w13; g.w2 = L->w2; g.ws13 = L->ws13; g.ws2 = L->ws2;
    g.w13_s = L->w13_s; g.w2_s = L->w2_s; g.ws13_s = L->ws13_s; g.ws2_s = L->ws2_s;
    g.h = L->hbuf; g.hsh = L->hsh; g.h_s = L->h_s; g.hsh_s = L->hsh_s; g.yperm = L->yperm; g.ysh = L->ysh;
    const int slots = (int)std::min<int64_t>(E, pairs) + (Fs > 0 ? 1 : 0);
    KL_TRY(launch_gemv(g, 1, slots, st));
    mark(L, ST_GEMM1, st);
    KL_TRY(launch_gemv(g, 2, slots, st));
    mark(L, ST_GEMM2, st);
  } else {
    // 5+6. routed experts (sorted rows) + shared expert (all T tokens)
    moe_status gs = run_expert_gemms(L, tile_bound, x, Fs > 0 ? T : 0, st);
    if (gs != MOE_OK) return gs;
  }
  // 7. weighted combine + residual (+ deferral split)
  if (!fused) {
    CombineArgs c{};
    c.T = T; c.H = H; c.k = k; c.n_imm = deferred_out ? k - n_def : k;
    c.pos = L->pos; c.topk_w = L->topk_w; c.yperm = L->yperm;
    c.ysh = Fs > 0 ? L->ysh : nullptr; c.sgate = L->cfg.shared_gated ? L->sgate : nullptr;
    c.residual = residual; c.deferred_in = deferred_in; c.y = y; c.deferred_out = deferred_out;
    KL_TRY(launch_combine(c, st));
    mark(L, ST_COMBINE, st);
  }
  (decode ? L->launches_decode : L->launches_prefill) = L->n_launch;
  if (dbg) {
    if (dbg->topk_idx)
      CUDA_TRY(cudaMemcpyAsync(dbg->topk_idx, L->topk_idx, pairs * 4, cudaMemcpyDeviceToDevice, st));
    if (dbg->topk_w) CUDA_TRY(cudaMemcpyAsync(dbg->topk_w, L->topk_w, pairs * 4, cudaMemcpyDeviceToDevice, st));
  }
  return MOE_OK;
}

moe_status moe_layer_forward(moe_layer *L, const void *x, const void *residual, int32_t T, void *y,
                             moe_routing_out *dbg, void *stream) {
  FwdArgs a{x, residual, T, 0, nullptr, y, nullptr, dbg, false, nullptr, false};
  return forward_impl(L, a, stream);
}

moe_status moe_layer_forward_deferred(moe_layer *L, const void *x, const void *residual, int32_t T,
                                      int32_t n_deferred, const void *deferred_in, void *y, void *deferred_out,
                                      moe_routing_out *dbg, void *stream) {
  FwdArgs a{x, residual, T, n_deferred, deferred_in, y, deferred_out, dbg, false, nullptr, false};
  return forward_impl(L, a, stream);
}

moe_status moe_layer_forward_chained(moe_layer *L, const void *x, const void *residual, int32_t T,
                                     int32_t n_deferred, moe_layer *prev, void *y, void *stream) {
  FwdArgs a{x, residual, T, n_deferred, nullptr, y, nullptr, nullptr, true, prev, false};
  return forward_impl(L, a, stream);
}

moe_status moe_ep_group_forward(moe_layer *const *layers, int32_t P, const void *const *x,
                                const void *const *residual, const int32_t *T, int32_t n_deferred,
                                const void *const *deferred_in, void *const *y, void *const *deferred_out,
                                void *stream) {
  if (!layers || !x || !y || !T || P < 2 || P > 32) return fail(MOE_ERR_INVALID_ARG, "bad group arguments");
  NvtxRange nvtx("moe_ep_group_forward");
  for (int r = 0; r < P; ++r) {
    moe_layer *L = layers[r];
    if (!L || L->ep.P != P || L->ep.rank != r || L->ep.comm)
      return fail(MOE_ERR_INVALID_ARG, "layer %d is not rank %d of an in-process group of %d", r, r, P);
    if (T[r] < 0 || T[r] > L->max_tokens) return fail(MOE_ERR_CAPACITY, "T[%d] = %d", r, T[r]);
    if (n_deferred < 0 || n_deferred > L->k - 1) return fail(MOE_ERR_INVALID_ARG, "n_deferred");
    if (T[r] > 0 && (!x[r] || !y[r])) return fail(MOE_ERR_INVALID_ARG, "x/y of rank %d", r);
  }
  for (int r = 1; r < P; ++r)
    if (layers[r]->cfg.device != layers[0]->cfg.device)
      return fail(MOE_ERR_UNSUPPORTED, "in-process EP group: all ranks on one device (the stream's)");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  const int64_t Tm = std::max(1, layers[0]->max_tokens);
  const int H = layers[0]->H, k = layers[0]->k;
  int caller_dev = 0;
  CUDA_TRY(cudaGetDevice(&caller_dev));
  struct Restore { int d; ~Restore() { cudaSetDevice(d); } } restore{caller_dev};
  CUDA_TRY(cudaSetDevice(layers[0]->cfg.device));
  moe_status s;
  for (int r = 0; r < P; ++r)
    if ((s = ep_phase_a(layers[r], x[r], T[r], st)) != MOE_OK) return s;
  // counts: rank d receives cnt_dev[d] of every source
  const bool fixed = layers[0]->ep.fixed;
  for (int r = 1; r < P; ++r)
    if (layers[r]->ep.fixed != fixed) return fail(MOE_ERR_INVALID_ARG, "ep_fixed_capacity differs across the group");
  // rows sent from src to d: the exact count (host-synchronised) or the whole Tm block (fixed)
  auto nrows = [&](int src, int d) -> int64_t { return fixed ? Tm : layers[src]->ep.cnt_host[d]; };
  if (fixed) {
    for (int r = 0; r < P; ++r) ep_fixed_layout(layers[r]);
  } else {
    for (int d = 0; d < P; ++d)
      for (int src = 0; src < P; ++src)
        CUDA_TRY(cudaMemcpyAsync(layers[d]->ep.cnt_dev + P + src, layers[src]->ep.cnt_dev + d, 4, cudaMemcpyDefault, st));
    for (int r = 0; r < P; ++r)
      if ((s = ep_counts_to_host(layers[r], st)) != MOE_OK) return s;
  }
  for (int d = 0; d < P; ++d)
    for (int src = 0; src < P; ++src) {
      const int64_t n = nrows(src, d);
      if (!n) continue;
      const int64_t ro = layers[d]->ep.roff[src], so = (int64_t)d * Tm;
      const int64_t rbytes = layers[d]->ep.row_bytes;
      CUDA_TRY(cudaMemcpyAsync(layers[d]->ep.recv_x + ro * rbytes, layers[src]->ep.send_x + so * rbytes, n * rbytes,
                               cudaMemcpyDefault, st));
      CUDA_TRY(cudaMemcpyAsync(layers[d]->topk_idx + ro * k, layers[src]->ep.send_idx + so * k, n * k * 4,
                               cudaMemcpyDefault, st));
      CUDA_TRY(cudaMemcpyAsync(layers[d]->topk_w + ro * k, layers[src]->ep.send_w + so * k, n * k * 4,
                               cudaMemcpyDefault, st));
    }
  for (int r = 0; r < P; ++r) {
    const bool want_def = deferred_out && deferred_out[r] && n_deferred > 0;
    if ((s = ep_phase_c(layers[r], x[r], T[r], n_deferred, want_def, st)) != MOE_OK) return s;
  }
  for (int src = 0; src < P; ++src)       // partial rows back to their origin
    for (int d = 0; d < P; ++d) {
      const int64_t n = nrows(src, d);
      if (!n) continue;
      const int64_t ro = layers[d]->ep.roff[src], so = (int64_t)d * Tm;
      CUDA_TRY(cudaMemcpyAsync(layers[src]->ep.back + so * H, layers[d]->ep.partial + ro * H, n * H * 2,
                               cudaMemcpyDefault, st));
      if (deferred_out && deferred_out[src] && n_deferred > 0)
        CUDA_TRY(cudaMemcpyAsync(layers[src]->ep.back_def + so * H, layers[d]->ep.partial_def + ro * H, n * H * 2,
                                 cudaMemcpyDefault, st));
    }
  for (int r = 0; r < P; ++r) {
    const bool want_def = deferred_out && deferred_out[r] && n_deferred > 0;
    if ((s = ep_phase_d(layers[r], residual ? residual[r] : nullptr, T[r],
                        deferred_in ? deferred_in[r] : nullptr, y[r], want_def ? deferred_out[r] : nullptr, st)) != MOE_OK)
      return s;
  }
  return MOE_OK;
}

moe_status moe_tp_group_forward(moe_layer *const *layers, int32_t P, const void *const *x,
                                const void *const *residual, int32_t T, int32_t n_deferred,
                                const void *const *deferred_in, void *const *y, void *const *deferred_out,
                                void *stream) {
  if (!layers || !x || !y || P < 2 || P > 32) return fail(MOE_ERR_INVALID_ARG, "bad group arguments");
  NvtxRange nvtx("moe_tp_group_forward");
  const int dev = layers[0] ? layers[0]->cfg.device : 0;
  for (int r = 0; r < P; ++r) {
    const moe_layer *L = layers[r];
    if (!L || L->tp_size != P || L->tp_rank != r || L->tp_comm)
      return fail(MOE_ERR_INVALID_ARG, "layer %d is not rank %d of an in-process TP group of %d", r, r, P);
    if (L->cfg.device != dev) return fail(MOE_ERR_UNSUPPORTED, "in-process TP group: all ranks on one device");
    if (!x[r] || !y[r]) return fail(MOE_ERR_INVALID_ARG, "x/y of rank %d", r);
  }
  if (T <= 0) return T == 0 ? MOE_OK : fail(MOE_ERR_INVALID_ARG, "T = %d", T);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  int caller_dev = 0;
  CUDA_TRY(cudaGetDevice(&caller_dev));
  CUDA_TRY(cudaSetDevice(dev));
  moe_status s = MOE_OK;
  for (int r = 0; r < P && s == MOE_OK; ++r) {
    const bool want_def = deferred_out && deferred_out[r] && n_deferred > 0;
    FwdArgs a{x[r], nullptr, T, n_deferred, nullptr, y[r], want_def ? deferred_out[r] : nullptr, nullptr, false,
              nullptr, true};
    s = forward_impl(layers[r], a, stream);
  }
  if (s == MOE_OK) {
    // the all-reduce of the fp32 partials, on one device: sum into rank 0, copy back
    const int H = layers[0]->H;
    const bool use_def = layers[0]->pending_use_def;
    const float *src[32];
    for (int part = 0; part < (use_def ? 2 : 1) && s == MOE_OK; ++part) {
      const size_t off = part ? (size_t)layers[0]->gemv_max_tokens * H : 0;
      for (int r = 0; r < P; ++r) src[r] = layers[r]->dacc + (part ? (size_t)layers[r]->gemv_max_tokens * H : 0);
      cudaError_t e = launch_sum_f32(layers[0]->dacc + off, src + 1, P - 1, (int64_t)T * H, st);
      for (int r = 1; r < P && e == cudaSuccess; ++r)
        e = cudaMemcpyAsync(layers[r]->dacc + (part ? (size_t)layers[r]->gemv_max_tokens * H : 0),
                            layers[0]->dacc + off, (size_t)T * H * 4, cudaMemcpyDeviceToDevice, st);
      if (e != cudaSuccess) s = fail(MOE_ERR_CUDA, "TP group reduce: %s", cudaGetErrorString(e));
    }
    for (int r = 0; r < P && s == MOE_OK; ++r) {
      moe_layer *L = layers[r];
      DecodeFinalizeArgs fa{};
      fa.T = T; fa.H = H; fa.use_def = use_def;
      fa.acc_imm = L->dacc; fa.acc_def = L->dacc + (size_t)L->gemv_max_tokens * H;
      fa.residual = residual ? residual[r] : nullptr;
      fa.deferred_in = deferred_in ? deferred_in[r] : nullptr;
      fa.y = y[r];
      fa.deferred_out = deferred_out ? deferred_out[r] : nullptr;
      cudaError_t e = launch_decode_finalize(fa, st);
      if (e != cudaSuccess) s = fail(MOE_ERR_CUDA, "finalize: %s", cudaGetErrorString(e));
    }
  }
  cudaSetDevice(caller_dev);
  return s;
}

moe_status moe_layer_profile(moe_layer *L, int32_t enable) {
  if (!L) return fail(MOE_ERR_INVALID_ARG, "null layer");
  if (enable && !L->ev[0]) {
    for (int i = 0; i <= moe_layer::kStages; ++i) CUDA_TRY(cudaEventCreate(&L->ev[i]));
  }
  L->prof = enable != 0;
  return MOE_OK;
}

moe_status moe_layer_stage_times(moe_layer *L, float *ms_out, int32_t cap, int32_t *n_out) {
  if (!L || !ms_out) return fail(MOE_ERR_INVALID_ARG, "null argument");
  if (!L->ev[0] || !L->ev_hit[0]) return fail(MOE_ERR_INVALID_ARG, "no profiled forward recorded");
  int last = 0;
  for (int i = 1; i <= moe_layer::kStages; ++i)
    if (L->ev_hit[i]) last = i;
  CUDA_TRY(cudaEventSynchronize(L->ev[last]));
  const int n = std::min<int>(cap, moe_layer::kStages);
  int prev = 0;
  for (int i = 0; i < n; ++i) {
    ms_out[i] = 0.f;
    if (L->ev_hit[i + 1]) {
      CUDA_TRY(cudaEventElapsedTime(&ms_out[i], L->ev[prev], L->ev[i + 1]));
      prev = i + 1;
    }
  }
  if (n_out) *n_out = n;
  return MOE_OK;
}

const char *moe_stage_name(int32_t i) {
  return (i >= 0 && i < moe_layer::kStages) ? kStageNames[i] : "";
}

// timing experiments (MOE_DEBUG_TRACE): copy the device timeline buffer (4096 u64) to the host
moe_status moe_layer_debug_trace(moe_layer *L, void *host, int32_t cap) {
  if (!L || !host) return fail(MOE_ERR_INVALID_ARG, "null argument");
  if (!L->trace) return fail(MOE_ERR_UNSUPPORTED, "layer created without MOE_DEBUG_TRACE");
  CUDA_TRY(cudaDeviceSynchronize());
  CUDA_TRY(cudaMemcpy(host, L->trace, (size_t)std::min(cap, 4096) * 8, cudaMemcpyDeviceToHost));
  CUDA_TRY(cudaMemset(L->trace, 0, 4096 * 8));
  return MOE_OK;
}

moe_status moe_layer_destroy(moe_layer *L) {
  if (!L) return MOE_OK;
  cudaSetDevice(L->cfg.device);
  for (int i = 0; i <= moe_layer::kStages; ++i)
    if (L->ev[i]) cudaEventDestroy(L->ev[i]);
  free_all(L);
  delete L;
  return MOE_OK;
}

moe_status moe_layer_get_info(const moe_layer *L, moe_layer_info *info) {
  if (!L || !info) return fail(MOE_ERR_INVALID_ARG, "null argument");
  info->weight_bytes = L->weight_bytes;
  info->workspace_bytes = L->workspace_bytes;
  info->gemv_max_tokens = L->gemv_max_tokens;
  info->kernels_per_forward_prefill = L->launches_prefill;   // counted by the last forward of each kind
  info->kernels_per_forward_decode = L->launches_decode;
  info->local_experts = L->E;
  return MOE_OK;
}

}  // extern "C"
