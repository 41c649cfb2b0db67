"""Optional on-box comparator (context only, never linked into the product):
FlashInfer's TRT-LLM fused MoE for Blackwell, `trtllm_fp8_block_scale_moe` (DeepSeek-V3 routing
from fp32 logits, 128x128 block-scaled FP8 weights, 1x128 activation scales, SwiGLU, finalize),
timed on V3-shaped synthetic inputs beside this library's layer.  It covers the routed experts
only (no shared expert, no router GEMM), so the library's routed-only time is printed beside it:
router-select + permute + scatter + both grouped GEMMs + combine minus the shared expert's share
is not separable in our fused launches, so we print the whole layer and the GEMM stages.

python scripts/flashinfer_comparator.py [T]"""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

T = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
H, F, E, K, NG, TG, SCALE = 7168, 2048, 256, 8, 8, 4, 2.5
dev = "cuda"
g = torch.Generator(device=dev).manual_seed(7)


def fp8_blocks(shape_rows, cols, nexp):
    w = (torch.randn(nexp, shape_rows, cols, generator=g, device=dev) / cols ** 0.5)
    amax = w.abs().reshape(nexp, shape_rows // 128, 128, cols // 128, 128).amax(dim=(2, 4)).clamp_min(1e-12)
    s = torch.exp2(torch.ceil(torch.log2(amax / 448.0)))
    q = (w / s.repeat_interleave(128, 1).repeat_interleave(128, 2)).to(torch.float8_e4m3fn)
    return q, s.float()


def timed(fn, iters=10, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ts = []
    for _ in range(iters):
        flush.zero_()
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    ts.sort()
    return ts[len(ts) // 2]


out = {"T": T, "shape": "V3 (H 7168, F 2048, E 256, top-8, groups 8/4, scale 2.5)"}
# ---- FlashInfer trtllm_fp8_block_scale_moe (routed experts only) ----
try:
    from flashinfer.fused_moe import trtllm_fp8_block_scale_moe
    w13, s13 = fp8_blocks(2 * F, H, E)
    w2, s2 = fp8_blocks(H, F, E)
    x = torch.randn(T, H, generator=g, device=dev)
    xa = x.abs().reshape(T, H // 128, 128).amax(-1).clamp_min(1e-12)
    xs = torch.exp2(torch.ceil(torch.log2(xa / 448.0)))
    xq = (x / xs.repeat_interleave(128, 1)).to(torch.float8_e4m3fn)
    logits = torch.randn(T, E, generator=g, device=dev).float()
    bias = (torch.rand(E, generator=g, device=dev) * 0.1 - 0.05).to(torch.bfloat16)

    def fi():
        return trtllm_fp8_block_scale_moe(logits, bias, xq, xs.t().contiguous(), w13, s13, w2, s2, E, K, NG, TG, F,
                                          0, E, SCALE, routing_method_type=2, use_shuffled_weight=False,
                                          weight_layout=0, tune_max_num_tokens=T)
    tuned = False
    try:                                      # let FlashInfer pick its tactics for this shape first
        from flashinfer.autotuner import autotune
        with autotune(True):
            fi()
        torch.cuda.synchronize()
        tuned = True
    except Exception:
        pass
    ms = timed(fi)
    fl = 2 * T * K * 3 * H * F
    out["flashinfer_trtllm_fp8_block_scale_moe"] = {"ms": ms, "tokens_per_s": T / (ms * 1e-3),
                                                    "routed_tflops": fl / (ms * 1e-3) / 1e12, "autotuned": tuned}
    del w13, w2
    torch.cuda.empty_cache()
except Exception as ex:  # the comparator is optional: report why it could not run
    out["flashinfer_trtllm_fp8_block_scale_moe"] = {"error": f"{type(ex).__name__}: {str(ex)[:400]}"}

# ---- this library: the whole V3 layer (router + shared expert included) and its stages ----
from inputs.presets import PRESETS
from inputs.synthetic import make_tokens, make_weights
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
p = PRESETS["v3"]
w = make_weights(p, dev)
x, _ = make_tokens(p, T, dev)
layer = moe.MoELayer(p, w, max_tokens=T)
y = torch.empty_like(x)
ms = timed(lambda: layer.forward(x, y=y))
layer.profile(True)
for _ in range(3):
    layer.forward(x, y=y)
st = layer.stage_times()
layer.profile(False)
out["this_library_layer"] = {"ms": ms, "tokens_per_s": T / (ms * 1e-3),
                             "stage_ms": {k: round(v, 4) for k, v in st.items() if v > 0},
                             "note": "includes the router GEMM and the shared expert (0.72 TF) that the comparator omits"}
print(json.dumps(out))
