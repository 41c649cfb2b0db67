"""Layer shapes of the BASELINE.json configs (data only -- no arithmetic).

Shapes: BASELINE.json `configs`; Table 1 (L334-343): DeepSeek-V3
256 experts / top-8, DeepSeek-V2(.5) 160 / top-6, Qwen2-57B 64 / top-8.
Gate rules: DESIGN.md reading R1 (public DeepSeek-V2/V3 / Qwen2-MoE
definitions; the paper only says "top-k or its variants", L98).
"""
from __future__ import annotations

from dataclasses import dataclass, replace

SCORE_SOFTMAX = 0
SCORE_SIGMOID = 1
GROUP_MAX = 0
GROUP_TOP2_SUM = 1
W_BF16 = 0
W_FP8 = 1
W_F32 = 2   # toy config only (BASELINE.json: "fp32 weights")
W_FP4 = 3   # e2m1 codes (packed 2 per byte) + power-of-two 128x128 block scales


@dataclass(frozen=True)
class LayerPreset:
    name: str
    hidden: int
    ffn: int
    n_experts: int
    top_k: int
    n_group: int = 1
    topk_group: int = 1
    group_score: int = GROUP_MAX
    score_fn: int = SCORE_SOFTMAX
    norm_topk: bool = False
    routed_scale: float = 1.0
    shared_ffn: int = 0
    shared_gated: bool = False
    wtype: int = W_BF16
    has_bias: bool = False
    decode_tokens: int = 1
    prefill_tokens: int = 512
    cfg_id: int = 0

    def with_(self, **kw) -> "LayerPreset":
        return replace(self, **kw)


PRESETS = {
    # BASELINE.json configs[0]: 8 experts top-2 softmax, H128, F256, 32 tokens,
    # fp32 weights; norm_topk=1 exercises the renormalisation path.
    "toy": LayerPreset("toy", 128, 256, 8, 2, norm_topk=True, wtype=W_F32,
                       decode_tokens=1, prefill_tokens=32, cfg_id=0),
    # configs[1]: DeepSeek-V2-Lite, 64 routed + 2 shared (Fs = 2 x 1408), top-6, greedy.
    "v2lite": LayerPreset("v2lite", 2048, 1408, 64, 6, shared_ffn=2816, wtype=W_BF16,
                          decode_tokens=1, prefill_tokens=512, cfg_id=1),
    # configs[2]: Qwen2-57B-A14B, 64 experts top-8, shared FFN 20480 (sigmoid-gated).
    "qwen2": LayerPreset("qwen2", 3584, 2560, 64, 8, shared_ffn=20480, shared_gated=True,
                         wtype=W_BF16, decode_tokens=1, prefill_tokens=2048, cfg_id=2),
    # configs[3]: DeepSeek-V2.5, 160 routed + 2 shared (Fs = 3072), top-6,
    # group_limited_greedy 8 groups / 3 kept, routed_scale 16, FP8.
    "v25": LayerPreset("v25", 5120, 1536, 160, 6, n_group=8, topk_group=3, group_score=GROUP_MAX,
                       routed_scale=16.0, shared_ffn=3072, wtype=W_FP8,
                       decode_tokens=4, prefill_tokens=4096, cfg_id=3),
    # configs[4]: DeepSeek-V3, 256 routed (8 groups, top-4 groups) + 1 shared,
    # top-8, sigmoid + bias, top-2-sum group score, renorm, scale 2.5, FP8.
    "v3": LayerPreset("v3", 7168, 2048, 256, 8, n_group=8, topk_group=4, group_score=GROUP_TOP2_SUM,
                      score_fn=SCORE_SIGMOID, norm_topk=True, routed_scale=2.5, shared_ffn=2048,
                      wtype=W_FP8, has_bias=True, decode_tokens=1, prefill_tokens=8192, cfg_id=4),
}

# Small stand-ins with the same gate rules and dtype as the large presets,
# sized so the CPU oracle checks them element by element in seconds while
# still spanning several GEMM tiles and a ragged tail.
SMALL = {
    "toy": PRESETS["toy"],
    "v2lite_s": PRESETS["v2lite"].with_(name="v2lite_s", hidden=512, ffn=384, shared_ffn=768,
                                        prefill_tokens=200),
    "qwen2_s": PRESETS["qwen2"].with_(name="qwen2_s", hidden=512, ffn=256, n_experts=16,
                                      shared_ffn=640, prefill_tokens=150),
    "v25_s": PRESETS["v25"].with_(name="v25_s", hidden=512, ffn=256, n_experts=32,
                                  shared_ffn=384, prefill_tokens=181),
    # hidden 384 (not a multiple of 256) takes the CUDA-core GEMM path
    "v2lite_h384": PRESETS["v2lite"].with_(name="v2lite_h384", hidden=384, ffn=256, n_experts=16,
                                           shared_ffn=512, prefill_tokens=77),
    "v3_s": PRESETS["v3"].with_(name="v3_s", hidden=512, ffn=256, n_experts=64,
                                shared_ffn=256, prefill_tokens=333),
    # DeepSeek-V3 gate with two groups of exactly 32 experts (the router's one-token CTA path
    # takes one group per warp)
    "v3_g32": PRESETS["v3"].with_(name="v3_g32", hidden=512, ffn=256, n_experts=64, n_group=2, topk_group=1,
                                  shared_ffn=256, prefill_tokens=200),
    # mid-size FP8: H = 2048 (16 W13 k-blocks = 4 scale groups), F = 1024 (8 W2
    # k-blocks = 2 groups), so both TMEM scale-column sets are exercised
    "v3_m": PRESETS["v3"].with_(name="v3_m", hidden=2048, ffn=1024, n_experts=32,
                                shared_ffn=1024, prefill_tokens=300),
    # 4-bit (e2m1) expert weights, DeepSeek-V3 gate (NEXT-3)
    "v3_s_fp4": PRESETS["v3"].with_(name="v3_s_fp4", hidden=512, ffn=256, n_experts=64, shared_ffn=256,
                                    prefill_tokens=333, wtype=W_FP4),
    "v3_m_fp4": PRESETS["v3"].with_(name="v3_m_fp4", hidden=2048, ffn=1024, n_experts=32, shared_ffn=1024,
                                    prefill_tokens=300, wtype=W_FP4),
}

# the DeepSeek-V3 layer with 4-bit expert weights (decode bytes halved, NEXT-3)
PRESETS["v3_fp4"] = PRESETS["v3"].with_(name="v3_fp4", wtype=W_FP4)
