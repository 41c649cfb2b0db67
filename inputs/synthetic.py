"""Seeded synthetic inputs shared by the tests, the bench and the oracle.

This module holds NONE of the method's arithmetic (no gate, no FFN, no
activation quantiser, no combine).  It only draws random tensors in the
layouts `include/moe.h` documents and, for FP8 presets, stores the expert
weights the way a block-scaled FP8 checkpoint stores them (e4m3 codes +
power-of-two scales per 128x128 block, reading R10).

Recipe:
  x, residual ~ N(0, 1) -> bf16 [T, H]      (post-RMSNorm scale)
  Wg ~ N(0, 1/H) -> bf16 [E, H]              (logits ~ N(0,1): near-balanced routing,
                                              "activated in a balanced manner")
  bias ~ U(-0.05, 0.05) fp32 [E]             (DeepSeek-V3 only)
  W1/W3 ~ N(0, 1/H), W2 ~ N(0, 1/F)          (routed and shared)
      -> bf16, fp32 (toy), e4m3 + UE8M0 128x128 scales (FP8 presets) or
         packed e2m1 + UE8M0 128x128 scales (FP4 presets)
  w_sg ~ N(0, 1/H) -> bf16 [H]              (Qwen2 shared-expert gate)
  skew > 0: per-expert logit offsets via a common direction (hot experts get
      ~4x the mean load at skew=1; "imbalanced expert selection")
Weights: seed 1000 + cfg_id; inputs: seed 2000 + cfg_id (+ a caller offset).
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Optional

import torch

from .presets import LayerPreset, W_BF16, W_F32, W_FP4, W_FP8

E4M3_MAX = 448.0


@dataclass
class LayerWeights:
    """Device or host tensors in the `moe_layer_weights` layout of include/moe.h."""
    gate_w: torch.Tensor                 # [E, H] bf16
    gate_bias: Optional[torch.Tensor]    # [E] fp32 or None
    w13: torch.Tensor                    # [E, 2F, H] bf16 / fp32 / uint8 (e4m3 codes)
    w13_scale: Optional[torch.Tensor]    # [E, 2F/128, H/128] fp32 (FP8 only)
    w2: torch.Tensor                     # [E, H, F]
    w2_scale: Optional[torch.Tensor]     # [E, H/128, F/128]
    ws13: Optional[torch.Tensor]         # [2Fs, H]
    ws13_scale: Optional[torch.Tensor]
    ws2: Optional[torch.Tensor]          # [H, Fs]
    ws2_scale: Optional[torch.Tensor]
    shared_gate_w: Optional[torch.Tensor]  # [H] bf16

    def to(self, device) -> "LayerWeights":
        f = lambda t: None if t is None else t.to(device)
        return LayerWeights(*(f(getattr(self, n)) for n in self.__dataclass_fields__))


def _gen(seed: int, device) -> torch.Generator:
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    return g


def _normal(shape, std, g, device):
    return torch.randn(shape, generator=g, device=device, dtype=torch.float32) * std


def fp8_block_encode(w: torch.Tensor):
    """Store fp32 weights [..., R, C] (R, C multiples of 128) as e4m3 codes with one
    power-of-two scale per 128x128 block: scale = 2^ceil(log2(amax/448)).
    This is checkpoint preparation (the input format), not hot-path math."""
    *lead, R, C = w.shape
    b = w.reshape(*lead, R // 128, 128, C // 128, 128)
    amax = b.abs().amax(dim=(-3, -1))                                 # [..., R/128, C/128]
    m, e = torch.frexp(amax / E4M3_MAX)                               # q = m * 2^e, m in [0.5, 1)
    scale = torch.where(m == 0.5, torch.ldexp(torch.ones_like(m), e - 1),
                        torch.ldexp(torch.ones_like(m), e))
    scale = torch.where(amax > 0, scale, torch.ones_like(scale))
    q = (b / scale[..., :, None, :, None]).clamp_(-E4M3_MAX, E4M3_MAX)
    codes = q.to(torch.float8_e4m3fn).view(torch.uint8).reshape(*lead, R, C)
    return codes.contiguous(), scale.contiguous()


E2M1_MAX = 6.0


def fp4_block_encode(w: torch.Tensor):
    """Store fp32 weights [..., R, C] as OCP e2m1 codes (sign bit 3, magnitudes
    0, .5, 1, 1.5, 2, 3, 4, 6) packed two per byte (element 2i in the low nibble
    of byte i) with one power-of-two scale per 128x128 block, 2^ceil(log2(amax/6)).
    Checkpoint preparation (the input format), not hot-path math; rounding is to
    the nearest magnitude (ties either way: both sides read the stored codes)."""
    *lead, R, C = w.shape
    b = w.reshape(*lead, R // 128, 128, C // 128, 128)
    amax = b.abs().amax(dim=(-3, -1))
    m, e = torch.frexp(amax / E2M1_MAX)
    scale = torch.where(m == 0.5, torch.ldexp(torch.ones_like(m), e - 1), torch.ldexp(torch.ones_like(m), e))
    scale = torch.where(amax > 0, scale, torch.ones_like(scale))
    q = (b / scale[..., :, None, :, None]).reshape(*lead, R, C)
    mid = torch.tensor([0.25, 0.75, 1.25, 1.75, 2.5, 3.5, 5.0], device=w.device)
    code = torch.bucketize(q.abs(), mid).to(torch.uint8) | ((q < 0).to(torch.uint8) << 3)
    packed = code[..., 0::2] | (code[..., 1::2] << 4)
    return packed.contiguous(), scale.contiguous()


def _weight(shape, std, wtype, g, device):
    w = _normal(shape, std, g, device)
    if wtype == W_FP8:
        return fp8_block_encode(w)
    if wtype == W_FP4:
        return fp4_block_encode(w)
    if wtype == W_BF16:
        return w.to(torch.bfloat16), None
    return w, None


def make_weights(p: LayerPreset, device="cpu", seed: Optional[int] = None,
                 skew: float = 0.0) -> LayerWeights:
    g = _gen(1000 + p.cfg_id if seed is None else seed, device)
    H, F, E = p.hidden, p.ffn, p.n_experts
    gate_w = _normal((E, H), H ** -0.5, g, device)
    if skew > 0:
        # hot experts: add a_e * d to row e, with d a unit direction that the
        # inputs also lean on (see make_tokens(skew=...)); a_e Zipf-like.
        d = _normal((H,), 1.0, g, device)
        d = d / d.norm()
        ranks = torch.randperm(E, generator=g, device=device).to(torch.float32)
        a = skew * 1.5 / (1.0 + ranks) ** 0.5
        gate_w = gate_w + a[:, None] * d[None, :]
    gate_w = gate_w.to(torch.bfloat16)
    bias = None
    if p.has_bias:
        bias = (torch.rand((E,), generator=g, device=device) * 0.1 - 0.05).float()
    # routed experts, generated one expert at a time (V3 fp32 temp would be 45 GB)
    w13_list, s13_list, w2_list, s2_list = [], [], [], []
    for _ in range(E):
        a, sa = _weight((2 * F, H), H ** -0.5, p.wtype, g, device)
        b, sb = _weight((H, F), F ** -0.5, p.wtype, g, device)
        w13_list.append(a); w2_list.append(b); s13_list.append(sa); s2_list.append(sb)
    w13 = torch.stack(w13_list)
    w2 = torch.stack(w2_list)
    del w13_list, w2_list
    w13_scale = torch.stack(s13_list) if p.wtype in (W_FP8, W_FP4) else None
    w2_scale = torch.stack(s2_list) if p.wtype in (W_FP8, W_FP4) else None
    ws13 = ws13_scale = ws2 = ws2_scale = sgw = None
    if p.shared_ffn:
        Fs = p.shared_ffn
        ws13, ws13_scale = _weight((2 * Fs, H), H ** -0.5, p.wtype, g, device)
        ws2, ws2_scale = _weight((H, Fs), Fs ** -0.5, p.wtype, g, device)
        if p.shared_gated:
            sgw = _normal((H,), H ** -0.5, g, device).to(torch.bfloat16)
    return LayerWeights(gate_w, bias, w13, w13_scale, w2, w2_scale, ws13, ws13_scale,
                        ws2, ws2_scale, sgw)


def make_tokens(p: LayerPreset, T: int, device="cpu", offset: int = 0, skew: float = 0.0,
                weights: Optional[LayerWeights] = None):
    """x, residual ~ N(0,1) bf16 [T, H].  With skew > 0 the tokens get a
    component along the hot-expert direction (needs the same skew in make_weights)."""
    g = _gen(2000 + p.cfg_id + 7919 * offset, device)
    x = _normal((T, p.hidden), 1.0, g, device)
    residual = _normal((T, p.hidden), 1.0, g, device).to(torch.bfloat16)
    if skew > 0:
        assert weights is not None
        gw = _gen(1000 + p.cfg_id, device)
        _normal((p.n_experts, p.hidden), 1.0, gw, device)     # replay gate draw
        d = _normal((p.hidden,), 1.0, gw, device)
        d = d / d.norm()
        x = x + 2.0 * d[None, :]
    return x.to(torch.bfloat16), residual
