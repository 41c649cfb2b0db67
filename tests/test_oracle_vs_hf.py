"""Pin the non-FP8 oracle against an implementation written by someone else:
HF transformers' DeepseekV3MoE, DeepseekV2Moe and Qwen2MoeSparseMoeBlock on CPU
(fp64).  HF's MoE output is routed + shared with NO residual add
(modeling_deepseek_v3.py DeepseekV3MoE.forward), so compare with residual=None.
Tokens in the 1e-5 tie band (north_star) are excluded."""
import numpy as np
import pytest
import torch

from oracle import moe_oracle as O

H, F, E, FS = 64, 32, 16, 48
T = 40


def _oracle_weights(gu, down, gate, bias, sh=None, sgw=None):
    exp = lambda e: (gu[e, :F], gu[e, F:], down[e])
    return O.OracleWeights(gate, bias, exp, (lambda: sh) if sh is not None else None, sgw)


def _check(hf_out, x, W, cfg, rtol=1e-9, atol=1e-10):
    orc = O.moe_layer(x, W, cfg)
    ties = set(O.tie_band_tokens(x, W, cfg).tolist())
    keep = [t for t in range(T) if t not in ties]
    assert len(keep) >= T - 2
    np.testing.assert_allclose(orc["y"][keep], hf_out[keep], rtol=rtol, atol=atol)


def test_vs_hf_deepseek_v3():
    from transformers.models.deepseek_v3.configuration_deepseek_v3 import DeepseekV3Config
    from transformers.models.deepseek_v3.modeling_deepseek_v3 import DeepseekV3MoE
    c = DeepseekV3Config(hidden_size=H, moe_intermediate_size=F, n_routed_experts=E, n_group=4,
                         topk_group=2, num_experts_per_tok=4, n_shared_experts=1, norm_topk_prob=True,
                         routed_scaling_factor=2.5, hidden_act="silu")
    m = DeepseekV3MoE(c).double().eval()
    g = torch.Generator().manual_seed(0)
    with torch.no_grad():
        m.experts.gate_up_proj.copy_(torch.randn(E, 2 * F, H, generator=g, dtype=torch.float64) / H ** 0.5)
        m.experts.down_proj.copy_(torch.randn(E, H, F, generator=g, dtype=torch.float64) / F ** 0.5)
        m.gate.weight.copy_(torch.randn(E, H, generator=g, dtype=torch.float64) / H ** 0.5)
        m.gate.e_score_correction_bias.copy_(torch.rand(E, generator=g, dtype=torch.float64) * 0.1 - 0.05)
        for lin in (m.shared_experts.gate_proj, m.shared_experts.up_proj, m.shared_experts.down_proj):
            lin.weight.copy_(torch.randn(lin.weight.shape, generator=g, dtype=torch.float64) / lin.weight.shape[1] ** 0.5)
        x = torch.randn(1, T, H, generator=g, dtype=torch.float64)
        y = m(x)[0].numpy()
    sh = (m.shared_experts.gate_proj.weight.detach().numpy(), m.shared_experts.up_proj.weight.detach().numpy(),
          m.shared_experts.down_proj.weight.detach().numpy())
    W = _oracle_weights(m.experts.gate_up_proj.detach().numpy(), m.experts.down_proj.detach().numpy(),
                        m.gate.weight.detach().numpy(), m.gate.e_score_correction_bias.numpy(), sh)
    cfg = O.OracleConfig(hidden=H, ffn=F, n_experts=E, top_k=4, n_group=4, topk_group=2,
                         group_score=O.GROUP_TOP2_SUM, score_fn=O.SCORE_SIGMOID, norm_topk=True,
                         routed_scale=2.5, shared_ffn=F)
    # HF DeepSeek routers cast to fp32 before the gate linear
    # (DeepseekV3TopkRouter.forward / DeepseekV2Moe.forward), hence ~1e-7 abs.
    _check(y, x[0].numpy(), W, cfg, rtol=1e-5, atol=2e-6)


@pytest.mark.parametrize("method", ["greedy", "group_limited_greedy"])
def test_vs_hf_deepseek_v2(method):
    from transformers.models.deepseek_v2.configuration_deepseek_v2 import DeepseekV2Config
    from transformers.models.deepseek_v2.modeling_deepseek_v2 import DeepseekV2Moe
    kw = dict(n_group=4, topk_group=2) if method != "greedy" else dict(n_group=1, topk_group=1)
    c = DeepseekV2Config(hidden_size=H, moe_intermediate_size=F, n_routed_experts=E, num_experts_per_tok=6,
                         n_shared_experts=2, routed_scaling_factor=16.0, topk_method=method,
                         hidden_act="silu", **kw)
    c.num_experts = E
    m = DeepseekV2Moe(c).double().eval()
    m.num_experts = E      # HF 5.5 group_limited_greedy reads self.num_experts, never set in __init__
    g = torch.Generator().manual_seed(1)
    with torch.no_grad():
        m.experts.gate_up_proj.copy_(torch.randn(E, 2 * F, H, generator=g, dtype=torch.float64) / H ** 0.5)
        m.experts.down_proj.copy_(torch.randn(E, H, F, generator=g, dtype=torch.float64) / F ** 0.5)
        m.gate.weight.copy_(torch.randn(E, H, generator=g, dtype=torch.float64) / H ** 0.5)
        for lin in (m.shared_experts.gate_proj, m.shared_experts.up_proj, m.shared_experts.down_proj):
            lin.weight.copy_(torch.randn(lin.weight.shape, generator=g, dtype=torch.float64) / lin.weight.shape[1] ** 0.5)
        x = torch.randn(1, T, H, generator=g, dtype=torch.float64)
        y = m(x)[0].numpy()
    sh = (m.shared_experts.gate_proj.weight.detach().numpy(), m.shared_experts.up_proj.weight.detach().numpy(),
          m.shared_experts.down_proj.weight.detach().numpy())
    W = _oracle_weights(m.experts.gate_up_proj.detach().numpy(), m.experts.down_proj.detach().numpy(),
                        m.gate.weight.detach().numpy(), None, sh)
    cfg = O.OracleConfig(hidden=H, ffn=F, n_experts=E, top_k=6, n_group=kw["n_group"],
                         topk_group=kw["topk_group"], group_score=O.GROUP_MAX, score_fn=O.SCORE_SOFTMAX,
                         norm_topk=False, routed_scale=16.0, shared_ffn=2 * F)
    _check(y, x[0].numpy(), W, cfg, rtol=1e-5, atol=2e-6)


@pytest.mark.parametrize("norm", [False, True])
def test_vs_hf_qwen2_moe(norm):
    from transformers.models.qwen2_moe.configuration_qwen2_moe import Qwen2MoeConfig
    from transformers.models.qwen2_moe.modeling_qwen2_moe import Qwen2MoeSparseMoeBlock
    c = Qwen2MoeConfig(hidden_size=H, moe_intermediate_size=F, num_experts=E, num_experts_per_tok=4,
                       shared_expert_intermediate_size=FS, norm_topk_prob=norm, hidden_act="silu")
    m = Qwen2MoeSparseMoeBlock(c).double().eval()
    g = torch.Generator().manual_seed(2)
    with torch.no_grad():
        m.experts.gate_up_proj.copy_(torch.randn(E, 2 * F, H, generator=g, dtype=torch.float64) / H ** 0.5)
        m.experts.down_proj.copy_(torch.randn(E, H, F, generator=g, dtype=torch.float64) / F ** 0.5)
        m.gate.weight.copy_(torch.randn(E, H, generator=g, dtype=torch.float64) / H ** 0.5)
        m.shared_expert_gate.weight.copy_(torch.randn(1, H, generator=g, dtype=torch.float64) / H ** 0.5)
        for lin in (m.shared_expert.gate_proj, m.shared_expert.up_proj, m.shared_expert.down_proj):
            lin.weight.copy_(torch.randn(lin.weight.shape, generator=g, dtype=torch.float64) / lin.weight.shape[1] ** 0.5)
        x = torch.randn(1, T, H, generator=g, dtype=torch.float64)
        y = m(x)[0].numpy()
    sh = (m.shared_expert.gate_proj.weight.detach().numpy(), m.shared_expert.up_proj.weight.detach().numpy(),
          m.shared_expert.down_proj.weight.detach().numpy())
    W = _oracle_weights(m.experts.gate_up_proj.detach().numpy(), m.experts.down_proj.detach().numpy(),
                        m.gate.weight.detach().numpy(), None, sh, m.shared_expert_gate.weight.detach().numpy()[0])
    cfg = O.OracleConfig(hidden=H, ffn=F, n_experts=E, top_k=4, score_fn=O.SCORE_SOFTMAX, norm_topk=norm,
                         shared_ffn=FS, shared_gated=True)
    # HF Qwen2 router: softmax(..., dtype=torch.float) -> fp32 routing weights
    _check(y, x[0].numpy(), W, cfg, rtol=1e-5, atol=2e-6)
