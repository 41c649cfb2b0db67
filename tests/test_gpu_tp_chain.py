"""GPU parity of the two §8(f) rows built on the fused decode stream, through the C ABI:
  * expert tensor parallelism (NEXT-1; Fig. 8b): P ranks each
    holding 1/P of every expert (moe.slice_tp), partials summed in fp32
    (moe_tp_group_forward, the in-process stand-in of the NCCL all-reduce);
  * Expert Deferral chained across layers (NEXT-2; Eq. 2):
    moe_layer_forward_chained, layer k computes layer k-1's deferred experts.
Both against the fp64 oracle (oracle/) on the same seeded inputs."""
import numpy as np
import pytest
import torch

from inputs.presets import PRESETS, SMALL
from inputs.synthetic import make_tokens, make_weights
from oracle import moe_oracle as O
from tests.parity import (TOL, check_output, check_tie_fraction, merged_routing, oracle_cfg, oracle_weights)

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def lib():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
    return moe


def _din(T, H, seed=7):
    return (torch.randn(T, H, generator=torch.Generator().manual_seed(seed)) * 0.5).to(torch.bfloat16)


# ------------------------------------------------------------------ expert TP
@pytest.mark.parametrize("name,P", [("v3_s", 2), ("qwen2_s", 2), ("v25_s", 2), ("v2lite_s", 2), ("v2lite_s", 3),
                                    ("v3_m", 4), ("v3_m", 3), ("v3_m_fp4", 4)])
@pytest.mark.parametrize("T", [1, 6, 16])
def test_tp_group_matches_oracle(lib, name, P, T):
    """Every rank's y (and deferred_out) equals the whole layer's (Eq. L241 middle
    case: residual + deferred_in, n_def slots deferred).  v2lite_s (F/128 = 3) and
    v3_m at P = 3 split the chunks raggedly."""
    p = SMALL[name]
    n_def = min(2, p.top_k - 1)
    w_cpu = make_weights(p, "cpu")
    x_cpu, r_cpu = make_tokens(p, T, "cpu", offset=11)
    din = _din(T, p.hidden)
    whole = lib.MoELayer(p, w_cpu.to("cuda"), max_tokens=16)
    routing = {}
    whole.forward(x_cpu.cuda(), routing=routing)            # routing, for the oracle's tie band
    grp = lib.TPGroup(p, w_cpu.to("cuda"), P, max_tokens=16)
    wb = [l.info().weight_bytes for l in grp.layers]
    assert max(wb) < whole.info().weight_bytes * (1.0 / P + 0.34), (wb, whole.info().weight_bytes)
    xs = [x_cpu.cuda()] * P
    ys, ds = grp.forward(xs, residuals=[r_cpu.cuda()] * P, n_deferred=n_def, deferred_in=[din.cuda()] * P,
                         want_deferred_out=True)
    torch.cuda.synchronize()
    cfg, W = oracle_cfg(p), oracle_weights(p, w_cpu)
    x64 = x_cpu.to(torch.float64).numpy()
    ties = O.tie_band_tokens(x64, W, cfg, n_deferred=n_def)
    idx, wt = merged_routing(x64, W, cfg, routing["topk_idx"].cpu().numpy(), ties)
    out = O.moe_layer(x64, W, cfg, residual=r_cpu.to(torch.float64).numpy(), n_deferred=n_def,
                      deferred_in=din.to(torch.float64).numpy(), forced_routing=(idx, wt))
    keep = np.setdiff1d(np.arange(T), ties)
    for r in range(P):
        check_output(f"tp/{name}/P{P}/T{T}/rank{r}/y", ys[r].float().cpu().numpy()[keep], out["y"][keep], TOL[p.wtype])
        check_output(f"tp/{name}/P{P}/T{T}/rank{r}/deferred_out", ds[r].float().cpu().numpy()[keep],
                     out["deferred_out"][keep], TOL[p.wtype])
    # every rank holds the same sum
    for r in range(1, P):
        assert torch.equal(ys[r], ys[0])
    grp.close()
    whole.close()


def test_tp_errors(lib):
    p = SMALL["v3_s"]                                     # F/128 = Fs/128 = 2
    w = make_weights(p, "cpu").to("cuda")
    with pytest.raises(lib.MoEError):                     # more ranks than chunks
        lib.MoELayer(p, lib.slice_tp(w, 0, 3, p.ffn, p.shared_ffn), max_tokens=16, tp_rank=0, tp_size=3)
    with pytest.raises(lib.MoEError):                     # rank out of range
        lib.MoELayer(p, w, max_tokens=16, tp_rank=2, tp_size=2)
    grp = lib.TPGroup(p, w, 2, max_tokens=64)
    x, r = make_tokens(p, 40, "cuda")                     # above the decode stream: refused, not silently partial
    with pytest.raises(lib.MoEError) as e:
        grp.forward([x, x], residuals=[r, r])
    assert e.value.status == -2
    with pytest.raises(lib.MoEError) as e:                # a rank of an in-process group alone: no silent partial
        grp.layers[0].forward(x[:4].contiguous())
    assert e.value.status == -1
    grp.close()


@pytest.mark.parametrize("name,Ps", [("v3", (2, 4, 8)), ("v25", (5, 8)), ("qwen2", (3, 8))])
def test_full_tp_matches_whole(lib, name, Ps):
    """Full-size layers, T = 1 and 4: the TP group's y equals the single-GPU
    forward within the north_star tolerance; per-rank weight bytes ~ 1/P.  V2.5
    (12 routed chunks) at P = 5 / 8 and Qwen2 at P = 3 are ragged splits."""
    p = PRESETS[name]
    w = make_weights(p, "cuda")
    whole = lib.MoELayer(p, w, max_tokens=16)
    wb_whole = whole.info().weight_bytes
    for P in Ps:
        grp = lib.TPGroup(p, w, P, max_tokens=16)
        assert max(l.info().weight_bytes for l in grp.layers) < wb_whole * (1.0 / P + 0.1)
        for T in (1, 4):
            x, r = make_tokens(p, T, "cuda", offset=P)
            ref = whole.forward(x, residual=r).float()
            ys = grp.forward([x] * P, residuals=[r] * P)
            check_output(f"tp_full/{name}/P{P}/T{T}", ys[0].float().cpu().numpy(), ref.cpu().numpy(), TOL[p.wtype])
        grp.close()
        torch.cuda.empty_cache()
    whole.close()


# ------------------------------------------------------------------ chained Expert Deferral
def _chain_oracle(p, ws, xs, rs, n_defs):
    """Eq. L241 over a chain of layers: O_k = I_k + S_k + R^def_{k-1}(I_{k-1}) + R^imm_k(I_k)
    with the k = 1 (no deferred_in) and k = L (n_def = 0) cases; layer k's input is the
    GPU's x_k (so every layer is checked on identical inputs)."""
    cfg = oracle_cfg(p)
    outs, din, ties = [], None, set()
    for k, (w, x, r, nd) in enumerate(zip(ws, xs, rs, n_defs)):
        W = oracle_weights(p, w)
        x64 = x.cpu().to(torch.float64).numpy()
        t = O.tie_band_tokens(x64, W, cfg, n_deferred=nd)
        ties |= set(t.tolist())
        o = O.moe_layer(x64, W, cfg, residual=None if r is None else r.cpu().to(torch.float64).numpy(),
                        n_deferred=nd, deferred_in=din)
        outs.append(o["y"])
        din = o["deferred_out"]
    return outs, sorted(ties)


@pytest.mark.parametrize("name", ["v3_s", "qwen2_s", "v2lite_s", "v3_m", "v25_s", "v3_s_fp4", "v3_g32"])
@pytest.mark.parametrize("T", [1, 5, 16])
def test_chained_deferral_matches_eq_L241(lib, name, T):
    """A 3-layer chain (k = 1: no deferred input; k = L: n_def = 0) against Eq.
    L241 evaluated by the oracle.  Each layer gets its own seeded tokens (the
    chain's data dependence x_{k+1} = O_k is not what is checked here, the
    deferred term R^def_{k-1}(I_{k-1}) joining O_k is) and residual = NULL
    (reading R12: a residual would dilute the error)."""
    p = SMALL[name]
    n_def = min(3, p.top_k - 1)
    L = 3
    ws = [make_weights(p, "cpu", seed=4000 + 17 * i) for i in range(L)]
    layers = [lib.MoELayer(p, w.to("cuda"), max_tokens=16) for w in ws]
    xs = [make_tokens(p, T, "cuda", offset=21 + i)[0] for i in range(L)]
    ys, prev = [], None
    for i, l in enumerate(layers):
        nd = n_def if i < L - 1 else 0                   # k = L: all experts immediate (L215)
        ys.append(l.forward_chained(xs[i], n_deferred=nd, prev=prev))
        prev = l
    torch.cuda.synchronize()
    outs, ties = _chain_oracle(p, ws, xs, [None] * L, [n_def] * (L - 1) + [0])
    check_tie_fraction(ties, T * L)
    keep = np.setdiff1d(np.arange(T), ties)
    for i in range(L):
        check_output(f"chain/{name}/T{T}/layer{i}", ys[i].float().cpu().numpy()[keep], outs[i][keep], TOL[p.wtype])
    for l in layers:
        l.close()


@pytest.mark.parametrize("name", ["v3_s", "v3_g32"])
@pytest.mark.parametrize("T", [1, 5])
def test_cyclic_chain_matches_eq_L241(lib, name, T):
    """Two layers used cyclically, A B A B, every call deferring (the steady state bench.py's
    decode.deferral.steady_state times): the second A takes B's deferred experts, so the
    sequence is the Eq. L241 chain over [wA, wB, wA, wB] whose last layer keeps its deferred
    slots pending."""
    p = SMALL[name]
    n_def = 3
    wA, wB = make_weights(p, "cpu", seed=4100), make_weights(p, "cpu", seed=4117)
    A = lib.MoELayer(p, wA.to("cuda"), max_tokens=16)
    B = lib.MoELayer(p, wB.to("cuda"), max_tokens=16)
    seq = [A, B, A, B]
    xs = [make_tokens(p, T, "cuda", offset=41 + i)[0] for i in range(4)]
    ys, prev = [], None
    for i, l in enumerate(seq):
        ys.append(l.forward_chained(xs[i], n_deferred=n_def, prev=prev))
        prev = l
    torch.cuda.synchronize()
    outs, ties = _chain_oracle(p, [wA, wB, wA, wB], xs, [None] * 4, [n_def] * 4)
    keep = np.setdiff1d(np.arange(T), ties)
    for i in range(4):
        check_output(f"cyclic/{name}/T{T}/call{i}", ys[i].float().cpu().numpy()[keep], outs[i][keep], TOL[p.wtype])
    A.close()
    B.close()


def test_chained_without_deferral_is_the_plain_forward(lib):
    p = SMALL["v3_s"]
    w = make_weights(p, "cpu").to("cuda")
    a = lib.MoELayer(p, w, max_tokens=16)
    x, r = make_tokens(p, 5, "cuda")
    y1 = a.forward(x, residual=r).float()
    y2 = a.forward_chained(x, residual=r, n_deferred=0).float()
    torch.cuda.synchronize()
    assert (y1 - y2).abs().max().item() <= 2 ** -6 * max(1.0, y1.abs().max().item())
    a.close()


def test_chained_errors(lib):
    p = SMALL["v3_s"]
    a = lib.MoELayer(p, make_weights(p, "cpu").to("cuda"), max_tokens=64)
    b = lib.MoELayer(p, make_weights(p, "cpu", seed=77).to("cuda"), max_tokens=64)
    x, r = make_tokens(p, 4, "cuda")
    with pytest.raises(lib.MoEError):                     # b's last call was not a chained deferral
        a.forward_chained(x, residual=r, n_deferred=2, prev=b)
    y = b.forward_chained(x, residual=r, n_deferred=2)
    with pytest.raises(lib.MoEError):                     # prev is this layer
        b.forward_chained(y, residual=y, n_deferred=2, prev=b)
    with pytest.raises(lib.MoEError):                     # other T
        a.forward_chained(y[:3].contiguous(), residual=y[:3].contiguous(), n_deferred=0, prev=b)
    a.forward_chained(y, residual=y, n_deferred=0, prev=b)
    with pytest.raises(lib.MoEError):                     # consumed once only
        a.forward_chained(y, residual=y, n_deferred=0, prev=b)
    x40, r40 = make_tokens(p, 40, "cuda")
    with pytest.raises(lib.MoEError) as e:                # prefill-size T: decode path only (L245)
        a.forward_chained(x40, residual=r40, n_deferred=2)
    assert e.value.status == -2
    torch.cuda.synchronize()
    a.close()
    b.close()


def test_full_v25_cyclic_chain_decode(lib):
    """Full DeepSeek-V2.5 layers (FP8, 160 experts, softmax + group-limited gate), T = 4,
    used cyclically A B A (every call defers 3 of 6 slots) -- the configuration whose
    steady-state deferral timing (profiles/r02/all_configs.md) is the fastest -- against
    the Eq. L241 oracle chain over [wA, wB, wA]."""
    p = PRESETS["v25"]
    T, n_def = 4, 3
    wA, wB = make_weights(p, "cuda", seed=5100), make_weights(p, "cuda", seed=5101)
    A = lib.MoELayer(p, wA, max_tokens=16)
    B = lib.MoELayer(p, wB, max_tokens=16)
    xs = [make_tokens(p, T, "cuda", offset=51 + i)[0] for i in range(3)]
    ys, prev = [], None
    for i, l in enumerate([A, B, A]):
        ys.append(l.forward_chained(xs[i], n_deferred=n_def, prev=prev))
        prev = l
    torch.cuda.synchronize()
    outs, ties = _chain_oracle(p, [wA, wB, wA], xs, [None] * 3, [n_def] * 3)
    keep = np.setdiff1d(np.arange(T), ties)
    for i in range(3):
        check_output(f"cyclic_full/v25/T{T}/call{i}", ys[i].float().cpu().numpy()[keep], outs[i][keep], TOL[p.wtype])
    A.close()
    B.close()


def test_full_v3_chain_decode(lib):
    """Full DeepSeek-V3 layers (FP8, 256 experts, n_def = 3, BF16 setting L257),
    a 3-layer chain at T = 1 and 4 vs the Eq. L241 oracle chain."""
    p = PRESETS["v3"]
    L = 3
    ws = [make_weights(p, "cuda", seed=5000 + i) for i in range(L)]
    layers = [lib.MoELayer(p, w, max_tokens=16) for w in ws]
    for T in (1, 4):
        xs = [make_tokens(p, T, "cuda", offset=5 + i)[0] for i in range(L)]
        ys, prev = [], None
        for i, l in enumerate(layers):
            ys.append(l.forward_chained(xs[i], n_deferred=3 if i < L - 1 else 0, prev=prev))
            prev = l
        torch.cuda.synchronize()
        outs, ties = _chain_oracle(p, ws, xs, [None] * L, [3, 3, 0])
        keep = np.setdiff1d(np.arange(T), ties)
        for i in range(L):
            check_output(f"chain_full/v3/T{T}/layer{i}", ys[i].float().cpu().numpy()[keep], outs[i][keep],
                         TOL[p.wtype])
    for l in layers:
        l.close()
