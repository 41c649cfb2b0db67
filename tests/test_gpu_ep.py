"""Expert parallelism through the C ABI on one GPU: an in-process group of P
ranks (moe_ep_group_forward: every transfer of the NCCL path done as device
copies) and the NCCL transport itself with a 1-rank communicator.  Each rank's
outputs are checked against the oracle on that rank's tokens."""
import numpy as np
import pytest
import torch

from inputs.presets import SMALL
from inputs.synthetic import make_tokens, make_weights
from oracle import moe_oracle as O
from tests.parity import TOL, oracle_cfg, oracle_weights, rel_l2

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def lib():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
    return moe


def _oracle_check(p, w_cpu, x, y, residual=None, n_def=0, din=None, dout=None):
    cfg, W = oracle_cfg(p), oracle_weights(p, w_cpu)
    x64 = x.to(torch.float64).numpy()
    if x64.shape[0] == 0:
        return
    ties = O.tie_band_tokens(x64, W, cfg, n_deferred=n_def)
    keep = np.setdiff1d(np.arange(x64.shape[0]), ties)
    out = O.moe_layer(x64, W, cfg, residual=None if residual is None else residual.to(torch.float64).numpy(),
                      n_deferred=n_def, deferred_in=None if din is None else din.cpu().to(torch.float64).numpy())
    assert rel_l2(y.float().cpu().numpy()[keep], out["y"][keep]) <= TOL[p.wtype]
    if dout is not None:
        assert rel_l2(dout.float().cpu().numpy()[keep], out["deferred_out"][keep]) <= TOL[p.wtype]


@pytest.mark.parametrize("name,P,Ts", [("v3_s", 2, [40, 33]), ("v3_s", 4, [25, 0, 61, 7]),
                                       ("qwen2_s", 2, [50, 19]), ("v25_s", 4, [30, 30, 30, 30]),
                                       ("v3_s", 8, [5, 9, 1, 0, 3, 17, 2, 8])])
def test_ep_group(lib, name, P, Ts):
    p = SMALL[name]
    w_cpu = make_weights(p, "cpu")
    group = lib.MoEGroup(p, w_cpu.to("cuda"), ep_size=P, max_tokens=max(Ts) or 1)
    xs = [make_tokens(p, t, "cpu", offset=r)[0] for r, t in enumerate(Ts)]
    ys = group.forward([x.cuda() for x in xs])
    torch.cuda.synchronize()
    for x, y in zip(xs, ys):
        _oracle_check(p, w_cpu, x, y)
    group.close()


def test_ep_group_deferral_and_residual(lib):
    p = SMALL["v3_s"]
    P, Ts = 2, [24, 31]
    w_cpu = make_weights(p, "cpu")
    group = lib.MoEGroup(p, w_cpu.to("cuda"), ep_size=P, max_tokens=32)
    xs, rs = zip(*[make_tokens(p, t, "cpu", offset=r) for r, t in enumerate(Ts)])
    dins = [(torch.randn(t, p.hidden, generator=torch.Generator().manual_seed(r)) * 0.5).to(torch.bfloat16)
            for r, t in enumerate(Ts)]
    ys, douts = group.forward([x.cuda() for x in xs], residuals=[r.cuda() for r in rs], n_deferred=3,
                              deferred_in=[d.cuda() for d in dins], want_deferred_out=True)
    torch.cuda.synchronize()
    for x, r, d, y, do in zip(xs, rs, dins, ys, douts):
        _oracle_check(p, w_cpu, x, y, residual=r, n_def=3, din=d, dout=do)
    group.close()


def test_ep_nccl_single_rank(lib):
    """The NCCL transport (send/recv to self) with a 1-rank communicator."""
    p = SMALL["v3_s"]
    w_cpu = make_weights(p, "cpu")
    uid = lib.get_unique_id()
    layer = lib.MoELayer(p, w_cpu.to("cuda"), max_tokens=64, ep_rank=0, ep_size=1, unique_id=uid)
    x, _ = make_tokens(p, 57, "cpu")
    y = layer.forward(x.cuda())
    torch.cuda.synchronize()
    _oracle_check(p, w_cpu, x, y)
    layer.close()


@pytest.mark.parametrize("name,P,Ts", [("v3_s", 2, [40, 33]), ("v3_s", 4, [25, 0, 61, 7]),
                                       ("qwen2_s", 2, [50, 19]), ("v3_s", 8, [5, 9, 1, 0, 3, 17, 2, 8])])
def test_ep_group_fixed_capacity(lib, name, P, Ts):
    """ep_fixed_capacity: whole max_tokens-row blocks both ways, no host synchronisation."""
    p = SMALL[name]
    w_cpu = make_weights(p, "cpu")
    group = lib.MoEGroup(p, w_cpu.to("cuda"), ep_size=P, max_tokens=max(Ts) or 1, ep_fixed=True)
    xs = [make_tokens(p, t, "cpu", offset=r)[0] for r, t in enumerate(Ts)]
    ys = group.forward([x.cuda() for x in xs])
    torch.cuda.synchronize()
    for x, y in zip(xs, ys):
        _oracle_check(p, w_cpu, x, y)
    group.close()


def test_ep_group_fixed_capacity_graph(lib):
    """The fixed-capacity EP forward captured in a CUDA graph and replayed on new tokens."""
    p = SMALL["v3_s"]
    P, Ts = 4, [24, 31, 0, 17]
    w_cpu = make_weights(p, "cpu")
    group = lib.MoEGroup(p, w_cpu.to("cuda"), ep_size=P, max_tokens=32, ep_fixed=True)
    xin = [torch.zeros(t, p.hidden, dtype=torch.bfloat16, device="cuda") for t in Ts]
    yout = [torch.empty_like(x) for x in xin]
    side = torch.cuda.Stream()
    side.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(side):
        group.forward(xin, ys=yout, stream=side)          # warm-up outside the capture
    torch.cuda.current_stream().wait_stream(side)
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph):
        group.forward(xin, ys=yout, stream=torch.cuda.current_stream())
    for rep in range(2):
        xs = [make_tokens(p, t, "cpu", offset=10 * rep + r)[0] for r, t in enumerate(Ts)]
        for dst, src in zip(xin, xs):
            dst.copy_(src)
        graph.replay()
        torch.cuda.synchronize()
        for x, y in zip(xs, yout):
            _oracle_check(p, w_cpu, x, y)
    del graph
    group.close()


def test_ep_nccl_single_rank_fixed_graph(lib):
    """The NCCL transport in fixed-capacity mode, captured in a CUDA graph (1-rank communicator)."""
    p = SMALL["v3_s"]
    w_cpu = make_weights(p, "cpu")
    uid = lib.get_unique_id()
    layer = lib.MoELayer(p, w_cpu.to("cuda"), max_tokens=64, ep_rank=0, ep_size=1, unique_id=uid, ep_fixed=True)
    xin = torch.zeros(57, p.hidden, dtype=torch.bfloat16, device="cuda")
    yout = torch.empty_like(xin)
    side = torch.cuda.Stream()
    side.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(side):
        layer.forward(xin, y=yout)
    torch.cuda.current_stream().wait_stream(side)
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph):
        layer.forward(xin, y=yout)
    for rep in range(2):
        x, _ = make_tokens(p, 57, "cpu", offset=rep)
        xin.copy_(x)
        graph.replay()
        torch.cuda.synchronize()
        _oracle_check(p, w_cpu, x, yout)
    del graph
    layer.close()


@pytest.mark.parametrize("name,P,Ts,fixed", [("v3_s", 2, [3, 5], False), ("v3_s", 4, [1, 0, 2, 1], False),
                                             ("qwen2_s", 2, [4, 1], False), ("v2lite_s", 4, [2, 2, 1, 3], False),
                                             ("v3_s", 4, [1, 1, 0, 2], True), ("v3_s_fp4", 2, [2, 3], False)])
def test_ep_group_decode_stream(lib, name, P, Ts, fixed):
    """Decode-sized EP (received rows and own tokens <= gemv_max_tokens): the expert side runs the
    fused decode stream (routed experts over the received rows, shared expert over the own tokens)."""
    p = SMALL[name]
    w_cpu = make_weights(p, "cpu")
    group = lib.MoEGroup(p, w_cpu.to("cuda"), ep_size=P, max_tokens=max(max(Ts), 1), ep_fixed=fixed)
    xs = [make_tokens(p, t, "cpu", offset=r)[0] for r, t in enumerate(Ts)]
    ys = group.forward([x.cuda() for x in xs])
    torch.cuda.synchronize()
    for x, y in zip(xs, ys):
        _oracle_check(p, w_cpu, x, y)
    group.close()


def test_ep_group_decode_stream_deferral(lib):
    p = SMALL["v3_s"]
    P, Ts = 2, [3, 4]
    w_cpu = make_weights(p, "cpu")
    group = lib.MoEGroup(p, w_cpu.to("cuda"), ep_size=P, max_tokens=4)
    xs, rs = zip(*[make_tokens(p, t, "cpu", offset=r) for r, t in enumerate(Ts)])
    dins = [(torch.randn(t, p.hidden, generator=torch.Generator().manual_seed(r)) * 0.5).to(torch.bfloat16)
            for r, t in enumerate(Ts)]
    ys, douts = group.forward([x.cuda() for x in xs], residuals=[r.cuda() for r in rs], n_deferred=3,
                              deferred_in=[d.cuda() for d in dins], want_deferred_out=True)
    torch.cuda.synchronize()
    for x, r, d, y, do in zip(xs, rs, dins, ys, douts):
        _oracle_check(p, w_cpu, x, y, residual=r, n_def=3, din=d, dout=do)
    group.close()
