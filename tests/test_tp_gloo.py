"""Multi-process (gloo, world_size 2, CPU) check of the expert tensor-parallel
decomposition behind moe_layer_config.tp_rank / tp_size (include/moe.h "Tensor
parallelism"): rank r holds only the
128-column FFN chunks [r n / P, (r+1) n / P) of every routed and shared expert
-- cut by the binding's own `moe.slice_tp`, W1/W3 rows and W2 columns of the
same chunks; a ragged split here (3 chunks over 2 ranks) -- computes its partial
expert sums, the partials are summed over the group (the library's NCCL
all-reduce; gloo here), and every rank then adds the residual and deferred_in
once.  Every rank's result must equal the single-process layer (PAPER.md L219 /
L241) -- the oracle, not the CUDA library."""
import os
import socket
from types import SimpleNamespace

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import moe_oracle as O

H, F, FS, E, K, P, NDEF = 16, 384, 256, 4, 2, 2, 1


def _weights(seed=0):
    rng = np.random.default_rng(seed)
    return SimpleNamespace(
        gate_w=torch.from_numpy(rng.normal(size=(E, H)) / H ** .5),
        w13=torch.from_numpy(rng.normal(size=(E, 2 * F, H)) / H ** .5), w13_scale=None,
        w2=torch.from_numpy(rng.normal(size=(E, H, F)) / F ** .5), w2_scale=None,
        ws13=torch.from_numpy(rng.normal(size=(2 * FS, H)) / H ** .5), ws13_scale=None,
        ws2=torch.from_numpy(rng.normal(size=(H, FS)) / FS ** .5), ws2_scale=None)


def _oracle_weights(w, f, fs):
    n = lambda t: t.numpy()
    return O.OracleWeights(n(w.gate_w), None,
                           lambda e: (n(w.w13[e, :f]), n(w.w13[e, f:]), n(w.w2[e])),
                           lambda: (n(w.ws13[:fs]), n(w.ws13[fs:]), n(w.ws2)))


def _cfg(f, fs):
    return O.OracleConfig(hidden=H, ffn=f, n_experts=E, top_k=K, shared_ffn=fs, norm_topk=True)


def _worker(rank, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=P)
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
    w = _weights()
    ws = moe.slice_tp(w, rank, P, F, FS)                   # this rank's resident slice
    f_r, fs_r = ws.w2.shape[2], ws.ws2.shape[1]
    rng = np.random.default_rng(7)                         # replicated tokens: every rank sees the same batch
    x, r, din = rng.normal(size=(5, H)), rng.normal(size=(5, H)), rng.normal(size=(5, H))
    # this rank's partial expert sums (no residual / deferred_in): the slice's FFN under the
    # FULL layer's routing (routing is replicated; the gate does not depend on the slice)
    full = _oracle_weights(w, F, FS)
    idx, wt, _ = O.route(x, full.gate_w, None, _cfg(F, FS))
    part = O.moe_layer(x, _oracle_weights(ws, f_r, fs_r), _cfg(f_r, fs_r), n_deferred=NDEF,
                       forced_routing=(idx, wt))
    y_p = torch.from_numpy(part["y"])
    d_p = torch.from_numpy(part["deferred_out"])
    dist.all_reduce(y_p)                                   # the library: ncclAllReduce(fp32, sum)
    dist.all_reduce(d_p)
    y = y_p.numpy() + r + din                              # finalize on every rank
    ref = O.moe_layer(x, full, _cfg(F, FS), residual=r, n_deferred=NDEF, deferred_in=din)
    err = max(float(np.abs(y - ref["y"]).max()), float(np.abs(d_p.numpy() - ref["deferred_out"]).max()))
    q.put((rank, (f_r, fs_r, err)))
    dist.destroy_process_group()


def test_tp_decomposition_gloo():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, port, q)) for r in range(P)]
    for pr in procs:
        pr.start()
    res = dict(q.get(timeout=120) for _ in range(P))
    for pr in procs:
        pr.join(timeout=60)
    assert res[0][:2] == (128, 128) and res[1][:2] == (256, 128), res    # ragged 3-chunk split, 1/P resident
    assert all(v[2] < 1e-12 for v in res.values()), res
