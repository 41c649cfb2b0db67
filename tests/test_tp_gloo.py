"""Multi-process (gloo, world_size 2, CPU) check of the decode tensor-parallel
decomposition behind moe_layer_set_decode_tp (PAPER.md
L195-197): rank r evaluates only the FFN column chunks c = r (mod P) of every
routed and shared expert -- W1/W3 rows and W2 columns of the same chunk, as the
fused decode stream does -- adds the residual on rank 0 only, and
`moe.decode_tp_forward` all-reduces the partials.  The sum must equal the
single-process layer -- the oracle, not the CUDA library."""
import os
import socket

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import moe_oracle as O

H, F, E, K, P, CH = 32, 24, 8, 3, 2, 4       # F / CH = 6 chunks; rank 0 takes 0,2,4, rank 1 takes 1,3,5


def _layer(seed=0):
    rng = np.random.default_rng(seed)
    Ws = [(rng.normal(size=(F, H)) / H ** .5, rng.normal(size=(F, H)) / H ** .5, rng.normal(size=(H, F)) / F ** .5)
          for _ in range(E)]
    Sh = (rng.normal(size=(F, H)) / H ** .5, rng.normal(size=(F, H)) / H ** .5, rng.normal(size=(H, F)) / F ** .5)
    W = O.OracleWeights(rng.normal(size=(E, H)) / H ** .5, None, lambda e: Ws[e], lambda: Sh)
    cfg = O.OracleConfig(hidden=H, ffn=F, n_experts=E, top_k=K, shared_ffn=F, norm_topk=True)
    return W, cfg


class _ChunkLayer:
    """Stands in for a MoELayer after set_decode_tp(rank, P): forward returns
    this rank's partial output (its chunks of every expert)."""

    def __init__(self, W, cfg, rank):
        self.W, self.cfg, self.rank = W, cfg, rank
        self.cols = np.concatenate([np.arange(c * CH, (c + 1) * CH) for c in range(F // CH) if c % P == rank])

    def _ffn(self, x, w1, w3, w2):
        c = self.cols
        return O.swiglu_ffn(x, w1[c], w3[c], w2[:, c])

    def forward(self, x, residual=None):
        xn = x.numpy()
        idx, w, _ = O.route(xn, self.W.gate_w, None, self.cfg)
        y = self._ffn(xn, *self.W.shared())
        for t in range(xn.shape[0]):
            for j in range(K):
                y[t] += w[t, j] * self._ffn(xn[t:t + 1], *self.W.expert(int(idx[t, j])))[0]
        if self.rank == 0 and residual is not None:
            y += residual.numpy()
        return torch.from_numpy(y)


def _worker(rank, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=P)
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
    W, cfg = _layer()
    rng = np.random.default_rng(7)                  # replicated tokens: every rank sees the same batch
    x, r = rng.normal(size=(5, H)), rng.normal(size=(5, H))
    y = moe.decode_tp_forward(_ChunkLayer(W, cfg, rank), torch.from_numpy(x), torch.from_numpy(r))
    ref = O.moe_layer(x, W, cfg, residual=r)["y"]
    q.put((rank, float(np.abs(y.numpy() - ref).max())))
    dist.destroy_process_group()


def test_decode_tp_decomposition_gloo():
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
    assert all(v < 1e-12 for v in res.values()), res
