"""Multi-process (gloo, world_size 2, CPU) check of the expert-parallel
decomposition the library implements: each rank routes its
own tokens, ships each token row once to every rank owning one of its experts
with the expert ids masked to that rank, the owner returns one weighted partial
row per (token, rank), and the origin adds the partials to its shared expert.
The sum must equal the single-process layer -- oracle only."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import moe_oracle as O

H, F, E, K, P = 32, 16, 8, 3, 2


def _layer(seed=0):
    rng = np.random.default_rng(seed)
    Ws = [(rng.normal(size=(F, H)) / H ** .5, rng.normal(size=(F, H)) / H ** .5, rng.normal(size=(H, F)) / F ** .5)
          for _ in range(E)]
    Sh = (rng.normal(size=(F, H)) / H ** .5, rng.normal(size=(F, H)) / H ** .5, rng.normal(size=(H, F)) / F ** .5)
    W = O.OracleWeights(rng.normal(size=(E, H)) / H ** .5, None, lambda e: Ws[e], lambda: Sh)
    cfg = O.OracleConfig(hidden=H, ffn=F, n_experts=E, top_k=K, shared_ffn=F, norm_topk=True)
    return W, cfg


def _worker(rank, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=P)
    W, cfg = _layer()
    rng = np.random.default_rng(100 + rank)
    T = 5 + 4 * rank
    x = rng.normal(size=(T, H))
    idx, w, _ = O.route(x, W.gate_w, None, cfg)
    E_loc = E // P
    # plan + pack: one row per (token, destination) with masked expert ids
    send = []
    for d in range(P):
        rows = [t for t in range(T) if np.any(idx[t] // E_loc == d)]
        ids = np.where(idx[rows] // E_loc == d, idx[rows], -1) if rows else np.zeros((0, K), int)
        send.append((np.array(rows, int), x[rows], ids, w[rows]))
    gathered = [None] * P
    dist.all_gather_object(gathered, [s[1:] for s in send])
    recv = [gathered[s][rank] for s in range(P)]
    # expert side: partial rows = sum over this rank's experts of w * FFN_e(x)
    partials = []
    for xr, ids, wr in recv:
        part = np.zeros((xr.shape[0], H))
        for i in range(xr.shape[0]):
            for j in range(K):
                if ids[i, j] >= 0:
                    w1, w3, w2 = W.expert(int(ids[i, j]))
                    part[i] += wr[i, j] * O.swiglu_ffn(xr[i:i + 1], w1, w3, w2)[0]
        partials.append(part)
    back = [None] * P
    dist.all_gather_object(back, partials)
    y = O.shared_expert(x, W, cfg)
    for d in range(P):
        rows = send[d][0]
        if len(rows):
            y[rows] += back[d][rank]
    ref = O.moe_layer(x, W, cfg)["y"]
    q.put((rank, float(np.abs(y - ref).max())))
    dist.destroy_process_group()


def test_ep_decomposition_gloo():
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
