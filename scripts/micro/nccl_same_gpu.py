"""Probe: can two NCCL ranks share one GPU (an EP/TP NCCL smoke test on a 1-GPU box)?"""
import os, sys
import torch, torch.multiprocessing as mp


def w(rank, port, q):
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
    import ctypes
    torch.cuda.set_device(0)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=2)
    uid = [moe.get_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(uid, src=0)
    lib = moe.load_library()
    try:
        from inputs.presets import SMALL
        from inputs.synthetic import make_weights, make_tokens
        p = SMALL["v3_s"]
        wt = moe.slice_tp(make_weights(p, "cpu"), rank, 2, p.ffn, p.shared_ffn).to("cuda")
        l = moe.MoELayer(p, wt, max_tokens=16, tp_rank=rank, tp_size=2, unique_id=uid[0])
        x, r = make_tokens(p, 3, "cuda")
        y = l.forward(x, residual=r)
        torch.cuda.synchronize()
        q.put((rank, "ok", float(y.float().abs().sum())))
    except Exception as e:
        q.put((rank, "err", str(e)[:300]))
    dist.destroy_process_group()


if __name__ == "__main__":
    import socket
    s = socket.socket(); s.bind(("127.0.0.1", 0)); port = s.getsockname()[1]; s.close()
    ctx = mp.get_context("spawn"); q = ctx.Queue()
    ps = [ctx.Process(target=w, args=(r, port, q)) for r in range(2)]
    [p.start() for p in ps]
    print([q.get(timeout=300) for _ in range(2)])
    [p.join(timeout=60) for p in ps]
