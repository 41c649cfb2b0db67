#!/usr/bin/env python
"""Benchmark of the B200 MoE routed-expert layer (BASELINE.json metric:
"MoE-layer prefill tokens/s & decode µs/layer; % of HBM or tensor peak").

A step = one full forward of the layer -- router logits, score/group top-k,
count/permute, FP8 activation quantisation, gather, grouped GEMM1+SwiGLU,
grouped GEMM2, shared expert, weighted combine -- over one batch of synthetic
tokens shaped like the DeepSeek-V3 MoE layer (256 routed experts in 8 groups,
top-4 groups, top-8, H 7168, F 2048, 1 shared expert, FP8 128x128 block-scaled
weights; BASELINE.json configs[4]), prefill T = 8192 tokens per GPU.

    python bench.py [--gpus N --steps K --warmup W] [--impl reference] [--config v3|v25|qwen2|v2lite|all]

N > 1: one process per GPU.  Launched without torchrun, `--gpus N` re-executes
itself under `torch.distributed.run --nproc-per-node N` (and exits with an
error if fewer than N GPUs are visible).  Each rank owns E/N experts (expert
parallelism over NCCL) and T tokens (weak scaling);
`--replicas` runs N independent single-GPU layers instead.  value = all ranks'
tokens / max-over-ranks time.

Inputs are resident in HBM when the timed region starts; L2 is flushed (a
256 MiB write, then a 256 MiB read so the dirty lines are written back before
the events start; all outside the timed events) before every timed step.  Each step is
timed with CUDA events on the launching stream.  `e2e` re-times the same step
through the public API with host (pinned) input/output buffers, H2D and D2H
inside the events.  The oracle (oracle/, a plain fp64 CPU program) is timed on
a bounded sample for `cpu_baseline` and, with --impl reference, as the
reference arm.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "MoE-layer prefill tokens/s & decode µs/layer; % of HBM or tensor peak"
PEAKS_FALLBACK = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        d["_source"] = "measured (MEASURED_PEAKS.json)"
        return d
    d = dict(PEAKS_FALLBACK)
    d["_source"] = "fallback (B200_PROFILING.md)"
    return d


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms during the timed region."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device = device
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [s.strip() for s in line.split(",")]
            if len(parts) == 7:
                self.rows.append(parts)

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            self.proc.wait(timeout=5)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = sorted(float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit())
        mx = max(float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit())
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[3 + i].lower() == "active"})
        return {"sm_mhz": sm[len(sm) // 2] if sm else None, "sm_max_mhz": mx, "reasons": reasons,
                "samples": len(self.rows)}


def dist_setup():
    import torch
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if ws > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    else:
        torch.cuda.set_device(local)
    return ws, rank, local


def barrier(ws):
    if ws > 1:
        import torch.distributed as dist
        dist.barrier()


def max_over_ranks(v: float, ws: int) -> float:
    if ws == 1:
        return v
    import torch
    import torch.distributed as dist
    t = torch.tensor([v], dtype=torch.float64, device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


# --------------------------------------------------------------------- oracle
def oracle_layer_call(p, w, x_rows):
    """Time ONE full-layer call of the CPU oracle (as it stands: every expert the
    batch hits is dequantised once in that call) on a bounded batch of tokens.
    Returns (tokens/s, distinct experts hit, seconds)."""
    import torch
    from oracle import moe_oracle as O
    from tests.parity import oracle_cfg, oracle_weights
    cfg, W = oracle_cfg(p), oracle_weights(p, w)
    x64 = x_rows.cpu().to(torch.float64).numpy()
    t0 = time.perf_counter()
    out = O.moe_layer(x64, W, cfg)
    dt = time.perf_counter() - t0
    return x64.shape[0] / dt, len(set(out["idx"].reshape(-1).tolist())), dt


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def cpu_cores():
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count()


def prefill_config(p, T, parallelism):
    """The `config` object of the prefill line (shared by both arms)."""
    weights = {0: "bf16", 1: "fp8_e4m3_block128_ue8m0", 2: "f32", 3: "fp4_e2m1_block128_ue8m0"}[p.wtype]
    return {"workload": f"{p.name}_moe_layer_prefill", "tokens_per_gpu": T, "hidden": p.hidden, "ffn": p.ffn,
            "experts": p.n_experts, "top_k": p.top_k, "shared_ffn": p.shared_ffn,
            "weights": weights, "parallelism": parallelism}


def run_reference(args):
    """--impl reference: the oracle (the reference is a paper, no installable code) timed on
    the host cores, on our arm's metric and config.  Each step is one full-layer oracle call
    (as it stands: every expert the batch hits is dequantised in the call) on a bounded
    sample of the workload's tokens -- `--ref-tokens` per step -- so the default run ends
    within a few minutes.  Under torchrun only rank 0 runs."""
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import torch
    from inputs.presets import PRESETS
    from inputs.synthetic import make_tokens, make_weights
    p = PRESETS[args.config]
    T = args.tokens or p.prefill_tokens
    dev = "cuda" if torch.cuda.is_available() else "cpu"
    w = make_weights(p, dev)
    nt = max(1, min(args.ref_tokens, T))
    x, _ = make_tokens(p, nt * (args.steps + args.warmup), dev)
    for i in range(args.warmup):
        oracle_layer_call(p, w, x[i * nt:(i + 1) * nt])
    dts, nexps = [], []
    for i in range(args.steps):
        j = args.warmup + i
        _, nexp, dt = oracle_layer_call(p, w, x[j * nt:(j + 1) * nt])
        dts.append(dt)
        nexps.append(nexp)
    dt = sum(dts)
    v = nt * args.steps / dt
    cfg = prefill_config(p, T, "single")
    cfg["sample"] = (f"{nt} tokens per step of the {T}-token workload (one full-layer oracle call per step, "
                     f"{min(nexps)}-{max(nexps)} distinct experts dequantised in the call)")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "tokens/s", "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": cfg,
            "cpu_baseline": {"value": v, "unit": "tokens/s", "cores": cpu_cores(), "cpu_model": cpu_model(),
                             "kind": "oracle", "sample": cfg["sample"]},
            "e2e": {"value": v, "unit": "tokens/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# --------------------------------------------------------------------- ours
def algorithmic(p, T, n_distinct):
    """Algorithmic FLOPs / bytes per stage."""
    H, F, Fs, k, E = p.hidden, p.ffn, p.shared_ffn, p.top_k, p.n_experts
    wb = {0: 2, 1: 1, 2: 4, 3: 0.5}[p.wtype]           # bf16, e4m3, f32, packed e2m1 bytes per weight
    blocked = p.wtype in (1, 3)                          # + one fp32 scale per 128x128 block
    exp_bytes = 3 * H * F * wb + (3 * (H // 128) * (F // 128) * 4 if blocked else 0)
    # one launch computes the routed experts AND the shared expert (two operand groups)
    return {
        "gemm1_swiglu": {"flops": 2.0 * T * k * 2 * F * H + 2.0 * T * 2 * Fs * H,
                         "bytes": n_distinct * 2 * H * F * wb + 2 * H * Fs * wb},
        "gemm2": {"flops": 2.0 * T * k * H * F + 2.0 * T * H * Fs, "bytes": n_distinct * H * F * wb + H * Fs * wb},
        "shared_gemm1": {"flops": 2.0 * T * 2 * Fs * H, "bytes": 2 * H * Fs * wb},
        "shared_gemm2": {"flops": 2.0 * T * H * Fs, "bytes": H * Fs * wb},
        "router_logits": {"flops": 2.0 * T * H * E, "bytes": E * H * 2 + T * H * 2},
        "layer_bytes": n_distinct * exp_bytes + (3 * H * Fs * wb if Fs else 0) + E * H * 2 + 2 * T * H * 2,
        "layer_flops": 2.0 * T * k * 3 * H * F + 2.0 * T * 3 * H * Fs + 2.0 * T * H * E,
    }


def flush_l2(flush):
    """Evict L2 before a timed step: write a 256 MiB buffer (> the 126 MB L2), then
    read a second one so the dirty zero lines are written back to HBM here, outside
    the timed events, instead of being evicted (written back) by the timed step."""
    import torch
    buf_w, buf_r, sink = flush
    buf_w.zero_()
    torch.sum(buf_r, 0, out=sink)


def timed_steps(layer, xs, y, steps, warmup, flush, profile=True):
    """Per-step CUDA-event times (ms) and per-stage ms; xs: list of inputs cycled."""
    import torch
    st = torch.cuda.current_stream()
    for i in range(warmup):
        layer.forward(xs[i % len(xs)], y=y)
    torch.cuda.synchronize()
    if profile:
        layer.profile(True)
    times, stages = [], {}
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for i in range(steps):
        flush_l2(flush)
        e0.record(st)
        layer.forward(xs[(warmup + i) % len(xs)], y=y)
        e1.record(st)
        e1.synchronize()
        times.append(e0.elapsed_time(e1))
        if profile:
            for k, v in layer.stage_times().items():
                stages.setdefault(k, []).append(v)
    if profile:
        layer.profile(False)
    return times, {k: sum(v) / len(v) for k, v in stages.items()}


def run_ours(args):
    import torch
    ws, rank, local = dist_setup()
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import build as b
    if rank == 0:
        b.build()
    barrier(ws)
    from inputs.presets import PRESETS
    from inputs.synthetic import make_tokens, make_weights
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
    peaks = load_peaks()
    p = PRESETS[args.config]
    T = args.tokens or p.prefill_tokens
    w = make_weights(p, "cuda")
    x, _ = make_tokens(p, T, "cuda", offset=rank)
    y = torch.empty_like(x)
    ep = ws > 1 and not args.replicas
    if ep:
        # expert parallelism over NCCL: rank r owns experts [r E/P, (r+1) E/P);
        # the router and the shared expert are replicated
        import torch.distributed as dist
        uid = [moe.get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        w = moe.slice_experts(w, rank, ws)
        torch.cuda.empty_cache()
        layer = moe.MoELayer(p, w, max_tokens=T, device=local, ep_rank=rank, ep_size=ws, unique_id=uid[0],
                             ep_fixed=args.ep_fixed)
    else:
        layer = moe.MoELayer(p, w, max_tokens=T, device=local)
    flush = (torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda"),
             torch.zeros(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda"),
             torch.zeros((), dtype=torch.float32, device="cuda"))
    info = layer.info()

    # ---------------- prefill, device-resident inputs ----------------
    barrier(ws)
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        times, stages = timed_steps(layer, [x], y, args.steps, args.warmup, flush, profile=not ep)
    torch.cuda.synchronize()
    barrier(ws)
    pinfo = layer.info()                 # kernel launches of the last (prefill) forward
    ms = max_over_ranks(sum(times) / len(times), ws)
    value = ws * T / (ms * 1e-3)

    # routing statistics of this batch (distinct experts hit, for the byte counts)
    if ep:
        n_distinct = p.n_experts // ws
    else:
        routing = {}
        layer.forward(x, y=y, routing=routing)
        counts = routing["expert_counts"].cpu()
        n_distinct = int((counts > 0).sum())
    alg = algorithmic(p, T, n_distinct)
    fp8 = p.wtype == 1
    # the prefill step is a few ms: the kernel runs at its burst clock, so the peak is the
    # burst figure (MEASURED_PEAKS.json bf16_tflops, FP8 = 2x, the nominal dtype ratio)
    tc_peak = (2.0 if fp8 else 1.0) * peaks["bf16_tflops"]
    if stages:
        dom = max((k for k in stages if k in alg), key=lambda k: stages[k])
        dom_ms = stages[dom]
    else:                      # expert parallel: whole-step rate of the routed FFN work on this rank
        dom, dom_ms = "layer_ep", ms
        alg[dom] = {"flops": alg["gemm1_swiglu"]["flops"] + alg["gemm2"]["flops"]}
    ach = alg[dom]["flops"] / (dom_ms * 1e-3) / 1e12
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tpath):
        traffic = json.load(open(tpath)).get(f"{p.name}:{T}:{dom}")
    layer_tflops = alg["layer_flops"] / (ms * 1e-3) / 1e12
    roofline = {"bound": "tensor", "kernel": dom, "achieved": ach, "peak": tc_peak, "unit": "TFLOP/s",
                "frac": ach / tc_peak, "traffic": traffic,
                "peak_source": f"{peaks['_source']}: bf16_tflops (burst) x {'2 (fp8/bf16 nominal ratio)' if fp8 else '1'}",
                "algorithmic": (f"2*T*(k*{'2F*H' if dom == 'gemm1_swiglu' else 'H*F'} + "
                                f"{'2Fs*H' if dom == 'gemm1_swiglu' else 'H*Fs'}) flops per launch (routed + shared "
                                f"expert operand groups), T={T}"),
                "kernel_ms": dom_ms,
                "layer": {"achieved": layer_tflops, "frac": layer_tflops / tc_peak,
                          "flops": alg["layer_flops"], "ms": ms},
                "stage_ms": {k: round(v, 4) for k, v in stages.items()}}

    # ---------------- decode, T = 1: a chain of distinct layers ----------------
    # The decode step is one CUDA graph replay over a stack of `--decode-layers`
    # distinct layer instances chained like consecutive model layers
    # (x_{i+1} = y_i = x_i + moe_i(x_i)); weights of the stack (8 x 11.3 GB for V3)
    # dwarf L2, and L2 is also flushed before every replay (outside the events).
    # value = replay time / layers.  The API is host-sync-free and capturable
    # (PAPER.md L193 captures the decode step in one CUDA graph).  Variants:
    #   deferral: the same chain with Expert Deferral across layers (moe_layer_forward_chained,
    #             PAPER.md L241; n_def = 3, the paper's BF16 setting L257; last layer 0)
    #   tp_rank:  one expert-TP rank's share (its 1/P slice of every expert, P = 2/4/8) --
    #             the all-reduce of the partials needs the other GPUs and is not in it
    #   tp_nccl:  N > 1 only: the expert-TP chain over the N GPUs, NCCL fp32 all-reduce inside
    decode = None
    if not args.no_decode and (not ep or not args.no_decode_tp_nccl):
        nl = max(1, args.decode_layers)
        xd, _ = make_tokens(p, args.steps + args.warmup, "cuda", offset=1000 + rank)
        rows = [xd[i:i + 1].contiguous() for i in range(xd.shape[0])]
        st = torch.cuda.current_stream()

        def time_chain(dlayers, n_def=0, chained=False, cyclic=False):
            # cyclic (chained only): every layer defers and layer 0 takes the last layer's deferred
            # experts of the previous replay -- a deep stack's steady state, without the two end
            # layers of a finite chain (the first streams 5 experts, the last 8 + 3)
            bufs = [rows[0].clone(), torch.empty_like(rows[0])]
            first = [True]

            def dstep():
                prev = dlayers[-1] if (cyclic and not first[0]) else None
                for i, l in enumerate(dlayers):
                    a_, b_ = bufs[i % 2], bufs[(i + 1) % 2]
                    if chained:
                        nd = n_def if (cyclic or i < len(dlayers) - 1) else 0
                        l.forward_chained(a_, residual=a_, n_deferred=nd, prev=prev, y=b_)
                        prev = l
                    else:
                        l.forward(a_, residual=a_, y=b_)
                first[0] = False

            side = torch.cuda.Stream()
            side.wait_stream(torch.cuda.current_stream())
            with torch.cuda.stream(side):
                for _ in range(2):
                    bufs[0].copy_(rows[0])
                    dstep()
            torch.cuda.current_stream().wait_stream(side)
            graph = torch.cuda.CUDAGraph()
            with torch.cuda.graph(graph):
                dstep()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            for i in range(args.warmup):
                bufs[0].copy_(rows[i])
                graph.replay()
            torch.cuda.synchronize()
            barrier(ws)
            tt = []
            for i in range(args.steps):
                bufs[0].copy_(rows[args.warmup + i])
                flush_l2(flush)
                barrier(ws)
                e0.record(st)
                graph.replay()
                e1.record(st)
                e1.synchronize()
                tt.append(e0.elapsed_time(e1) / len(dlayers))
            del graph
            return max_over_ranks(sum(tt) / len(tt), ws) * 1e3

        algd = algorithmic(p, 1, p.top_k)
        hbm = lambda us: {"bound": "hbm", "achieved": algd["layer_bytes"] / (us * 1e-6) / 1e9,
                          "peak": peaks["hbm_gbs"], "unit": "GB/s",
                          "frac": algd["layer_bytes"] / (us * 1e-6) / 1e9 / peaks["hbm_gbs"],
                          "bytes": algd["layer_bytes"]}
        if not ep:
            dlayers = [layer] + [moe.MoELayer(p, w, max_tokens=16, device=local) for _ in range(nl - 1)]
            dus = time_chain(dlayers)
            _, dstages = timed_steps(layer, rows, torch.empty_like(rows[0]), min(args.steps, 5), 1, flush)
            dinfo = layer.info()
            decode = {"us_per_layer": dus, "tokens": 1, "layers_in_graph": nl, "mode": "cuda_graph_replay",
                      "gpu_launches_per_layer": dinfo.kernels_per_forward_decode, "roofline": hbm(dus)}
            decode["roofline"]["stage_us_eager"] = {k: round(v * 1e3, 2) for k, v in dstages.items()}
            if not args.no_deferral and p.top_k > 3:
                dd = time_chain(dlayers, n_def=3, chained=True)
                dc = time_chain(dlayers, n_def=3, chained=True, cyclic=True)
                decode["deferral"] = {"n_deferred": 3, "us_per_layer": dd, "speedup_vs_no_deferral": dus / dd,
                                      "roofline": hbm(dd),
                                      "mode": "moe_layer_forward_chained: layer i streams layer i-1's deferred "
                                              "experts while its own router runs (PAPER.md L241); finite chain, "
                                              "last layer n_def = 0",
                                      "steady_state": {"us_per_layer": dc, "speedup_vs_no_deferral": dus / dc,
                                                       "roofline": hbm(dc),
                                                       "mode": "cyclic chain: every layer defers, layer 0 takes "
                                                               "the last layer's deferred experts of the previous "
                                                               "replay (same bytes per layer as plain)"}}
            for l in dlayers[1:]:
                l.close()
            del dlayers
            torch.cuda.empty_cache()
            # expert TP: one rank's share (rank 0's slice of every expert as a layer of its own)
            tp = {}
            if not args.no_decode_tp:
                for P in (2, 4, 8):
                    if p.ffn // 128 < P or (p.shared_ffn and p.shared_ffn // 128 < P):
                        continue
                    ws0 = moe.slice_tp(w, 0, P, p.ffn, p.shared_ffn)
                    p0 = p.with_(ffn=ws0.w2.shape[2], shared_ffn=ws0.ws2.shape[1] if p.shared_ffn else 0)
                    tl = [moe.MoELayer(p0, ws0, max_tokens=16, device=local) for _ in range(nl)]
                    tp[str(P)] = round(time_chain(tl), 2)
                    for l in tl:
                        l.close()
                    del tl, ws0
                    torch.cuda.empty_cache()
            decode["tp_rank_us_per_layer"] = tp
        elif p.ffn // 128 >= ws and (not p.shared_ffn or p.shared_ffn // 128 >= ws):
            # expert TP over the N GPUs of this run (NCCL all-reduce in the graph)
            import torch.distributed as dist
            tl = []
            try:
                wr = moe.slice_tp(make_weights(p, "cuda"), rank, ws, p.ffn, p.shared_ffn)
                for _ in range(nl):
                    uid = [moe.get_unique_id() if rank == 0 else None]
                    dist.broadcast_object_list(uid, src=0)
                    tl.append(moe.MoELayer(p, wr, max_tokens=16, device=local, tp_rank=rank, tp_size=ws,
                                           unique_id=uid[0]))
                del wr
                dus = time_chain(tl)
                decode = {"tp_nccl_us_per_layer": dus, "tokens": 1, "layers_in_graph": nl, "tp": ws,
                          "mode": "cuda_graph_replay, expert TP over NCCL (fp32 all-reduce of the partials)",
                          "roofline": hbm(dus)}
            except Exception as ex:          # keep the prefill line even if this variant fails
                decode = {"tp_nccl_error": f"{type(ex).__name__}: {ex}"}
            for l in tl:
                l.close()
            torch.cuda.empty_cache()

    # ---------------- e2e through the public API, host buffers ----------------
    # Every step copies its inputs from pinned host memory and reads its output back
    # inside the timed region.  `value`: the steps pipelined the way a server runs
    # them -- H2D of step i+1 and D2H of step i-1 (two copy streams) overlap step i's
    # forward (double-buffered device tensors, event-ordered) -- total / steps.
    # `serial_ms_per_step`: each step alone (copy in, forward, copy out, then the next).
    e2e = None
    if not args.no_e2e and not ep:
        st = torch.cuda.current_stream()
        nb = 2
        xh0 = x.cpu().pin_memory()
        xh = [xh0] * args.steps                              # the same pinned input, copied every step
        yh = [torch.empty_like(xh0).pin_memory() for _ in range(nb)]
        xdev = [torch.empty_like(x) for _ in range(nb)]
        ydev = [torch.empty_like(x) for _ in range(nb)]
        s_in, s_out = torch.cuda.Stream(), torch.cuda.Stream()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        for i in range(args.warmup):
            xdev[0].copy_(xh[i % args.steps], non_blocking=True)
            layer.forward(xdev[0], y=ydev[0])
            yh[0].copy_(ydev[0], non_blocking=True)
        torch.cuda.synchronize()
        # serial: one step at a time
        et = []
        for i in range(args.steps):
            flush_l2(flush)
            e0.record(st)
            xdev[0].copy_(xh[i], non_blocking=True)
            layer.forward(xdev[0], y=ydev[0])
            yh[0].copy_(ydev[0], non_blocking=True)
            e1.record(st)
            e1.synchronize()
            et.append(e0.elapsed_time(e1))
        serial_ms = max_over_ranks(sum(et) / len(et), ws)
        # pipelined
        ev_in = [torch.cuda.Event() for _ in range(args.steps)]
        ev_fw = [torch.cuda.Event() for _ in range(args.steps)]
        ev_out = [torch.cuda.Event() for _ in range(args.steps)]
        flush_l2(flush)
        torch.cuda.synchronize()
        e0.record(st)
        s_in.wait_stream(st)
        s_out.wait_stream(st)
        for i in range(args.steps):
            b = i % nb
            with torch.cuda.stream(s_in):
                if i >= nb:
                    s_in.wait_event(ev_fw[i - nb])          # xdev[b] no longer read by step i-nb
                xdev[b].copy_(xh[i], non_blocking=True)
                ev_in[i].record(s_in)
            st.wait_event(ev_in[i])
            if i >= nb:
                st.wait_event(ev_out[i - nb])               # ydev[b] read back by step i-nb
            layer.forward(xdev[b], y=ydev[b], stream=st)
            ev_fw[i].record(st)
            with torch.cuda.stream(s_out):
                s_out.wait_event(ev_fw[i])
                yh[b].copy_(ydev[b], non_blocking=True)
                ev_out[i].record(s_out)
        st.wait_stream(s_out)
        e1.record(st)
        e1.synchronize()
        ems = max_over_ranks(e0.elapsed_time(e1) / args.steps, ws)
        ref = layer.forward(xdev[(args.steps - 1) % nb].copy_(xh[-1]))   # the last step's output, recomputed
        torch.cuda.synchronize()
        assert torch.equal(ref.cpu(), yh[(args.steps - 1) % nb]), "pipelined e2e read back a stale output"
        e2e = {"value": ws * T / (ems * 1e-3), "unit": "tokens/s", "h2d_bytes_per_step": int(x.numel() * 2),
               "d2h_bytes_per_step": int(y.numel() * 2), "ms_per_step": ems, "mode": "pipelined (H2D / forward / D2H "
               "on three streams, double-buffered)", "serial_ms_per_step": serial_ms,
               "serial_value": ws * T / (serial_ms * 1e-3)}

    # ---------------- CPU oracle on a bounded sample (rank 0, N = 1) ----------------
    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu:
        nt = min(args.cpu_tokens, T)
        v, nexp, dt = oracle_layer_call(p, w, x[:nt])
        cpu = {"value": v, "unit": "tokens/s", "cores": cpu_cores(), "cpu_model": cpu_model(), "kind": "oracle",
               "sample": f"one full-layer oracle call (oracle.moe_layer) on the first {nt} tokens of the same "
                         f"batch: {nexp} distinct experts, each dequantised once in the call; {dt:.1f} s, fp64 "
                         "numpy, BLAS threads = the host cores"}

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "tokens/s", "n_gpus": ws, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
                "vs_baseline": None, "dtype": "e4m3" if fp8 else "bf16", "data": "synthetic",
                "config": dict(prefill_config(p, T, (f"ep{ws} (NCCL " + (
                    "fixed-capacity all-to-all, no host sync" if args.ep_fixed else "all-to-all-v, counts via the host")
                    + " dispatch/combine)" if ep else f"replica x{ws}") if ws > 1 else "single"),
                    l2="flushed before every step (256 MiB write, then 256 MiB read so the dirty lines are written "
                       "back before the events, outside the timed events); inputs resident in HBM",
                    distinct_experts_hit=n_distinct),
                "layer_tflops": layer_tflops,
                "roofline": roofline, "decode": decode, "e2e": e2e, "cpu_baseline": cpu,
                "gpu_launches": pinfo.kernels_per_forward_prefill * args.steps,
                "clocks": clk.summary()}
        print(json.dumps(line), flush=True)
    layer.close()
    if ws > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="v3")
    ap.add_argument("--tokens", type=int, default=0)
    ap.add_argument("--no-decode", action="store_true")
    ap.add_argument("--no-decode-tp", action="store_true", help="skip the decode-TP per-rank timing")
    ap.add_argument("--no-deferral", action="store_true", help="skip the chained Expert Deferral decode timing")
    ap.add_argument("--no-decode-tp-nccl", action="store_true", help="N > 1: skip the decode timing with expert TP over NCCL")
    ap.add_argument("--decode-layers", type=int, default=8, help="distinct layers chained in the decode graph")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-tokens", type=int, default=16, help="tokens of the cpu_baseline oracle call")
    ap.add_argument("--ref-tokens", type=int, default=8, help="--impl reference: tokens per step (oracle call)")
    ap.add_argument("--replicas", action="store_true", help="N>1: independent replicas instead of expert parallel")
    ap.add_argument("--ep-fixed", action="store_true",
                    help="N>1: fixed-capacity EP exchange (no host sync, capturable; more bytes on the wire)")
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "ours":
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
        return
    ws = os.environ.get("WORLD_SIZE")
    if args.gpus > 1 and ws is None:
        # one process per GPU: re-execute under torchrun (the driver launches it that way itself)
        import torch
        n = torch.cuda.device_count()
        if n < args.gpus:
            print(f"bench.py: --gpus {args.gpus} needs {args.gpus} visible GPUs, found {n}", file=sys.stderr)
            sys.exit(2)
        import socket
        with socket.socket() as sk:
            sk.bind(("127.0.0.1", 0))
            port = sk.getsockname()[1]
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
        sys.exit(subprocess.call(cmd))
    if ws is not None and int(ws) != args.gpus:
        print(f"bench.py: WORLD_SIZE={ws} but --gpus {args.gpus}", file=sys.stderr)
        sys.exit(2)
    if args.config == "all":
        for c in ("v3", "v25", "qwen2", "v2lite"):
            args.config = c
            run_ours(args)
        return
    run_ours(args)


if __name__ == "__main__":
    main()
