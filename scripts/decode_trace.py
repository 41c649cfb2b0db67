"""Device timeline of one decode forward (MOE_DEBUG_TRACE=1 set by this script):
route kernel phases, per-CTA fused-kernel unit phases, finalize (globaltimer ns)."""
import os, sys, ctypes
os.environ["MOE_DEBUG_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from inputs.presets import PRESETS
from inputs.synthetic import make_tokens, make_weights
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
cfg = sys.argv[1] if len(sys.argv) > 1 else "v3"
T = int(sys.argv[2]) if len(sys.argv) > 2 else 1
p = PRESETS[cfg]
w = make_weights(p, "cuda")
x, _ = make_tokens(p, T, "cuda", offset=5)
NL = int(sys.argv[3]) if len(sys.argv) > 3 else 1     # >1: trace the middle layer of a chained graph
TP = int(sys.argv[4]) if len(sys.argv) > 4 else 1     # >1: expert TP, rank 0's slice as a layer of its own
NDEF = int(sys.argv[5]) if len(sys.argv) > 5 else 0   # >0: chained Expert Deferral (moe_layer_forward_chained)
if TP > 1:
    w = moe.slice_tp(w, 0, TP, p.ffn, p.shared_ffn)
    p = p.with_(ffn=w.w2.shape[2], shared_ffn=w.ws2.shape[1] if p.shared_ffn else 0)
layers = [moe.MoELayer(p, w, max_tokens=16) for _ in range(NL)]
layer = layers[NL // 2]
lib = layer._lib
buf = np.zeros(4096, dtype=np.uint64)
y = torch.empty_like(x)
fw = torch.empty(64 << 20, device="cuda"); fr = torch.zeros(64 << 20, device="cuda"); sink = torch.zeros((), device="cuda")
bufs = [x.clone(), torch.empty_like(x)]
def step():
    prev = None
    for i, l in enumerate(layers):
        a, b = bufs[i % 2], bufs[(i + 1) % 2]
        if NDEF:
            l.forward_chained(a, residual=a, n_deferred=NDEF if i < len(layers) - 1 else 0, prev=prev, y=b)
            prev = l
        else:
            l.forward(a, residual=a, y=b)
if NL > 1:
    s_ = torch.cuda.Stream(); s_.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s_):
        step(); step()
    torch.cuda.current_stream().wait_stream(s_)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        step()
allb = [np.zeros(4096, dtype=np.uint64) for _ in layers]
for it in range(4):
    fw.zero_(); torch.sum(fr, 0, out=sink)
    if NL > 1:
        bufs[0].copy_(x); g.replay()
    else:
        layer.forward(x, y=y)
    torch.cuda.synchronize()
    for l, b in zip(layers, allb):
        assert lib.moe_layer_debug_trace(l._h, b.ctypes.data, 4096) == 0
buf = allb[NL // 2]
if NL > 1:
    # the chain's period: route entry of every layer, its finalize end, and the gap to the next layer
    base = int(allb[0][0])
    ent = [(int(b[0]) - base) / 1e3 for b in allb]
    fin = [(int(b[2001]) - base) / 1e3 for b in allb]
    print("chain: route entry / finalize end per layer (us):",
          " ".join(f"{e:.1f}/{f:.1f}" for e, f in zip(ent, fin)))
    print("chain: period per layer (route entry to next route entry):",
          " ".join(f"{ent[i + 1] - ent[i]:.1f}" for i in range(NL - 1)),
          "| finalize end -> next route entry:", " ".join(f"{ent[i + 1] - fin[i]:.1f}" for i in range(NL - 1)))
t0 = int(buf[0])
rel = lambda v: (int(v) - t0) / 1e3
if buf[6]:
    print(f"route select cycles: first pass {int(buf[5])}, warm second pass {int(buf[6])}")
if buf[1900]:
    print("route one-token select (us): scores " + " ".join(f"{rel(buf[1900 + i]):.2f}" for i in range(4)) +
          "  (scores, groups, candidates, merged)")
print(f"route: entry 0, tail start {rel(buf[1]):.1f}, select done {rel(buf[2]):.1f}, permute done {rel(buf[3]):.1f}, end {rel(buf[4]):.1f} us")
cta = buf[8:8 + 8 * 148].reshape(148, 8).astype(np.int64)
act = cta[cta[:, 5] > 0]
def st(v):
    v = np.sort(v); return f"min {v[0]:6.1f} med {v[len(v)//2]:6.1f} max {v[-1]:6.1f}"
print("fused CTAs with a unit:", len(act))
for j, name in enumerate(["entry", "past_pdl", "unit", "accA", "h_ready", "unit_end"]):
    print(f"  {name:9s}", st((act[:, j] - t0) / 1e3))
print("  phaseA", st((act[:, 3] - act[:, 2]) / 1e3), " epiA", st((act[:, 4] - act[:, 3]) / 1e3),
      " phaseB", st((act[:, 5] - act[:, 4]) / 1e3))
sh = act[(act[:, 6] >> 30) == 1]
if len(sh):
    print("  shared units end", st((sh[:, 5] - t0) / 1e3))
order = np.argsort(act[:, 5])[::-1][:8]
for i in order:
    u = act[i]
    print(f"  slowest: sm {u[7]:3d} grp {u[6] >> 30} exp {(u[6] >> 16) & 0x3fff:3d} chunk {u[6] & 0xffff:2d} unit {(u[2]-t0)/1e3:6.1f} accA {(u[3]-t0)/1e3:6.1f} h {(u[4]-t0)/1e3:6.1f} end {(u[5]-t0)/1e3:6.1f}")
print(f"finalize: past pdl {rel(buf[2000]):.1f}, end {rel(buf[2001]):.1f} us")
lead = buf[1300:1300 + 4 * 148].reshape(148, 4).astype(np.int64)
ld = lead[lead[:, 0] > 0]
if len(ld):
    acc = cta[:, 3]
    print("cluster leaders (us): partials in " + st(np.array([rel(v) for v in ld[:, 0]])) +
          " | summed " + st(np.array([rel(v) for v in ld[:, 1]])) + " | swiglu " + st(np.array([rel(v) for v in ld[:, 2]])) +
          " | pushed " + st(np.array([rel(v) for v in ld[:, 3]])))
gq = buf[2100:2100 + 8 * 148].reshape(148, 8).astype(np.int64)
gq = gq[gq[:, 0] > 0]
if len(gq):
    for w in range(2):
        g4 = gq[:, 4 * w:4 * w + 4]
        print(f"leader gate warp {w} (us): exchanged " + st(np.array([rel(v) for v in g4[:, 0]])) + " | h " +
              st(np.array([rel(v) for v in g4[:, 1]])) + " | amax " + st(np.array([rel(v) for v in g4[:, 2]])) +
              " | quant " + st(np.array([rel(v) for v in g4[:, 3]])))
