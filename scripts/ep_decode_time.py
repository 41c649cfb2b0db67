"""Expert-parallel decode on one GPU (in-process group, every rank's kernels on this device):
the time of one group forward (all P ranks' work, serialised) for full-size layers, T tokens on
rank 0 and none elsewhere (batch-1 decode keeps its token on its owner).
MOE_EP_DECODE_GEMM=1 runs the expert side through the prefill grouped GEMMs instead of the
fused decode stream (A/B)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from inputs.presets import PRESETS
from inputs.synthetic import make_tokens, make_weights
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
cfg = sys.argv[1] if len(sys.argv) > 1 else "v3"
P = int(sys.argv[2]) if len(sys.argv) > 2 else 8
T = int(sys.argv[3]) if len(sys.argv) > 3 else 1
p = PRESETS[cfg]
w = make_weights(p, "cuda")
g = moe.MoEGroup(p, w, ep_size=P, max_tokens=max(T, 1))
del w
torch.cuda.empty_cache()
x, _ = make_tokens(p, T, "cuda")
xs = [x] + [x[:0] for _ in range(P - 1)]
ys = [torch.empty_like(t) for t in xs]
for _ in range(3):
    g.forward(xs, ys=ys) if "ys" in g.forward.__code__.co_varnames else g.forward(xs)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
ts = []
for _ in range(10):
    e0.record(); g.forward(xs); e1.record(); e1.synchronize()
    ts.append(e0.elapsed_time(e1) * 1e3)
ts.sort()
print(json.dumps({"config": cfg, "P": P, "T": T, "gemm_path": os.environ.get("MOE_EP_DECODE_GEMM") == "1",
                  "group_forward_us_median": ts[len(ts) // 2]}))
g.close()
