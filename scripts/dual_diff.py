"""Debug: the same forward with and without dual units (MOE_SWAP_DUAL read at create), rows compared."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from inputs.presets import PRESETS
from inputs.synthetic import make_tokens, make_weights
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
cfg = sys.argv[1] if len(sys.argv) > 1 else "qwen2"
T = int(sys.argv[2]) if len(sys.argv) > 2 else 2048
p = PRESETS[cfg]
w = make_weights(p, "cuda")
x, _ = make_tokens(p, T, "cuda")
outs = {}
for d in ("0", "1"):
    os.environ["MOE_SWAP_DUAL"] = d
    l = moe.MoELayer(p, w, max_tokens=T)
    r = {}
    outs[d] = (l.forward(x, routing=r).float(), r)
    torch.cuda.synchronize()
    l.close()
y0, r0 = outs["0"]; y1, r1 = outs["1"]
err = ((y1 - y0).norm(dim=1) / y0.norm(dim=1).clamp_min(1e-6)).cpu()
print("rows with rel err > 1e-2:", int((err > 1e-2).sum()), "of", T, " max", float(err.max()))
idx = r0["topk_idx"].cpu()
cnt = r0["expert_counts"].cpu()
bad = (err > 1e-2).nonzero().flatten()[:2000]
from collections import Counter
# per-expert: rank of each bad token within the expert's segment
pos = {}
for e in range(p.n_experts):
    toks = (idx == e).any(dim=1).nonzero().flatten().tolist()
    for i, t in enumerate(toks):
        pos.setdefault(t, []).append((e, i, int(cnt[e])))
c = Counter()
for t in bad.tolist():
    for e, i, n in pos.get(t, []):
        c[("rank>=256" if i >= 256 else "rank<256", "n>256" if n > 256 else "n<=256")] += 1
print(c.most_common())
print("experts with n > 256:", int((cnt > 256).sum()), " max count", int(cnt.max()))
