import sys, numpy as np, torch
sys.path.insert(0, '.')
from inputs.presets import SMALL
from inputs.synthetic import make_tokens, make_weights
from oracle import moe_oracle as O
from tests.parity import oracle_cfg, oracle_weights, rel_l2
from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
import itertools
for name, Ts in itertools.product(("v3_s",), ([3, 5], [5, 3], [5, 5], [3, 3], [1, 5])):
    p = SMALL[name]
    w = make_weights(p, "cpu")
    g = moe.MoEGroup(p, w.to("cuda"), ep_size=2, max_tokens=5)
    xs = [make_tokens(p, t, "cpu", offset=r)[0] for r, t in enumerate(Ts)]
    ys = g.forward([x.cuda() for x in xs]); torch.cuda.synchronize()
    cfg, W = oracle_cfg(p), oracle_weights(p, w)
    for x, y in zip(xs, ys):
        x64 = x.double().numpy()
        full = O.moe_layer(x64, W, cfg)["y"]
        sh = O.shared_expert(x64, W, cfg) if p.shared_ffn else 0 * full
        yy = y.float().cpu().numpy()
        print(name, Ts, "full", rel_l2(yy, full), "vs shared only", rel_l2(yy, sh), "vs routed only", rel_l2(yy, full - sh))
    g.close()
