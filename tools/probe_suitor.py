"""Suitor diagnostics on config O (CUALIGN_MATCH_DEBUG=1 prints per-launch scan stats)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_sc_xiangkfah23_b200 as ca
from synth import make_config

inst = make_config("O")
s = torch.cuda.Stream(); torch.cuda.set_stream(s)
h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=s)
for it in range(1, 31):
    h.iterate(1)
    if it in (1, 2, 5, 10, 20, 30):
        print("iter", it, flush=True)
        h.round()
        torch.cuda.synchronize()
st = h.get_state(with_S=False)
for k in ("yc", "zc"):
    x = st[k]
    print(k, "frac x>0", float(np.mean(x > 0)), "distinct", len(np.unique(x)))
