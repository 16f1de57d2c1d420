"""Suitor diagnostics on config O (probe build: CUALIGN_LIB=.../libcualign_bp_probes.so
CUALIGN_MATCH_DEBUG=1 prints per-launch scan statistics to stderr).
    python tools/probe_suitor.py [--pre 80]"""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_sc_xiangkfah23_b200 as ca
from synth import make_config

ap = argparse.ArgumentParser()
ap.add_argument("--pre", type=int, default=80)
args = ap.parse_args()
inst = make_config("O")
s = torch.cuda.Stream(); torch.cuda.set_stream(s)
h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=s)
h.run(args.pre)
for rep in range(3):
    r = h.round()
    torch.cuda.synchronize()
    print("round", {k: r[k] for k in ("card_y", "card_z", "rounds_y", "rounds_z")}, flush=True)
st = h.get_state(with_S=False)
for k in ("yc", "zc"):
    x = st[k]
    print(k, "frac x>0", float(np.mean(x > 0)), "distinct", len(np.unique(x)))
