"""Isolated per-kernel timing of the rounding on config O (no concurrent square):
after `warm` BP iterations, repeat round() with event timing on.
usage: python tools/probe_round.py [reps] [warm]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_sc_xiangkfah23_b200 as ca
from synth import make_config

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 20
warm = int(sys.argv[2]) if len(sys.argv) > 2 else 20
inst = make_config("O")
s = torch.cuda.Stream(); torch.cuda.set_stream(s)
h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=s)
h.run(warm, with_round=False)
for _ in range(3):
    h.round(sync=False)
torch.cuda.synchronize()
h.stats(reset=True)
h.set_timing(True)
for _ in range(reps):
    h.round(sync=False)
torch.cuda.synchronize()
h.set_timing(False)
st = h.stats(reset=True)
print({k: round(v / reps, 4) for k, v in st["class_ms"].items() if v}, os.environ.get("CUALIGN_SUITOR_PERSIST"),
      os.environ.get("CUALIGN_SUITOR_G"))
