"""Digest of the state after n graph steps on a config (compare variants across processes).
usage: python tools/probe_digest.py CONFIG SCALE N [flags]"""
import hashlib, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_sc_xiangkfah23_b200 as ca
from synth import make_config

name, scale, n = sys.argv[1], float(sys.argv[2]), int(sys.argv[3])
flags = int(sys.argv[4], 0) if len(sys.argv) > 4 else 0
inst = make_config(name, scale=scale)
s = torch.cuda.Stream(); torch.cuda.set_stream(s)
h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, flags, stream=s)
h.run(n)
st = h.get_state()
for k in ("d", "yc", "zc", "yp", "zp", "Sp"):
    print(k, hashlib.sha1(np.ascontiguousarray(st[k]).tobytes()).hexdigest()[:16])
print("best", h.get_best(with_mate=False)[1]["best_score"])
