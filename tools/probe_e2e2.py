"""Mimic bench.py's sequence to find where e2e time goes (diagnostics)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_sc_xiangkfah23_b200 as ca
from synth import make_config

FLAGS = int(sys.argv[1], 0) if len(sys.argv) > 1 else 0
inst = make_config("O")
s = torch.cuda.Stream(); torch.cuda.set_stream(s)
t = time.perf_counter()
h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, FLAGS, stream=s)
torch.cuda.synchronize(); print("first init", time.perf_counter() - t)
h.run(10); torch.cuda.synchronize()
h.run(300); torch.cuda.synchronize()
h.set_timing(True); h.run(20); h.set_timing(False); torch.cuda.synchronize(); h.stats(reset=True)
def pin(x): return torch.from_numpy(np.ascontiguousarray(x)).pin_memory()
class G: pass
GA, GB, GL = G(), G(), G()
GA.n, GA.rowptr, GA.col = inst.A.n, pin(inst.A.rowptr), pin(inst.A.col)
GB.n, GB.rowptr, GB.col = inst.B.n, pin(inst.B.rowptr), pin(inst.B.col)
GL.a, GL.b, GL.w = pin(inst.L.a), pin(inst.L.b), pin(inst.L.w)
t = time.perf_counter(); del h; torch.cuda.synchronize(); print("del", time.perf_counter() - t)
t = time.perf_counter(); torch.cuda.empty_cache(); print("empty_cache", time.perf_counter() - t)
for rep in range(3):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    h2 = ca.CuAlignBP(GA, GB, GL, inst.alpha, inst.beta, inst.gamma, FLAGS, stream=s)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    for _ in range(100):
        h2.run(1); h2.get_best(with_mate=False)
    t2 = time.perf_counter()
    h2.get_best()
    h2.close()
    t3 = time.perf_counter()
    print(f"rep {rep}: init {t1-t0:.3f} steps {t2-t1:.3f} close {t3-t2:.3f}")
