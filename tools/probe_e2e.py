"""Break down the end-to-end align time (diagnostics)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_sc_xiangkfah23_b200 as ca
from synth import make_config

inst = make_config("O")
s = torch.cuda.Stream(); torch.cuda.set_stream(s)
def pin(x): return torch.from_numpy(np.ascontiguousarray(x)).pin_memory()
class G: pass
GA, GB, GL = G(), G(), G()
GA.n, GA.rowptr, GA.col = inst.A.n, pin(inst.A.rowptr), pin(inst.A.col)
GB.n, GB.rowptr, GB.col = inst.B.n, pin(inst.B.rowptr), pin(inst.B.col)
GL.a, GL.b, GL.w = pin(inst.L.a), pin(inst.L.b), pin(inst.L.w)
for rep in range(3):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    h = ca.CuAlignBP(GA, GB, GL, inst.alpha, inst.beta, inst.gamma, stream=s)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    h.run(1); h.get_best(with_mate=False)
    t2 = time.perf_counter()
    for _ in range(99):
        h.run(1); h.get_best(with_mate=False)
    t3 = time.perf_counter()
    m, info = h.get_best()
    t4 = time.perf_counter()
    h.close()
    print(f"rep {rep}: init {t1-t0:.4f}s first-step(capture) {t2-t1:.4f}s 99 steps {t3-t2:.4f}s ({(t3-t2)/99*1e3:.3f} ms/step) best {t4-t3:.4f}s total {t4-t0:.4f}s")
