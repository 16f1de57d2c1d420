"""Phase timing of align() on config O (diagnostics): init, first step,
steady steps (run(1) + get_best), get_best with the matching."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_sc_xiangkfah23_b200 as ca
from synth import make_config

inst = make_config("O")
s = torch.cuda.Stream(); torch.cuda.set_stream(s)
for rep in range(2):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=s)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    h.run(1); h.get_best(with_mate=False)
    t2 = time.perf_counter()
    for _ in range(99):
        h.run(1); h.get_best(with_mate=False)
    t3 = time.perf_counter()
    h.run(20); torch.cuda.synchronize()
    t4 = time.perf_counter()
    mate, info = h.get_best()
    t5 = time.perf_counter()
    h.close()
    torch.cuda.synchronize(); t6 = time.perf_counter()
    print(f"rep {rep}: init {t1-t0:.4f} first {t2-t1:.4f} 99 steps {t3-t2:.4f} ({(t3-t2)/99*1e3:.3f} ms) "
          f"run(20) {(t4-t3)/20*1e3:.3f} ms/it get_best {t5-t4:.4f} close {t6-t5:.4f}", flush=True)
