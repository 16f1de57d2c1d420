"""Init (a1-a2) timing on a config: first and second handle (pool warm),
with CUALIGN_INIT_TRACE phase lines on stderr.  Usage:
    python tools/probe_init.py [config] [scale] [k]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_sc_xiangkfah23_b200 as ca  # noqa: E402
from synth import make_config  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "O"
scale = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
k = int(sys.argv[3]) if len(sys.argv) > 3 else None
inst = make_config(cfg, scale=scale, k=k) if k else make_config(cfg, scale=scale)
torch.cuda.init()
for rep in range(3):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma)
    torch.cuda.synchronize()
    dt = time.perf_counter() - t0
    sz = h.sizes()
    print(f"{cfg} scale {scale} rep {rep}: init {dt*1e3:.1f} ms squares {sz['squares']} "
          f"({sz['squares']/dt/1e9:.2f} G squares/s incl. upload)", flush=True)
    h.close()
