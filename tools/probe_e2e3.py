"""e2e breakdown on config O: init / run_trace(n) / get_best, pipelined vs not
(CUALIGN_PIPELINE read once per process: run twice)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import paper_conf_sc_xiangkfah23_b200 as ca  # noqa: E402
from synth import make_config  # noqa: E402

inst = make_config("O", scale=float(sys.argv[1]) if len(sys.argv) > 1 else 1.0)


def pin(x):
    return torch.from_numpy(np.ascontiguousarray(x)).pin_memory()


class G:
    pass


GA, GB, GL = G(), G(), G()
GA.n, GA.rowptr, GA.col = inst.A.n, pin(inst.A.rowptr), pin(inst.A.col)
GB.n, GB.rowptr, GB.col = inst.B.n, pin(inst.B.rowptr), pin(inst.B.col)
GL.a, GL.b, GL.w = pin(inst.L.a), pin(inst.L.b), pin(inst.L.w)
stream = torch.cuda.Stream()
torch.cuda.set_stream(stream)
for rep in range(3):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    h = ca.CuAlignBP(GA, GB, GL, inst.alpha, inst.beta, inst.gamma, stream=stream)
    t1 = time.perf_counter()
    h.run_trace(2)
    t2 = time.perf_counter()
    h.run_trace(98)
    t3 = time.perf_counter()
    mate, info = h.get_best()
    t4 = time.perf_counter()
    h.close()
    print(f"rep {rep}: init {1e3*(t1-t0):.1f} ms, first 2 steps {1e3*(t2-t1):.1f} ms, 98 steps {1e3*(t3-t2):.1f} ms "
          f"({1e3*(t3-t2)/98:.3f} ms/step), best {1e3*(t4-t3):.1f} ms, total {1e3*(t4-t0):.1f} ms", flush=True)
