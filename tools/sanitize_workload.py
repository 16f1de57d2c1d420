"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck):
config T through every schedule of the hand-rolled synchronisation -- the
square pass's bulk-copy / mbarrier ring, the last-arriver top-2 merge, the
Suitor CAS chains and slot reset, the step graphs (pipelined, serial, forked),
exact mode, the pointer-round matching, loopback shards -- plus the
standalone matching, quality and kNN entry points.
    compute-sanitizer --tool <tool> python tools/sanitize_workload.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import paper_conf_sc_xiangkfah23_b200 as ca
from synth import make_config


def main():
    inst = make_config("T")
    A, B, L = inst.A, inst.B, inst.L
    kw = dict(alpha=inst.alpha, beta=inst.beta, gamma=inst.gamma)
    for sched in (1, 2, 3):
        with ca.CuAlignBP(A, B, L, schedule=sched, **kw) as h:
            h.run(6)
            h.get_best()
    with ca.CuAlignBP(A, B, L, **kw) as h:
        h.run_trace(40)          # library's own schedule
        h.iterate(2)
        h.round()
        h.round_mates()
        h.sample_squares(np.arange(10, dtype=np.int32))
        st = h.get_state()
        h.set_state(st["yp"], st["zp"], st["Sp"], st["p"])
        h.iterate(1)
    for flags in (ca.FLAG_EXACT, ca.FLAG_MATCH_ROUNDS, ca.FLAG_ROUND_DAMPED | ca.FLAG_OTHERMAX_LITERAL, ca.FLAG_FP32_S):
        with ca.CuAlignBP(A, B, L, flags=flags, **kw) as h:
            h.run(4)
            h.iterate(1)
            h.round()
    with ca.CuAlignBP(A, B, L, world=3, **kw) as h:   # loopback shards (sharded rounding merge)
        h.run(4)
        h.get_best()
    ca.match(L, L.n_a, L.n_b, L.w)
    mate, _, _ = ca.align(A, B, L, n_iter=5)
    ca.quality(A, B, ca.alignment_map(mate, L), np.asarray(inst.truth, np.int32))
    rng = np.random.default_rng(0)
    ca.knn(rng.normal(size=(300, 64)).astype(np.float32), rng.normal(size=(700, 64)).astype(np.float32), 8)
    print("sanitize workload done")


if __name__ == "__main__":
    main()
