"""NEXT-4 density sweep (synthetic analog of the paper's Figs. 4-5,
PAPER.md:331-339): quality (NCV-GS^3 etc. against the ground truth) and run
time as the candidate graph L gets denser.

Workload: config P's generator (Chung-Lu power-law A, B = P(A) with 5 % edge
noise, honest kNN candidates from structural features) at n = 4000 (the size
of the paper's Synthetic_4000, Table 1), k candidates per A vertex for each k
in --ks; density = k / n_B (the paper's "density = 100 - sparsity").  Each
point: align() for --iters iterations (GPU, C ABI), then the quality of the
best alignment (cualign_quality_eval) and the per-iteration time of a timed
graph replay.  Writes one JSON object per point to --out.

usage: python tools/density_sweep.py [--n 4000] [--ks 2,5,10,20,40,100,200] [--iters 100] [--out FILE]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=4000)
    ap.add_argument("--ks", default="2,5,10,20,40,100,200")
    ap.add_argument("--iters", type=int, default=100)
    ap.add_argument("--out", default="gpurun_out/density_sweep.jsonl")
    args = ap.parse_args()
    import torch
    import paper_conf_sc_xiangkfah23_b200 as ca
    from synth import make_config

    os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    rows = []
    for k in [int(x) for x in args.ks.split(",")]:
        inst = make_config("P", scale=args.n / 10_000, k=k)
        truth = np.asarray(inst.truth, dtype=np.int32)
        t0 = time.perf_counter()
        mate, info, _ = ca.align(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma,
                                 n_iter=args.iters, stream=stream)
        t_align = info["t_result"] - t0
        q = ca.quality(inst.A, inst.B, ca.alignment_map(mate, inst.L), truth)
        with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=stream) as h:
            h.run(5)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            h.run(args.iters)
            e1.record(stream)
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1) / args.iters
            sz = h.sizes()
        row = dict(n_a=inst.A.n, n_b=inst.B.n, edges_a=q["edges_a"], k=k, density=k / inst.B.n,
                   m=sz["m"], s=sz["s"], iters=args.iters, ms_per_iter=ms, align_s=t_align,
                   best_score=info["best_score"], best_iter=info["best_iter"],
                   **{key: q[key] for key in ("nc", "ec", "ics", "s3", "ncv", "ncv_gs3", "conserved", "aligned")})
        rows.append(row)
        print(json.dumps(row), flush=True)
    with open(args.out, "w") as fh:
        for r in rows:
            fh.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
