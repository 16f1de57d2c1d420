"""Single-GPU measurements of the large configs (BASELINE.json:configs[3..4]):

  S  social-shaped pair, n = 1e6 each, proxy k = 20 -> m = 2e7, s ~ 1e9
  R  R-MAT scale 20 (edge factor 8), proxy k in --ks: iteration time and
     matching time vs nnz(S) (the configs[4] sweep; 1 GPU here)

Each point: generate (seeded, synth/), init through the C ABI (L layouts +
S build, timed), --warm graph steps, then --n timed steps of the full step
graph (BP iteration + rounding) with CUDA events on the launching stream,
then --n iterate-only and --n round-only steps with per-kernel event nodes
(the split of the step).  One JSON object per point to stdout and --out.

usage: python tools/scale_sweep.py [--points S,R5,R10,R20,R35,R50] [--n 20]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

BYTES_PER_NZ, BYTES_PER_EDGE = 20, 80  # fp64 algorithmic bytes


def read_peak():
    try:
        with open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                               "MEASURED_PEAKS.json")) as fh:
            return float(json.load(fh)["hbm_gbs"])
    except Exception:
        return 6650.0


def point(name, k, args, stream, ca, make_config):
    import torch
    t0 = time.perf_counter()
    inst = make_config(name, k=k)
    t_gen = time.perf_counter() - t0
    row = dict(config=name, k=k, n_a=inst.A.n, n_b=inst.B.n, m=int(inst.L.m), gen_s=round(t_gen, 1))
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    try:
        h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=stream)
    except ca.CuAlignError as e:  # e.g. ENOMEM: reported, not fatal
        row["error"] = str(e)
        return row
    torch.cuda.synchronize()
    row["init_s"] = time.perf_counter() - t0
    with h:
        sz = h.sizes()
        s = int(sz["s"])
        row.update(s=s, squares=s // 2, device_gb=sz.get("device_bytes", 0) / 1e9)
        row["sbuild_squares_per_s"] = (s / 2) / row["init_s"]
        h.run(args.warm)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        h.run(args.n)
        e1.record(stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / args.n
        row.update(ms_per_step=ms, iters_per_s=1e3 / ms, squares_per_s=(s / 2) * 1e3 / ms)
        h.stats(reset=True)
        h.set_timing(True)
        h.run(args.n, with_round=False)
        torch.cuda.synchronize()
        it = h.stats(reset=True)["class_ms"]
        h.run(args.n, with_round=True, iterate=False)
        torch.cuda.synchronize()
        rd = h.stats(reset=True)["class_ms"]
        h.set_timing(False)
        it = {c: v / args.n for c, v in it.items() if v}
        rd = {c: v / args.n for c, v in rd.items() if v}
        bp_ms = sum(it.values())
        row.update(bp_ms=bp_ms, round_ms=sum(rd.values()), iterate_kernel_ms=it, round_kernel_ms=rd)
        alg = BYTES_PER_NZ * s + BYTES_PER_EDGE * row["m"]
        peak = read_peak()
        row["iteration_hbm_frac"] = alg / (bp_ms * 1e-3) / 1e9 / peak
        if it.get("square"):
            row["square_hbm_frac"] = BYTES_PER_NZ * s / (it["square"] * 1e-3) / 1e9 / peak
        best = h.get_best(with_mate=False)[1]
        row["best_score"] = best["best_score"]
    return row


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--points", default="S,R5,R10,R20,R35,R50")
    ap.add_argument("--n", type=int, default=20)
    ap.add_argument("--warm", type=int, default=21)  # >= 21: the schedule selection runs here
    ap.add_argument("--out", default="gpurun_out/scale_sweep.jsonl")
    args = ap.parse_args()
    import torch
    import paper_conf_sc_xiangkfah23_b200 as ca
    from synth import make_config
    os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    with open(args.out, "w") as fh:
        for p in args.points.split(","):
            name, k = p[0], (int(p[1:]) if len(p) > 1 else None)
            row = point(name, k, args, stream, ca, make_config)
            print(json.dumps(row), flush=True)
            fh.write(json.dumps(row) + "\n")
            fh.flush()


if __name__ == "__main__":
    main()
