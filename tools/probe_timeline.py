"""Kernel timeline (CUPTI activity through torch.profiler: start, end,
stream of every kernel, CUDA-graph kernels included) of a few steps of
config O after --pre steps, to see the step's critical path.
    python tools/probe_timeline.py [--pre 10] [--n 3] [--schedule 0]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--pre", type=int, default=10)
    ap.add_argument("--n", type=int, default=3)
    ap.add_argument("--schedule", type=int, default=0)
    ap.add_argument("--config", default="O")
    args = ap.parse_args()
    import torch
    from torch.profiler import profile, ProfilerActivity
    import paper_conf_sc_xiangkfah23_b200 as ca
    from synth import make_config
    inst = make_config(args.config)
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=s, schedule=args.schedule)
    h.run(args.pre)
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        h.run(args.n)
        torch.cuda.synchronize()
    rows = []
    for ev in prof.events():
        if ev.device_type.name != "CUDA":
            continue
        nm = ev.name.replace("(anonymous namespace)::", "").replace("cualign::", "").replace("void ", "")
        nm = nm.split("(")[0][:48]
        rows.append((ev.time_range.start, ev.time_range.end, nm, getattr(ev, "device_resource_id", None)))
    rows.sort()
    t0 = rows[0][0] if rows else 0
    out = [{"t0_us": round(a - t0, 1), "t1_us": round(b - t0, 1), "dur_us": round(b - a, 1), "kernel": n,
            "stream": st} for a, b, n, st in rows]
    print(json.dumps({"schedule": h.sizes()["schedule"], "steps": args.n, "kernels": out}, indent=0))


if __name__ == "__main__":
    main()
