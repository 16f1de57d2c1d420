"""Step time of each step schedule (cualign_params.schedule: 1 pipelined,
2 serial, 3 forked) on the BASELINE configs: one handle per schedule, 40
warm steps, then --n device-timed steps on the launching stream.
    python tools/probe_schedules.py [--points O,P,T] [--n 100]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--points", default="O,P,T,S,R5,R50")
    ap.add_argument("--n", type=int, default=100)
    args = ap.parse_args()
    import torch
    import paper_conf_sc_xiangkfah23_b200 as ca
    from synth import make_config
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    for pt in args.points.split(","):
        name, k = pt[0], (int(pt[1:]) if len(pt) > 1 else None)
        inst = make_config(name, k=k)
        row = {"config": pt}
        for sched, label in ((1, "pipelined"), (2, "serial"), (3, "forked")):
            with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=s,
                              schedule=sched) as h:
                h.run(40)
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                h.run(args.n)
                e1.record(s)
                torch.cuda.synchronize()
                row[label] = e0.elapsed_time(e1) / args.n
            torch.cuda.empty_cache()
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
