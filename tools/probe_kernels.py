"""Per-kernel device durations of the step's kernels in situ (CUPTI activity
through torch.profiler; kernels inside CUDA graphs included), config O at a
fixed state:  round-only, iterate-only and full-step graph replays.
    python tools/probe_kernels.py [--pre 80] [--n 20] [--config O]"""
import argparse
import json
import os
import sys
from collections import defaultdict

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--pre", type=int, default=80)
    ap.add_argument("--n", type=int, default=20)
    ap.add_argument("--config", default="O")
    ap.add_argument("--k", type=int, default=None)
    args = ap.parse_args()
    import torch
    from torch.profiler import profile, ProfilerActivity
    import paper_conf_sc_xiangkfah23_b200 as ca
    from synth import make_config
    inst = make_config(args.config, k=args.k)
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=s)
    h.run(args.pre)
    torch.cuda.synchronize()
    out = {}
    for name, kw in (("round", dict(with_round=True, iterate=False)), ("iterate", dict(with_round=False)),
                     ("step", dict())):
        h.run(3, **kw)
        torch.cuda.synchronize()
        with profile(activities=[ProfilerActivity.CUDA]) as prof:
            h.run(args.n, **kw)
            torch.cuda.synchronize()
        agg = defaultdict(lambda: [0, 0.0])
        t0, t1 = None, None
        for ev in prof.events():
            if ev.device_type.name != "CUDA":
                continue
            nm = ev.name.replace("(anonymous namespace)::", "").replace("cualign::", "").replace("void ", "")
            nm = nm.split("(")[0][:60]
            agg[nm][0] += 1
            agg[nm][1] += ev.device_time_total if hasattr(ev, "device_time_total") else ev.cuda_time_total
        out[name] = {k: {"n_per_step": v[0] / args.n, "us_per_step": v[1] / args.n} for k, v in
                     sorted(agg.items(), key=lambda x: -x[1][1])}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
