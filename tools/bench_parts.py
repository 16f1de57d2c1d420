"""Per-part timing at a FIXED BP state (diagnostics, not the bench contract).

Runs config O for --pre iterations (graph), then times N rounds alone and N
iterations alone, each with per-kernel event timing inside the captured graph.
    python tools/bench_parts.py [--pre 300] [--n 50]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--pre", type=int, default=300)
    ap.add_argument("--n", type=int, default=50)
    ap.add_argument("--config", default="O")
    ap.add_argument("--scale", type=float, default=1.0)
    args = ap.parse_args()
    import torch
    import paper_conf_sc_xiangkfah23_b200 as ca
    from synth import make_config
    inst = make_config(args.config, scale=args.scale)
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=s)
    h.run(args.pre)
    torch.cuda.synchronize()
    h.stats(reset=True)
    # rounds only, at the fixed state (graph replays, event nodes per kernel)
    h.set_timing(True)
    h.run(args.n, with_round=True, iterate=False)
    torch.cuda.synchronize()
    r = h.stats(reset=True)
    h.run(args.n, with_round=False)
    torch.cuda.synchronize()
    it = h.stats(reset=True)
    h.set_timing(False)
    out = {"round_ms": {k: v / args.n for k, v in r["class_ms"].items() if v},
           "iterate_ms": {k: v / args.n for k, v in it["class_ms"].items() if v},
           "last": h.get_best(with_mate=False)[1]}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
