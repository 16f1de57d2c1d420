"""Per-step device time and round work over the first iterations of config
O (events around each graph step), to see how the step cost evolves with p.
    python tools/probe_steps.py [--n 120]"""
import argparse, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=120)
    ap.add_argument("--config", default="O")
    args = ap.parse_args()
    import torch
    import paper_conf_sc_xiangkfah23_b200 as ca
    from synth import make_config
    inst = make_config(args.config)
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=s)
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(args.n + 1)]
    ev[0].record(s)
    for k in range(args.n):
        h.run(1)
        ev[k + 1].record(s)
    torch.cuda.synchronize()
    ms = [ev[k].elapsed_time(ev[k + 1]) for k in range(args.n)]
    # split of a few steps: iterate-only / round-only at fixed states
    out = {"ms_per_step": [round(x, 4) for x in ms]}
    h2 = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=s)
    split = []
    for p in range(1, args.n + 1):
        h2.set_timing(True)
        h2.run(1, with_round=False)
        torch.cuda.synchronize()
        it = h2.stats(reset=True)["class_ms"]
        h2.run(1, with_round=True, iterate=False)
        torch.cuda.synchronize()
        rd = h2.stats(reset=True)["class_ms"]
        info = h2.get_best(with_mate=False)[1]
        if p in (1, 2, 3, 5, 8, 12, 16, 20, 25, 30, 40, 60, 80, 100, 120):
            split.append({"p": p, "iter_ms": round(sum(it.values()), 4), "square": round(it.get("square", 0), 4),
                          "round_ms": round(sum(rd.values()), 4), "match": round(rd.get("match", 0), 4),
                          "eval": round(rd.get("eval", 0), 4), "rounds_y": info["rounds_y"], "rounds_z": info["rounds_z"],
                          "card_y": info["card_y"], "card_z": info["card_z"]})
    out["split"] = split
    print(json.dumps(out))


if __name__ == "__main__":
    main()
