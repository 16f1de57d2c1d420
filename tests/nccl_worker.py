"""One rank of a real NCCL sharded run on a single GPU.

`tests/test_gpu_nccl.py` starts `world` of these processes, all on cuda:0.
NCCL refuses two ranks on one device of one host ("Duplicate GPU"); a
distinct NCCL_HOSTID per rank (set by the launcher) makes each rank look like
its own host, so the communicator forms over NCCL's socket transport and every
collective of the sharded path (all-gather, grouped broadcasts / reduces,
all-reduces) runs through libnccl exactly as it does across B200s.  The
torch.distributed group (gloo) only carries the unique id and the results.

Rank 0 also runs the unsharded handle on the same instance; every rank writes
its per-iteration round infos, its owned slice of the per-edge state and the
best matching to <out>/rank<r>.npz.
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="O")
    ap.add_argument("--scale", type=float, default=0.01)
    ap.add_argument("--iters", type=int, default=6)
    ap.add_argument("--flags", type=int, default=0)
    ap.add_argument("--out", required=True)
    args = ap.parse_args()

    import torch
    import torch.distributed as dist
    import paper_conf_sc_xiangkfah23_b200 as ca
    from synth import make_config

    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    dist.init_process_group("gloo")
    torch.cuda.set_device(0)
    inst = make_config(args.config, scale=args.scale)
    obj = [ca.nccl_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0)

    keys = ("score_y", "score_z", "overlap_y", "overlap_z", "card_y", "card_z", "best_score", "best_iter",
            "source", "iter")
    res = {}
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, args.flags,
                      world=world, rank=rank, nccl_id=obj[0]) as h:
        sz = h.sizes()
        e0, e1 = sz["edge_begin"], sz["edge_end"]
        rounds = []
        for it in range(args.iters):
            # the later half through run(): the sharded step replayed from
            # its captured graph (NCCL calls inside), the rounding eager
            if it < args.iters // 2:
                h.iterate(1)
            else:
                h.run(1, with_round=False)
            r = h.round()
            rounds.append([float(r[k]) for k in keys])
        st = h.get_state(with_S=False)
        mate, _ = h.get_best()
        res.update(rounds=np.array(rounds), e0=e0, e1=e1, mate=mate,
                   merge_rounds=h.sizes()["merge_rounds"],
                   **{k: st[k][e0:e1] for k in ("yc", "zc", "yp", "zp", "d")})
    if rank == 0:
        with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, args.flags) as h1:
            rounds = []
            for _ in range(args.iters):
                h1.iterate(1)
                r = h1.round()
                rounds.append([float(r[k]) for k in keys])
            st = h1.get_state(with_S=False)
            mate, _ = h1.get_best()
            res.update(ref_rounds=np.array(rounds), ref_mate=mate,
                       **{"ref_" + k: st[k] for k in ("yc", "zc", "yp", "zp", "d")})
    np.savez(os.path.join(args.out, f"rank{rank}.npz"), **res)
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
