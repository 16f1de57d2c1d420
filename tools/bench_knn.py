"""NEXT-2 kNN sparsification (cualign_knn) throughput on the tensor cores.

For each (n_a, n_b, d, k): seeded N(0,1) float32 embeddings already on the
device; time --reps calls of ca.knn (bf16 unit rows + tcgen05 similarity
tiles + fused running top-k + merge) with CUDA events on the current stream.
Reports the dense-equivalent TFLOP/s (2 n_a n_b d per call) and similarity
pairs/s; the contraction is bf16 in / fp32 accumulate.

usage: python tools/bench_knn.py [--shapes 65536x65536x128x20,...] [--reps 3]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--shapes", default="32768x32768x64x20,65536x65536x128x20,200000x200000x128x20,100000x100000x256x20")
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    import torch
    import paper_conf_sc_xiangkfah23_b200 as ca
    g = torch.Generator(device="cuda").manual_seed(20231112)
    for shp in args.shapes.split(","):
        n_a, n_b, d, k = (int(x) for x in shp.split("x"))
        YA = torch.randn(n_a, d, device="cuda", generator=g)
        YB = torch.randn(n_b, d, device="cuda", generator=g)
        ca.knn(YA, YB, k)  # warm-up (module load, attributes)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(args.reps):
            ca.knn(YA, YB, k)
        e1.record()
        torch.cuda.synchronize()
        s = e0.elapsed_time(e1) / 1e3 / args.reps
        flops = 2.0 * n_a * n_b * d
        print(json.dumps(dict(n_a=n_a, n_b=n_b, d=d, k=k, s_per_call=s, tflops=flops / s / 1e12,
                              pairs_per_s=n_a * n_b / s)), flush=True)
        del YA, YB


if __name__ == "__main__":
    main()
