"""B200-native NetAlignBP + locally-dominant matching engine (cuAlign, SC-W 2023).

The compute path is libcualign_bp.so (CUDA, sm_100a; C ABI in
include/cualign_bp.h).  This package is the thin Python binding over it plus
the end-to-end `align` helper and the sharded (multi-GPU) driver.
"""
import time

from ._lib import (CuAlignBP, CuAlignError, match, quality, alignment_map, knn, KnnCandidates, load_library, version, nccl_unique_id,
                   FLAG_DEVICE_PTRS, FLAG_EXACT, FLAG_OTHERMAX_LITERAL, FLAG_ROUND_DAMPED,
                   FLAG_TIMING, FLAG_MATCH_ROUNDS, FLAG_FP32_S, EXPORTED, LIB_PATH, KERNEL_CLASS_NAMES)


def align(A, B, L, alpha=1.0, beta=2.0, gamma=0.99, n_iter=100, flags=0, device=0, stream=None, **shard):
    """End-to-end alignment (Alg. 2): init (S build), n_iter
    x (iterate + round), best.  Returns (mate_a, info, per-round infos).
    shard: world / rank / nccl_id of a sharded run (see CuAlignBP)."""
    t0 = time.perf_counter()
    with CuAlignBP(A, B, L, alpha, beta, gamma, flags, device, stream, **shard) as h:
        t1 = time.perf_counter()
        infos = h.run_trace(n_iter)  # graph replays; every step's round info to the host
        t2 = time.perf_counter()
        mate, info = h.get_best()
        info["t_result"] = time.perf_counter()            # result on the host (before teardown)
        info["phases_s"] = {"init": t1 - t0, "iterations": t2 - t1, "best": info["t_result"] - t2}
        info["schedule"] = h.sizes()["schedule"]
    return mate, info, infos


__all__ = ["CuAlignBP", "CuAlignError", "match", "quality", "alignment_map", "knn", "KnnCandidates", "align", "load_library", "version", "nccl_unique_id",
           "FLAG_DEVICE_PTRS", "FLAG_EXACT", "FLAG_OTHERMAX_LITERAL", "FLAG_ROUND_DAMPED",
           "FLAG_TIMING", "FLAG_MATCH_ROUNDS", "FLAG_FP32_S", "EXPORTED", "LIB_PATH", "KERNEL_CLASS_NAMES"]
