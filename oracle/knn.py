"""kNN sparsification oracle (NEXT-2) -- TEST INFRASTRUCTURE
ONLY (tests/, bench/tools may import it; the CUDA path never does).

Alg. 1 lines 7-14 (text :121): for every u in V_A and v in
V_B, s(u, v) = cosine_similarity(Y_A(u), Y_B(v)) (l.9), then keep the kNN
edges (l.12-14).  Readings:
  * Z19: "k least-weighted edges" of a *similarity* is read as the k MOST
    similar B vertices of each A vertex; ties go to the lower B index;
  * a zero embedding has similarity 0 with everything;
  * precision: the tensor-core path multiplies the unit vectors rounded to
    bf16 (round to nearest even) and accumulates in fp32.  The oracle follows
    the same definition with exact arithmetic: unit vectors in fp64 (sum of
    squares in ascending coordinate order, sqrt, divide), rounded to bf16,
    dot products of the bf16 values in fp64 (every product is exact).
    `cosine_fp64` gives the unrounded cosine for comparison.
Plain numpy, written for checking by eye, not speed.
"""
from __future__ import annotations

import numpy as np


def round_bf16(x: np.ndarray) -> np.ndarray:
    """fp64 -> nearest bf16 (ties to even), returned as fp64.  Done as
    fp64 -> fp32 (nearest) -> bf16 (nearest even on the top 16 bits) only when
    the fp32 step is exact for the final rounding; to avoid double rounding
    the bf16 rounding is applied to the fp64 value directly."""
    x = np.asarray(x, dtype=np.float64)
    out = np.empty_like(x)
    flat, res = x.ravel(), out.ravel()
    for i in range(flat.shape[0]):
        v = float(flat[i])
        if v == 0.0 or not np.isfinite(v):
            res[i] = v
            continue
        m, e = np.frexp(v)            # v = m * 2^e, 0.5 <= |m| < 1
        # bf16 keeps 8 significant bits: |m| * 2^8 rounded to an integer, ties to even
        scaled = m * 256.0
        r = np.round(scaled)          # numpy rounds half to even
        res[i] = np.ldexp(r / 256.0, e)
    return out


def unit_rows(Y: np.ndarray) -> np.ndarray:
    """Rows divided by their Euclidean norm (fp64; zero rows stay zero)."""
    Y = np.asarray(Y, dtype=np.float64)
    out = np.zeros_like(Y)
    for i in range(Y.shape[0]):
        ss = 0.0
        for j in range(Y.shape[1]):       # ascending coordinate order
            ss = ss + Y[i, j] * Y[i, j]
        if ss > 0.0:
            nrm = np.sqrt(ss)
            out[i] = Y[i] / nrm
    return out


def similarity_bf16(YA: np.ndarray, YB: np.ndarray) -> np.ndarray:
    """s(u, v) of the tensor-core definition: dot products of the bf16-rounded
    unit vectors, exact products summed in fp64."""
    ua = round_bf16(unit_rows(YA))
    ub = round_bf16(unit_rows(YB))
    return ua @ ub.T


def cosine_fp64(YA: np.ndarray, YB: np.ndarray) -> np.ndarray:
    return unit_rows(YA) @ unit_rows(YB).T


def knn_from_similarity(S: np.ndarray, k: int):
    """Top-k per row by (similarity desc, column asc); returns L as (a, b, w)
    sorted by (a, b) -- the canonical edge order of cualign_edges."""
    n_a, n_b = S.shape
    k = min(k, n_b)
    a_out, b_out, w_out = [], [], []
    for u in range(n_a):
        order = sorted(range(n_b), key=lambda v: (-S[u, v], v))[:k]
        for v in sorted(order):
            a_out.append(u)
            b_out.append(v)
            w_out.append(S[u, v])
    return (np.asarray(a_out, dtype=np.int32), np.asarray(b_out, dtype=np.int32),
            np.asarray(w_out, dtype=np.float64))


def knn(YA: np.ndarray, YB: np.ndarray, k: int):
    """Alg. 1 l.7-14 under the readings above."""
    return knn_from_similarity(similarity_bf16(YA, YB), k)
