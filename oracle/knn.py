"""kNN sparsification oracle (NEXT-2) -- TEST INFRASTRUCTURE
ONLY (tests/, bench/tools may import it; the CUDA path never does).

Alg. 1 lines 7-14 (text :121): for every u in V_A and v in
V_B, s(u, v) = cosine_similarity(Y_A(u), Y_B(v)) (l.9), then keep the kNN
edges (l.12-14).  Readings:
  * Z19: "k least-weighted edges" of a *similarity* is read as the k MOST
    similar B vertices of each A vertex; ties go to the lower B index;
  * a zero embedding has similarity 0 with everything.
The reference is the paper's cosine in fp64 (`cosine_fp64`): unit vectors
(sum of squares in ascending coordinate order, sqrt, divide) and their dot
products.  An implementation that computes in lower precision is judged
against it with the rigorous error bound `dot_error_bound` (below), not
against a copy of its own rounding.
Plain numpy, written for checking by eye, not speed.
"""
from __future__ import annotations

import numpy as np


def unit_rows(Y: np.ndarray) -> np.ndarray:
    """Rows divided by their Euclidean norm (fp64; zero rows stay zero).  The
    sum of squares runs over the coordinates in ascending order (one column
    at a time, all rows together)."""
    Y = np.asarray(Y, dtype=np.float64)
    ss = np.zeros(Y.shape[0])
    for j in range(Y.shape[1]):
        ss = ss + Y[:, j] * Y[:, j]
    out = np.zeros_like(Y)
    nz = ss > 0.0
    out[nz] = Y[nz] / np.sqrt(ss[nz])[:, None]
    return out


def cosine_fp64(YA: np.ndarray, YB: np.ndarray) -> np.ndarray:
    """s(u, v) = cos(Y_A(u), Y_B(v)) (Alg. 1 l.9), all pairs, fp64."""
    return unit_rows(YA) @ unit_rows(YB).T


def dot_error_bound(YA: np.ndarray, YB: np.ndarray, unit_roundoff: float, acc_roundoff: float) -> np.ndarray:
    """Rigorous bound on |s~(u, v) - s(u, v)| for a dot product of the unit
    vectors whose inputs are each rounded to a format with unit roundoff
    `unit_roundoff` (bf16: 2^-8) and accumulated in a format with unit
    roundoff `acc_roundoff` (fp32: 2^-24) over d terms.  With
    u~_i = u_i (1 + a_i), v~_i = v_i (1 + b_i), |a_i|, |b_i| <= r:
        |u~.v~ - u.v| <= (2 r + r^2) sum_i |u_i v_i|
    and the accumulation of d products adds at most
        gamma_d sum_i |u~_i v~_i| <= gamma_d (1 + r)^2 sum_i |u_i v_i|,
    gamma_d = d q / (1 - d q) (standard recursive-summation bound, q = acc
    roundoff; it also covers any summation order and fused products).
    The extra 1e-15 absorbs the fp64 error of computing the reference itself."""
    UA, UB = np.abs(unit_rows(YA)), np.abs(unit_rows(YB))
    d = UA.shape[1]
    r, q = float(unit_roundoff), float(acc_roundoff)
    gamma_d = d * q / (1.0 - d * q)
    absdot = UA @ UB.T
    return (2 * r + r * r + gamma_d * (1 + r) ** 2) * absdot + 1e-15


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
    """Alg. 1 l.7-14 under the readings above (fp64 cosine)."""
    return knn_from_similarity(cosine_fp64(YA, YB), k)
