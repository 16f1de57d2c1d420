"""Small shared helpers for the tests (no method arithmetic)."""
from __future__ import annotations

import json
import os
from fractions import Fraction

import numpy as np

from synth import (Graph, Candidates, csr_from_pairs, er_graph, random_candidates,
                   complete_candidates, permuted_noisy_copy)

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load_golden(name):
    with open(os.path.join(GOLDEN, name)) as fh:
        return json.load(fh)


def graph_from_edges(n, edges) -> Graph:
    if len(edges) == 0:
        return Graph(n=n, rowptr=np.zeros(n + 1, dtype=np.int64), col=np.zeros(0, dtype=np.int32))
    e = np.asarray(edges, dtype=np.int64)
    return csr_from_pairs(n, e[:, 0], e[:, 1])


def candidates_from_lists(n_a, n_b, a, b, w) -> Candidates:
    return Candidates(n_a=n_a, n_b=n_b, a=np.asarray(a, dtype=np.int32),
                      b=np.asarray(b, dtype=np.int32), w=np.asarray(w, dtype=np.float64))


def golden_instance(g):
    A = graph_from_edges(g["A"]["n"], g["A"]["edges"])
    B = graph_from_edges(g["B"]["n"], g["B"]["edges"])
    w = [float(Fraction(x)) for x in g["L"]["w"]]
    L = candidates_from_lists(A.n, B.n, g["L"]["a"], g["L"]["b"], w)
    return A, B, L


def tiny_instance(seed, n=6, n_edges=7, k=3, weights="uniform", n_b=None, permuted=False):
    rng = np.random.default_rng(seed)
    n_b = n if n_b is None else n_b
    A = er_graph(n, min(n_edges, n * (n - 1) // 2), rng)
    if permuted:
        B, perm = permuted_noisy_copy(A, rng, noise=0.0)
        L = random_candidates(n, n, k, rng, weights=weights, truth=perm)
        return A, B, L, perm
    B = er_graph(n_b, min(n_edges, n_b * (n_b - 1) // 2), rng)
    L = random_candidates(n, n_b, k, rng, weights=weights)
    return A, B, L, None


def S_from_csr(rowptr, col, m):
    S = np.zeros((m, m), dtype=np.int8)
    for e in range(m):
        S[e, col[rowptr[e]:rowptr[e + 1]]] = 1
    return S
