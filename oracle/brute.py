"""Brute-force references for tiny inputs -- TEST INFRASTRUCTURE ONLY.

These pin the oracle (they are not the oracle itself):
  * overlap_direct: the number of overlapped edges of a matching straight from
    the words of PAPER.md:60 ("an edge (i, j) in E_A is overlapped to an edge
    (i', j') in E_B if both (i, i') and (j, j') are in M"), with no S (pin P11).
  * S_dense: S_{(i,i'),(j,j')} = 1 iff (i, j) in E_A and (i', j') in E_B
    (PAPER.md:66), by looping over all pairs with dense adjacency (pin P1).
  * best_alignment: the Eq. 1 optimum over every matching of
    L, by enumerating permutations (n <= 7) (pin P12).
  * max_weight_matching: maximum-weight matching of L by enumeration (pin P10).
"""
from __future__ import annotations

import itertools

import numpy as np


def dense_adj(g) -> np.ndarray:
    adj = np.zeros((g.n, g.n), dtype=bool)
    for u in range(g.n):
        for x in range(g.rowptr[u], g.rowptr[u + 1]):
            adj[u, g.col[x]] = True
    return adj


def S_dense(A, B, L) -> np.ndarray:
    """Dense m x m 0/1 matrix S by the definition."""
    adjA, adjB = dense_adj(A), dense_adj(B)
    m = L.m
    S = np.zeros((m, m), dtype=np.int8)
    for e in range(m):
        i, ip = int(L.a[e]), int(L.b[e])
        for f in range(m):
            j, jp = int(L.a[f]), int(L.b[f])
            if adjA[i, j] and adjB[ip, jp]:
                S[e, f] = 1
    return S


def overlap_direct(A, B, mate_b_of_a: dict) -> int:
    """Number of A edges {i, j} whose images (M(i), M(j)) form a B edge."""
    adjB = dense_adj(B)
    cnt = 0
    for i in range(A.n):
        for x in range(A.rowptr[i], A.rowptr[i + 1]):
            j = int(A.col[x])
            if i < j and i in mate_b_of_a and j in mate_b_of_a:
                if adjB[mate_b_of_a[i], mate_b_of_a[j]]:
                    cnt += 1
    return cnt


def score_of(A, B, L, edges, alpha, beta):
    """Eq. 1 objective of the matching given as a list of L edge ids."""
    mate = {int(L.a[e]): int(L.b[e]) for e in edges}
    weight = float(sum(L.w[e] for e in edges))
    return alpha * weight + beta * overlap_direct(A, B, mate), weight


def best_alignment(A, B, L, alpha, beta):
    """max over matchings M of L of alpha*w(M) + beta*overlap(M).

    Valid for w >= 0, alpha, beta >= 0 (the objective is monotone under adding
    edges), so every optimum extends to a permutation: enumerate pi in S_n and
    keep the L-restriction {(a, pi(a)) in L}.  Requires n_A == n_B <= 7."""
    assert A.n == B.n and A.n <= 7
    assert np.all(L.w >= 0) and alpha >= 0 and beta >= 0
    eid = {(int(a), int(b)): e for e, (a, b) in enumerate(zip(L.a, L.b))}
    best = -1.0
    best_edges = None
    for pi in itertools.permutations(range(B.n)):
        edges = [eid[(a, pi[a])] for a in range(A.n) if (a, pi[a]) in eid]
        sc, _ = score_of(A, B, L, edges, alpha, beta)
        if sc > best:
            best, best_edges = sc, edges
    return best, best_edges


def max_weight_matching(L, x=None) -> float:
    """Maximum total weight of a matching of L under weights x (default w),
    only positive weights useful; by enumeration over A vertices."""
    x = L.w if x is None else x
    by_a = {}
    for e in range(L.m):
        if x[e] > 0:
            by_a.setdefault(int(L.a[e]), []).append(e)
    verts = sorted(by_a)

    def rec(k, used):
        if k == len(verts):
            return 0.0
        best = rec(k + 1, used)
        for e in by_a[verts[k]]:
            b = int(L.b[e])
            if b not in used:
                used.add(b)
                best = max(best, x[e] + rec(k + 1, used))
                used.remove(b)
        return best

    return rec(0, set())
