"""The BASELINE.json configurations as seeded synthetic instances.

BASELINE.json:configs[0..4] (shorthand T, P, O, S, R as in SURVEY.md §8(a)):
  T  tiny: A = ER(200, avg deg 6), B = P(A)+5%, top-10 kNN, 20 iterations
  P  PPI-shaped: Chung-Lu ~10k vertices / ~50k edges, top-20 kNN (~200k), 100 it.
  O  ontology-shaped: 300k x 200k vertices, L ~5M, S ~50M squares, 1 GPU
  S  social-shaped: ~1M each, L ~20M, S ~500M squares
  R  R-MAT scale 20, k = 5..50
Parameters alpha=1, beta=2, gamma=0.99 are our choice (reading Z1: the paper
gives none).  Seeds: 20231112 + config index.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from .graphs import (Graph, Candidates, er_graph, chung_lu_graph, rmat_graph,
                     permuted_noisy_copy, induced_subgraph, knn_candidates,
                     proxy_candidates, small_world_power_law)


@dataclass
class Instance:
    name: str
    A: Graph
    B: Graph
    L: Candidates
    truth: np.ndarray            # truth[a] = ground-truth image in B, -1 if none
    alpha: float = 1.0
    beta: float = 2.0
    gamma: float = 0.99
    n_iter: int = 20
    seed: int = 0
    meta: dict = field(default_factory=dict)


SEED0 = 20231112

CONFIGS = {
    "T": dict(index=0, n_iter=20,
              desc="tiny: ER n=200 avg deg 6; B=P(A)+5%; top-10 kNN; 20 iterations"),
    "P": dict(index=1, n_iter=100,
              desc="PPI-shaped: Chung-Lu tau=2.5 n=1e4, 5e4 edges; B=P(A)+5%; top-20 kNN; 100 iterations"),
    "O": dict(index=2, n_iter=100,
              desc="ontology-shaped: clustered power-law n_A=3e5 (avg deg 18), B=P(A[V']) |V'|=2e5 +5%; proxy k=16.67 -> m~5e6; s~1e8"),
    "S": dict(index=3, n_iter=100,
              desc="social-shaped: clustered power-law n=1e6 each; B=P(A)+5%; proxy k=20 -> m=2e7; s~1e9"),
    "R": dict(index=4, n_iter=20,
              desc="R-MAT scale 20 edge factor 8 (0.57,0.19,0.19,0.05); proxy k in {5..50}"),
}

# Locality-proxy calibration: average A degree and
# lambda chosen so that s = nnz(S) lands near the BASELINE.json targets.
# Graphs: small_world_power_law (ring lattice of half-width h = clustering, plus
# a Chung-Lu tau=2.5 layer of n_random_per_vertex * n edges = hubs).
# Calibrated with the closed form s = sum((A L) o (L B)) (pin P3) at scale 0.1
# / 0.03: O gives s/m = 20.1 (s ~ 1.0e8 at m = 5e6); S gives s/m ~ 50.
O_PARAMS = dict(n_a=300_000, n_b=200_000, h=7, n_random=2.0, k=16.67, lam=0.9, two_hop=0.5, tau=2.5)
S_PARAMS = dict(n=1_000_000, h=7, n_random=2.0, k=20.0, lam=0.9, two_hop=0.5, tau=2.5)


def _pair_from_A(A: Graph, rng, noise=0.05):
    B, perm = permuted_noisy_copy(A, rng, noise)
    return B, perm


def make_config(name: str, scale: float = 1.0, k: int | None = None,
                seed: int | None = None) -> Instance:
    """Build config `name` (T, P, O, S, R).  `scale` shrinks vertex/edge counts
    (same shape) for tests; `k` overrides the candidate count for R."""
    cfg = CONFIGS[name]
    seed = SEED0 + cfg["index"] if seed is None else seed
    rng = np.random.default_rng(seed)
    if name == "T":
        n = max(8, int(200 * scale))
        A = er_graph(n, 3 * n, rng)
        B, perm = _pair_from_A(A, rng)
        L = knn_candidates(A, B, 10 if k is None else k, rng)
        truth = perm
    elif name == "P":
        n = max(16, int(10_000 * scale))
        A = chung_lu_graph(n, 5 * n, 2.5, rng)
        B, perm = _pair_from_A(A, rng)
        L = knn_candidates(A, B, 20 if k is None else k, rng)
        truth = perm
    elif name == "O":
        p = O_PARAMS
        n_a = max(32, int(p["n_a"] * scale))
        n_b = max(16, int(p["n_b"] * scale))
        A = small_world_power_law(n_a, p["h"], int(p["n_random"] * n_a), p["tau"], rng)
        keep = np.sort(rng.choice(n_a, size=n_b, replace=False))
        sub = induced_subgraph(A, keep)
        B, perm = _pair_from_A(sub, rng)
        truth = np.full(n_a, -1, dtype=np.int64)
        truth[keep] = perm
        L = proxy_candidates(B, truth, p["k"] if k is None else k, p["lam"], rng,
                             two_hop=p["two_hop"])
    elif name == "S":
        p = S_PARAMS
        n = max(32, int(p["n"] * scale))
        A = small_world_power_law(n, p["h"], int(p["n_random"] * n), p["tau"], rng)
        B, perm = _pair_from_A(A, rng)
        truth = perm
        L = proxy_candidates(B, truth, p["k"] if k is None else k, p["lam"], rng,
                             two_hop=p["two_hop"])
    elif name == "R":
        scale_bits = max(6, int(round(20 + np.log2(scale)))) if scale != 1.0 else 20
        A = rmat_graph(scale_bits, 8, (0.57, 0.19, 0.19, 0.05), rng)
        B, perm = _pair_from_A(A, rng)
        truth = perm
        L = proxy_candidates(B, truth, 10 if k is None else k, 0.6, rng)
    else:
        raise KeyError(name)
    return Instance(name=name, A=A, B=B, L=L, truth=np.asarray(truth, dtype=np.int64),
                    n_iter=cfg["n_iter"], seed=seed,
                    meta=dict(desc=cfg["desc"], scale=scale, k=k))


# Size of the full config O instance (default seed), measured once with the
# closed form s = sum((A L) o (L B)) (scipy; pin P3) -- used only to scale the
# oracle's bounded-sample rate to the full workload in bench.py.
O_FULL_M = 5_001_168
O_FULL_S = 100_181_414


def O_full_work():
    return O_FULL_M, O_FULL_S
