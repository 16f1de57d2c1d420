"""Pins of the quality oracle (oracle/quality.py, NEXT-4): a hand-derived
example, the closed form of a perfect alignment, the tie to the main oracle's
overlap (x'Sx/2, PAPER.md:66 = conserved edges), and bounds that
hold for any alignment."""
import math
from fractions import Fraction

import numpy as np
import pytest

from oracle import Oracle
from oracle.quality import quality
from synth import make_config
from tests.util import graph_from_edges, load_golden, tiny_instance


def test_Q1_hand_example():
    g = load_golden("Q1.json")
    A = graph_from_edges(g["A"]["n"], g["A"]["edges"])
    B = graph_from_edges(g["B"]["n"], g["B"]["edges"])
    q = quality(A, B, np.array(g["map"]), np.array(g["truth"]))
    ex = g["expect"]
    for k in ("edges_a", "edges_b", "aligned", "truth_total", "correct", "conserved", "induced"):
        assert q[k] == ex[k], k
    for k in ("nc", "ec", "ics", "s3", "ncv", "gs3"):
        assert q[k] == pytest.approx(float(Fraction(ex[k])), abs=1e-15), k
    assert q["ncv_gs3"] ** 2 == pytest.approx(float(Fraction(ex["ncv_gs3_squared"])), abs=1e-15)


@pytest.mark.parametrize("name", ["T", "P"])
def test_true_permutation_scores_one(name):
    """B = P(A) without noise and M = P: every measure is 1."""
    from synth.graphs import permuted_noisy_copy
    inst = make_config(name, scale=0.1 if name == "P" else 1.0)
    rng = np.random.default_rng(5)
    B, perm = permuted_noisy_copy(inst.A, rng, noise=0.0)
    q = quality(inst.A, B, perm.astype(np.int32), perm.astype(np.int32))
    for k in ("nc", "ec", "ics", "s3", "ncv", "gs3", "ncv_gs3"):
        assert q[k] == 1.0, k
    assert q["conserved"] == q["edges_a"] == q["induced"] == q["edges_b"]


@pytest.mark.parametrize("seed", range(5))
def test_conserved_equals_oracle_overlap(seed):
    """conserved (edge definition) = x'Sx/2 of the C oracle."""
    A, B, L, _ = tiny_instance(seed, n=12, n_edges=25, k=4, permuted=True)
    o = Oracle(A, B, L, 1.0, 2.0)
    x = np.random.default_rng(seed).normal(size=o.m)
    mate, _ = o.greedy(x)
    ev = o.evaluate(mate)
    mp = np.where(mate >= 0, L.b[np.maximum(mate, 0)], -1)
    q = quality(A, B, mp)
    assert q["conserved"] == ev["overlap"]
    assert q["aligned"] == int(np.sum(mate >= 0))


@pytest.mark.parametrize("seed", range(8))
def test_bounds_random_alignments(seed):
    rng = np.random.default_rng(100 + seed)
    A, B, L, perm = tiny_instance(seed, n=15, n_edges=30, k=3, permuted=True)
    k = int(rng.integers(0, A.n + 1))
    src = rng.choice(A.n, k, replace=False)
    dst = rng.choice(B.n, k, replace=False)
    mp = np.full(A.n, -1, dtype=np.int32)
    mp[src] = dst
    q = quality(A, B, mp, perm)
    assert 0 <= q["conserved"] <= min(q["edges_a"], q["induced"])
    assert q["s3"] <= min(q["ec"], q["ics"]) + 1e-15
    assert 0.0 <= q["nc"] <= 1.0 and 0.0 <= q["ncv"] <= 1.0
    assert q["correct"] == int(np.sum((mp == perm) & (perm >= 0)))
    assert q["ncv_gs3"] == pytest.approx(math.sqrt(q["ncv"] * q["s3"]))


def test_rejects_non_injective():
    A = graph_from_edges(3, [[0, 1]])
    B = graph_from_edges(3, [[0, 1]])
    with pytest.raises(ValueError):
        quality(A, B, np.array([0, 0, -1]))
