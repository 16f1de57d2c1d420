"""Pins for the oracle's BP iteration (Alg. 2 lines 9-16).

P5 iteration-1 closed form (and d(2) = d(1) for w >= 0).
P6 integer regime: exactness and the bound |y|, |z| <= max d.
P7 worked example W1 (tests/golden/W1.json), exact dyadic values p = 1..3.
P8 worked example W2 (tests/golden/W2.json), both readings of othermax (Z4).
Plus: agreement with Alg. 2 written on dense matrices (tests/dense_alg2.py), in
exact rationals on tiny inputs -- catches transposes, row/column swaps and
dropped terms in the sparse oracle.
"""
from fractions import Fraction

import numpy as np
import pytest

import oracle
from oracle import Oracle, gamma_power
from synth import make_config
from tests import dense_alg2 as D
from tests.util import load_golden, golden_instance, tiny_instance


def _pairs_values(o, pairs, Sp):
    rowptr, col, _ = o.get_S()
    out = []
    for e, f in pairs:
        row = list(col[rowptr[e]:rowptr[e + 1]])
        out.append(Sp[rowptr[e] + row.index(f)])
    return out


def test_P7_worked_example_W1():
    g = load_golden("W1.json")
    A, B, L = golden_instance(g)
    gamma = float(Fraction(g["gamma"]))
    o = Oracle(A, B, L, g["alpha"], g["beta"])
    for it in g["iterations"]:
        o.step_gamma(gamma)
        st = o.get_state()
        for key in ("d", "yc", "zc", "yp", "zp"):
            assert list(st[key]) == [float(Fraction(x)) for x in it[key]], (it["p"], key)
        assert _pairs_values(o, g["S_pairs"], st["Sp"]) == [float(Fraction(x)) for x in it["Sp"]]
        info = o.round()
        r = g["rounding"]
        assert sorted(e for e in info["mate_y"] if e >= 0) == r["mate_edges_each_p"]
        assert sorted(e for e in info["mate_z"] if e >= 0) == r["mate_edges_each_p"]
        assert info["score"] == float(Fraction(r["score"]))
        assert info["overlap_y"] == r["overlap"]
        assert info["best_iter"] == r["best_iter"]
    mate, best, it = o.get_best()
    assert best == float(Fraction(g["rounding"]["best_score"]))


def test_W1_golden_rederived_in_exact_rationals():
    """The golden W1 table equals Alg. 2 in matrix form evaluated in Fractions."""
    g = load_golden("W1.json")
    m = 4
    S = [[0] * m for _ in range(m)]
    for e, f in g["S_pairs"]:
        S[e][f] = 1
    w = [Fraction(x) for x in g["L"]["w"]]
    st = D.zero_state(m)
    gamma = Fraction(g["gamma"])
    for it in g["iterations"]:
        gp = gamma ** it["p"]
        st = D.step(S, w, g["L"]["a"], g["L"]["b"], g["alpha"], g["beta"], gp, 1 - gp, st)
        for key in ("d", "yc", "zc", "yp", "zp"):
            assert st[key] == [Fraction(x) for x in it[key]]
        assert [st["Sp"][e][f] for e, f in g["S_pairs"]] == [Fraction(x) for x in it["Sp"]]
        assert [st["F"][e][f] for e, f in g["S_pairs"]] == [Fraction(x) for x in it["F"]]


@pytest.mark.parametrize("reading", ["maxplus", "literal"])
def test_P8_worked_example_W2(reading):
    g = load_golden("W2.json")
    A, B, L = golden_instance(g)
    flags = oracle.OTHERMAX_LITERAL if reading == "literal" else 0
    o = Oracle(A, B, L, g["alpha"], g["beta"], flags)
    for it in g[reading]:
        o.step(1.0, 0.0)  # gamma = 1: g = 1, h = 0
        st = o.get_state()
        assert list(st["yc"]) == [float(x) for x in it["yc"]], it["p"]
        assert list(st["zc"]) == [float(x) for x in it["zc"]], it["p"]
        info = o.round()
        if "My" in it:
            assert sorted(e for e in info["mate_y"] if e >= 0) == it["My"]
            assert sorted(e for e in info["mate_z"] if e >= 0) == it["Mz"]
    mate, best, best_it = o.get_best()
    assert best == g["best_score"] and best_it == g["best_iter"]


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("literal", [False, True])
def test_oracle_equals_dense_matrix_alg2_exactly(seed, literal):
    """Integer data (alpha, beta, w integer; gamma = 1/2 dyadic): fp64 is exact
    for the first iterations, so the sparse oracle must equal the exact
    rational dense formulation bit for bit."""
    A, B, L, _ = tiny_instance(seed, n=6, n_edges=9, k=3, weights="int")
    alpha, beta = 1, 2
    o = Oracle(A, B, L, alpha, beta, oracle.OTHERMAX_LITERAL if literal else 0)
    rowptr, col, _ = o.get_S()
    m = L.m
    S = [[0] * m for _ in range(m)]
    for e in range(m):
        for f in col[rowptr[e]:rowptr[e + 1]]:
            S[e][int(f)] = 1
    w = [Fraction(int(x)) for x in L.w]
    st = D.zero_state(m)
    for p in range(1, 5):
        gp = Fraction(1, 2) ** p
        o.step(float(gp), float(1 - gp))
        st = D.step(S, w, list(L.a), list(L.b), alpha, beta, gp, 1 - gp, st, literal)
        got = o.get_state()
        for key in ("d", "yc", "zc", "yp", "zp"):
            assert list(got[key]) == [float(x) for x in st[key]], (p, key)
        want_sp = [float(st["Sp"][e][int(f)]) for e in range(m) for f in col[rowptr[e]:rowptr[e + 1]]]
        assert list(got["Sp"]) == want_sp


@pytest.mark.parametrize("seed", range(4))
def test_oracle_close_to_dense_float(seed):
    """Generic float data: oracle vs dense formulation in fp64 within 1e-12."""
    A, B, L, _ = tiny_instance(seed, n=7, n_edges=12, k=4)
    alpha, beta, gamma = 1.0, 2.0, 0.99
    o = Oracle(A, B, L, alpha, beta)
    rowptr, col, _ = o.get_S()
    m = L.m
    S = [[0] * m for _ in range(m)]
    for e in range(m):
        for f in col[rowptr[e]:rowptr[e + 1]]:
            S[e][int(f)] = 1
    st = D.zero_state(m, 0.0)
    for p in range(1, 12):
        gp = gamma_power(gamma, p)
        o.step(gp, 1.0 - gp)
        st = D.step(S, list(L.w), list(L.a), list(L.b), alpha, beta, gp, 1.0 - gp, st)
        got = o.get_state()
        for key in ("d", "yc", "zc", "yp", "zp"):
            np.testing.assert_allclose(got[key], st[key], rtol=0, atol=1e-12)


@pytest.mark.parametrize("name", ["T"])
def test_P5_iteration1_closed_form(name):
    inst = make_config(name)
    alpha, beta, gamma = 1.0, 2.0, 0.5  # dyadic gamma: products exact
    o = Oracle(inst.A, inst.B, inst.L, alpha, beta)
    rowptr, col, _ = o.get_S()
    r = np.diff(rowptr).astype(np.float64)
    o.step_gamma(gamma)
    st = o.get_state()
    d = alpha * inst.L.w + beta * r
    np.testing.assert_allclose(st["d"], d, rtol=1e-15, atol=0)
    assert np.array_equal(st["yc"], st["d"]) and np.array_equal(st["zc"], st["d"])
    np.testing.assert_allclose(st["yp"], gamma * st["d"], rtol=1e-15)
    rows = np.repeat(np.arange(inst.L.m), np.diff(rowptr))
    np.testing.assert_allclose(st["Sp"], gamma * (st["d"][rows] - beta), rtol=1e-14, atol=1e-14)
    # iteration 2 with w >= 0: F == beta again, so d(2) == d(1)
    d1 = st["d"].copy()
    o.step_gamma(gamma)
    assert np.array_equal(o.get_state()["d"], d1)


@pytest.mark.parametrize("seed", range(4))
def test_P6_integer_regime_bounds_and_exactness(seed):
    """gamma = 1, integer alpha, beta, w: every value is an integer (exact)."""
    A, B, L, _ = tiny_instance(seed, n=7, n_edges=12, k=4, weights="int")
    alpha, beta = 2.0, 3.0
    o = Oracle(A, B, L, alpha, beta)
    rowptr, _, _ = o.get_S()
    dmax = alpha * L.w.max() + beta * np.diff(rowptr).max()
    for _ in range(15):
        o.step(1.0, 0.0)
        st = o.get_state()
        for key in ("d", "yc", "zc", "yp", "zp", "Sp"):
            assert np.all(st[key] == np.round(st[key])), key
        assert np.all(np.abs(st["yc"]) <= dmax) and np.all(np.abs(st["zc"]) <= dmax)
