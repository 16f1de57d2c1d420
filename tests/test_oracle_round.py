"""Pins for the oracle's rounding, evaluation and best-so-far (Alg. 2 l.17-24,
PAPER.md:170-177; matching :207-209; objective Eq. 1 :64-72).

P9  greedy == the locally dominant algorithm run step by step as PAPER.md:209
    describes it (oracle/ld_matching.py), fuzzed with massive ties and negatives.
P10 1/2 bound: w(greedy) >= 1/2 w(max-weight matching) (brute force, scipy LSA).
P11 overlap via S == direct count of overlapped A edges.
P12 brute-force optimum: bestScore <= OPT; recoverable instances reach OPT.
P13 S empty: BP reduces to max-product BP for bipartite matching; the rounded
    messages reach the assignment optimum (scipy.optimize.linear_sum_assignment).
P14 alpha = 0, beta = 1 on B = P(A): OPT overlap = |E_A|.
"""
import numpy as np
import pytest
from scipy.optimize import linear_sum_assignment

from oracle import Oracle
from oracle.brute import best_alignment, max_weight_matching, overlap_direct, score_of
from oracle.ld_matching import locally_dominant
from synth import make_config, complete_candidates, random_candidates, er_graph
from tests.util import tiny_instance, graph_from_edges


@pytest.mark.parametrize("seed", range(30))
@pytest.mark.parametrize("weights", ["ties", "ties_signed", "uniform"])
def test_P9_greedy_equals_locally_dominant(seed, weights):
    rng = np.random.default_rng(seed)
    n_a, n_b = int(rng.integers(2, 12)), int(rng.integers(2, 12))
    L = random_candidates(n_a, n_b, int(rng.integers(1, min(n_b, 5) + 1)), rng, weights=weights)
    A = graph_from_edges(n_a, [])
    B = graph_from_edges(n_b, [])
    o = Oracle(A, B, L, 1.0, 1.0)
    mate, _ = o.greedy(L.w)
    assert list(mate) == locally_dominant(L, L.w)


@pytest.mark.parametrize("seed", range(20))
def test_P10_half_approximation(seed):
    rng = np.random.default_rng(1000 + seed)
    n = int(rng.integers(2, 7))
    L = random_candidates(n, n, int(rng.integers(1, n + 1)), rng, weights="uniform")
    o = Oracle(graph_from_edges(n, []), graph_from_edges(n, []), L, 1.0, 1.0)
    mate, _ = o.greedy(L.w)
    got = sum(L.w[e] for e in mate if e >= 0)
    opt = max_weight_matching(L)
    assert got >= 0.5 * opt - 1e-12
    assert got <= opt + 1e-12


@pytest.mark.parametrize("seed", range(5))
def test_P10_half_approximation_lsa(seed):
    rng = np.random.default_rng(seed)
    n = 40
    L = complete_candidates(n, n, rng=rng)
    o = Oracle(graph_from_edges(n, []), graph_from_edges(n, []), L, 1.0, 1.0)
    mate, card = o.greedy(L.w)
    got = sum(L.w[e] for e in mate if e >= 0)
    W = L.w.reshape(n, n)
    r, c = linear_sum_assignment(-W)
    opt = W[r, c].sum()
    assert got >= 0.5 * opt and got <= opt + 1e-9
    assert card == n  # complete positive L: greedy is perfect


@pytest.mark.parametrize("seed", range(10))
def test_P11_overlap_via_S_equals_direct_count(seed):
    A, B, L, _ = tiny_instance(seed, n=7, n_edges=11, k=4)
    o = Oracle(A, B, L, 1.0, 2.0)
    for xs in range(4):
        x = np.random.default_rng(xs).random(L.m) - 0.2
        mate, _ = o.greedy(x)
        ev = o.evaluate(mate)
        m_dict = {int(L.a[e]): int(L.b[e]) for e in mate if e >= 0}
        assert ev["overlap"] == overlap_direct(A, B, m_dict)
        assert ev["weight"] == pytest.approx(sum(L.w[e] for e in mate if e >= 0), abs=1e-12)
        assert ev["score"] == pytest.approx(1.0 * ev["weight"] + 2.0 * ev["overlap"], abs=1e-12)


@pytest.mark.parametrize("seed", range(12))
def test_P12_best_never_exceeds_bruteforce_optimum(seed):
    A, B, L, _ = tiny_instance(seed, n=6, n_edges=8, k=3)
    alpha, beta = 1.0, 2.0
    opt, _ = best_alignment(A, B, L, alpha, beta)
    o = Oracle(A, B, L, alpha, beta)
    infos = o.align(25, 0.99)
    mate, best, _ = o.get_best()
    assert best <= opt + 1e-12
    for inf in infos:
        assert inf["score_y"] <= opt + 1e-12 and inf["score_z"] <= opt + 1e-12
    # the best matching's score re-evaluates to best
    edges = [e for e in mate if e >= 0]
    sc, _ = score_of(A, B, L, edges, alpha, beta)
    assert sc == pytest.approx(best, abs=1e-12)


def _asymmetric_graph(n, rng):
    # a connected graph with a trivial automorphism group is typical for ER at
    # this density; we simply accept whatever automorphisms exist: the check is
    # on the objective value (reading Z25).
    return er_graph(n, 2 * n - 2, rng)


@pytest.mark.parametrize("seed", range(10))
def test_P12_recoverable_instances_reach_optimum(seed):
    rng = np.random.default_rng(500 + seed)
    n = 7
    A = _asymmetric_graph(n, rng)
    from synth import permuted_noisy_copy
    B, perm = permuted_noisy_copy(A, rng, noise=0.0)
    L = random_candidates(n, n, 3, rng, weights="uniform", truth=perm)
    alpha, beta = 0.1, 1.0
    opt, _ = best_alignment(A, B, L, alpha, beta)
    # the truth alignment is feasible and has overlap |E_A|
    truth_edges = [int(np.nonzero((L.a == a) & (L.b == perm[a]))[0][0]) for a in range(n)]
    sc_truth, _ = score_of(A, B, L, truth_edges, alpha, beta)
    assert opt >= sc_truth - 1e-12
    o = Oracle(A, B, L, alpha, beta)
    o.align(40, 0.99)
    _, best, _ = o.get_best()
    assert best <= opt + 1e-12
    assert best >= 0.8 * opt  # BP is a heuristic; recovery is typical, not guaranteed


@pytest.mark.parametrize("seed", range(6))
def test_P13_empty_S_reaches_assignment_optimum(seed):
    rng = np.random.default_rng(seed)
    n = 6
    L = complete_candidates(n, n, rng=rng)
    A, B = graph_from_edges(n, []), graph_from_edges(n, [])
    o = Oracle(A, B, L, 1.0, 2.0)
    assert o.s == 0
    o.align(60, 0.999)
    mate, best, _ = o.get_best()
    W = L.w.reshape(n, n)
    r, c = linear_sum_assignment(-W)
    assert best == pytest.approx(W[r, c].sum(), abs=1e-12)


@pytest.mark.parametrize("seed", range(6))
def test_P14_subgraph_isomorphism_setting(seed):
    rng = np.random.default_rng(900 + seed)
    n = 6
    A = er_graph(n, 7, rng)
    from synth import permuted_noisy_copy
    B, perm = permuted_noisy_copy(A, rng, noise=0.0)
    L = random_candidates(n, n, 3, rng, truth=perm)
    opt, _ = best_alignment(A, B, L, 0.0, 1.0)
    assert opt == A.n_edges
    o = Oracle(A, B, L, 0.0, 1.0)
    o.align(30, 0.99)
    _, best, _ = o.get_best()
    assert best <= A.n_edges


def test_Z8_selection_and_best_semantics():
    """M_y wins ties; best is updated only on a strictly greater score; bestM
    stays empty while no score exceeds 0 (reading Z8)."""
    n = 3
    A, B = graph_from_edges(n, []), graph_from_edges(n, [])
    L = complete_candidates(n, n, w=-np.ones(n * n))  # all weights negative
    o = Oracle(A, B, L, 1.0, 1.0)
    o.step(1.0, 0.0)
    info = o.round()
    assert info["score_y"] == 0.0 and info["score_z"] == 0.0
    assert info["source"] == 0 and info["improved"] == 0
    mate, best, it = o.get_best()
    assert best == 0.0 and it == 0 and np.all(mate == -1)


@pytest.mark.parametrize("reading", ["undamped", "damped"])
def test_P16_worked_example_W3_round_source(reading):
    """Worked example W3 (tests/golden/W3.json, reading Z5): the oracle's
    rounding uses y^c, z^c (Alg. 2 l.17/19) or, with
    ROUND_DAMPED, y^p, z^p (text :201).  At p = 2 the four greedy matchings
    differ and the two readings pick different sources, so swapping y and z
    or c and p fails here."""
    import oracle
    from fractions import Fraction
    from tests.util import load_golden, golden_instance
    g = load_golden("W3.json")
    A, B, L = golden_instance(g)
    gamma = float(Fraction(g["gamma"]))
    p2 = g["iterations"][1]
    assert len({tuple(p2["undamped"]["My"]), tuple(p2["undamped"]["Mz"]),
                tuple(p2["damped"]["My"]), tuple(p2["damped"]["Mz"])}) == 4
    assert p2["undamped"]["source"] != p2["damped"]["source"]
    o = Oracle(A, B, L, g["alpha"], g["beta"], oracle.ROUND_DAMPED if reading == "damped" else 0)
    for it in g["iterations"]:
        o.step_gamma(gamma)
        st = o.get_state()
        for key in ("d", "yc", "zc", "yp", "zp"):
            assert list(st[key]) == [float(Fraction(x)) for x in it[key]], (it["p"], key)
        info = o.round()
        want = it[reading]
        assert sorted(e for e in info["mate_y"] if e >= 0) == want["My"], it["p"]
        assert sorted(e for e in info["mate_z"] if e >= 0) == want["Mz"], it["p"]
        for k in ("score_y", "score_z", "weight_y", "weight_z", "best_score"):
            assert info[k] == float(Fraction(want[k])), (it["p"], k)
        for k in ("overlap_y", "overlap_z", "source", "best_iter"):
            assert info[k] == want[k], (it["p"], k)
    mate, best, best_it = o.get_best()
    last = g["iterations"][-1][reading]
    assert best == float(Fraction(last["best_score"])) and best_it == last["best_iter"]
    src = g["iterations"][best_it - 1][reading]
    want_best = src["My"] if src["source"] == 0 else src["Mz"]
    assert sorted(e for e in mate if e >= 0) == want_best
