"""GPU parity: the CUDA path (through the C ABI) against the oracle, element by
element, on the same seeded inputs.

Bars (BASELINE.json:north_star):
  * S (row pointers, columns): bit-exact.
  * fp64 messages y^c, z^c, y^p, z^p, d, S^p: |gpu - oracle|_inf <= 1e-9 *
    max(|oracle|_inf, 1) every iteration (fast mode); bit-exact in
    CUALIGN_FLAG_EXACT mode and in the integer regime (P6).
  * matchings and integer overlap counts: bit-exact given identical messages.
"""
import numpy as np
import pytest

import oracle
from oracle import Oracle, gamma_power
from synth import make_config, random_candidates, complete_candidates
from tests.util import tiny_instance, graph_from_edges, load_golden, golden_instance, candidates_from_lists

pytestmark = pytest.mark.gpu

TOL = 1e-9


@pytest.fixture(scope="module")
def ca():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_xiangkfah23_b200 as ca
    ca.load_library()
    return ca


def rel_err(got, want):
    scale = max(float(np.max(np.abs(want))) if want.size else 0.0, 1.0)
    return float(np.max(np.abs(got - want))) / scale if want.size else 0.0


def assert_state_close(g, o, tol=TOL, keys=("d", "yc", "zc", "yp", "zp", "Sp"), where=""):
    for k in keys:
        e = rel_err(g[k], o[k])
        assert e <= tol, f"{where} {k}: rel err {e:.3e} > {tol}"


def assert_state_equal(g, o, keys=("d", "yc", "zc", "yp", "zp", "Sp"), where=""):
    for k in keys:
        bad = np.nonzero(g[k] != o[k])[0]
        assert bad.size == 0, f"{where} {k}: {bad.size} differ, first {bad[:5]} {g[k][bad[:3]]} vs {o[k][bad[:3]]}"


INSTANCES = {
    "T": lambda: make_config("T"),
    "P": lambda: make_config("P"),
    "P10": lambda: make_config("P", scale=0.1),
    "O005": lambda: make_config("O", scale=0.005),
}


# ---------------------------------------------------------------- a2: S build
@pytest.mark.parametrize("name", ["T", "P10", "O005"])
def test_S_bit_exact(ca, name):
    inst = INSTANCES[name]()
    o = Oracle(inst.A, inst.B, inst.L, inst.alpha, inst.beta)
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma) as h:
        rp, col = h.get_S()
        orp, ocol, _ = o.get_S()
        assert np.array_equal(rp, orp)
        assert np.array_equal(col, ocol)
        sz = h.sizes()
        assert sz["s"] == o.s and sz["squares"] * 2 == o.s


@pytest.mark.parametrize("seed", range(6))
def test_S_bit_exact_tiny_and_ragged(ca, seed):
    A, B, L, _ = tiny_instance(seed, n=9, n_edges=14, k=1 + seed % 5, n_b=5 + seed)
    o = Oracle(A, B, L, 1.0, 2.0)
    with ca.CuAlignBP(A, B, L, 1.0, 2.0, 0.9) as h:
        rp, col = h.get_S()
        orp, ocol, _ = o.get_S()
        assert np.array_equal(rp, orp) and np.array_equal(col, ocol)


def test_S_hub_rows_longer_than_a_warp(ca):
    """A star centre with 100 neighbours in A and B and complete-ish L: rows of
    S much longer than 32 and neighbour lists spanning many warp chunks."""
    n = 101
    edges = [(0, j) for j in range(1, n)] + [(j, j + 1) for j in range(1, n - 1)]
    A = graph_from_edges(n, edges)
    B = graph_from_edges(n, edges)
    rng = np.random.default_rng(3)
    L = random_candidates(n, n, 40, rng, truth=np.arange(n))
    o = Oracle(A, B, L, 1.0, 2.0)
    with ca.CuAlignBP(A, B, L, 1.0, 2.0, 0.9) as h:
        rp, col = h.get_S()
        orp, ocol, _ = o.get_S()
        assert np.array_equal(rp, orp) and np.array_equal(col, ocol)
        assert np.max(np.diff(rp)) > 64


def test_S_long_candidate_rows(ca):
    """The S build's group map: L rows longer than one
    group (> 32 candidates), groups cut by the sum of B degrees, a B hub whose
    degree alone exceeds the map (its edges take the binary-search path), hub
    A vertices, A vertices without candidates."""
    rng = np.random.default_rng(11)
    n_a, n_b = 90, 400
    ea = [(0, j) for j in range(1, 60)] + [(int(u), int(v)) for u, v in rng.integers(0, n_a, (300, 2)) if u != v]
    eb = [(0, j) for j in range(1, 300)] + [(1, j) for j in range(2, 120)] + \
        [(int(u), int(v)) for u, v in rng.integers(0, n_b, (900, 2)) if u != v]
    A = graph_from_edges(n_a, sorted(set((min(u, v), max(u, v)) for u, v in ea)))
    B = graph_from_edges(n_b, sorted(set((min(u, v), max(u, v)) for u, v in eb)))
    a, b = [], []
    for i in range(n_a):
        if i % 11 == 5:
            continue  # no candidates
        k = 140 if i % 3 == 0 else (65 if i % 3 == 1 else 12)
        cand = set(rng.choice(n_b, size=k, replace=False).tolist())
        if i % 2 == 0:
            cand.add(0)  # the B hub (degree 299 > the map's 256 inserts)
        for j in sorted(cand):
            a.append(i)
            b.append(int(j))
    L = candidates_from_lists(n_a, n_b, a, b, rng.uniform(0.1, 1.0, len(a)))
    o = Oracle(A, B, L, 1.0, 2.0)
    with ca.CuAlignBP(A, B, L, 1.0, 2.0, 0.9) as h:
        rp, col = h.get_S()
        orp, ocol, _ = o.get_S()
        assert np.array_equal(rp, orp) and np.array_equal(col, ocol)
        assert o.s > 1000


def test_S_heavy_vertex(ca):
    """An A hub whose candidate list (sum of its neighbours' L rows) exceeds
    the group-map build's limit: its rows go to the warp-per-e build, the
    other rows to the group map, all in one S (complete L: S = A (x) B)."""
    rng = np.random.default_rng(5)
    n_a, n_b = 130, 200
    ea = [(0, j) for j in range(1, n_a)] + [(int(u), int(v)) for u, v in rng.integers(1, n_a, (60, 2)) if u != v]
    eb = [(0, j) for j in range(1, 40)] + [(int(u), int(v)) for u, v in rng.integers(0, n_b, (500, 2)) if u != v]
    A = graph_from_edges(n_a, sorted(set((min(u, v), max(u, v)) for u, v in ea)))
    B = graph_from_edges(n_b, sorted(set((min(u, v), max(u, v)) for u, v in eb)))
    L = complete_candidates(n_a, n_b, rng.uniform(0.1, 1.0, n_a * n_b))
    o = Oracle(A, B, L, 1.0, 2.0)
    with ca.CuAlignBP(A, B, L, 1.0, 2.0, 0.9) as h:
        rp, col = h.get_S()
        orp, ocol, _ = o.get_S()
        assert np.array_equal(rp, orp) and np.array_equal(col, ocol)
        assert (n_a - 1) * n_b * n_b > 1 << 22  # vertex 0 is heavy: candidates x row length


# ------------------------------------------------------- a3-a6: BP iteration
def _run_both(ca, inst, n_iter, flags=0, gamma=None, alpha=None, beta=None, check=None):
    alpha = inst.alpha if alpha is None else alpha
    beta = inst.beta if beta is None else beta
    gamma = inst.gamma if gamma is None else gamma
    oflags = (oracle.OTHERMAX_LITERAL if flags & ca.FLAG_OTHERMAX_LITERAL else 0) | \
             (oracle.ROUND_DAMPED if flags & ca.FLAG_ROUND_DAMPED else 0)
    o = Oracle(inst.A, inst.B, inst.L, alpha, beta, oflags)
    h = ca.CuAlignBP(inst.A, inst.B, inst.L, alpha, beta, gamma, flags)
    for p in range(1, n_iter + 1):
        o.step_gamma(gamma)
        h.iterate(1)
        check(p, h.get_state(), o.get_state(), o, h)
    return o, h


@pytest.mark.parametrize("name,n_iter", [("T", 20), ("P10", 30), ("O005", 10), ("P", 100)])
def test_fast_mode_trajectory_within_1e9(ca, name, n_iter):
    """Every iteration within 1e-9 of the oracle (SURVEY §8(c) parity
    contract), T and P at BASELINE.json's full size and iteration count."""
    inst = INSTANCES[name]()

    def check(p, g, o, *_):
        assert_state_close(g, o, where=f"{name} p={p}")

    o, h = _run_both(ca, inst, n_iter, check=check)
    h.close()


@pytest.mark.parametrize("name,n_iter", [("T", 20), ("P10", 15)])
@pytest.mark.parametrize("literal", [False, True])
def test_exact_mode_trajectory_bitwise(ca, name, n_iter, literal):
    inst = INSTANCES[name]()
    flags = ca.FLAG_EXACT | (ca.FLAG_OTHERMAX_LITERAL if literal else 0)

    def check(p, g, o, *_):
        assert_state_equal(g, o, where=f"{name} p={p}")

    o, h = _run_both(ca, inst, n_iter, flags=flags, check=check)
    h.close()


@pytest.mark.parametrize("seed", range(3))
def test_integer_regime_fast_mode_bitwise(ca, seed):
    """P6: gamma = 1, integer alpha, beta, w: all values are integers, exact in
    any summation order -> the fast path equals the oracle bit for bit."""
    inst = make_config("T", seed=77 + seed)
    inst.L.w[:] = np.random.default_rng(seed).integers(1, 5, size=inst.L.m).astype(np.float64)

    def check(p, g, o, oo, hh):
        assert_state_equal(g, o, where=f"p={p}")
        ri = hh.round()
        ro = oo.round()
        for k in ("card_y", "card_z", "overlap_y", "overlap_z", "source", "improved", "best_iter"):
            assert ri[k] == ro[k], (p, k, ri[k], ro[k])
        for k in ("score_y", "score_z", "weight_y", "weight_z", "best_score"):
            assert ri[k] == ro[k], (p, k)

    o, h = _run_both(ca, inst, 12, gamma=1.0, alpha=2.0, beta=3.0, check=check)
    mate_g, _ = h.get_best()
    mate_o, _, _ = o.get_best()
    assert np.array_equal(mate_g, mate_o)
    h.close()


@pytest.mark.parametrize("name", ["P10", "O005"])
def test_one_step_parity_from_injected_state(ca, name):
    """set_state a random (y^p, z^p, S^p) into both, one iteration, compare."""
    inst = INSTANCES[name]()
    o = Oracle(inst.A, inst.B, inst.L, inst.alpha, inst.beta)
    rng = np.random.default_rng(11)
    m, s = o.m, o.s
    yp, zp = rng.normal(size=m) * 3, rng.normal(size=m) * 3
    Sp = rng.normal(size=s) * 2
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma) as h:
        for p in (7, 40):
            o.set_state(yp, zp, Sp, p)
            h.set_state(yp, zp, Sp, p)
            o.step_gamma(inst.gamma)
            h.iterate(1)
            g, oo = h.get_state(), o.get_state()
            assert_state_close(g, oo, tol=1e-12, where=f"p={p}")
            assert g["p"] == oo["p"] == p + 1


def test_get_state_roundtrip(ca):
    inst = make_config("T")
    rng = np.random.default_rng(5)
    with ca.CuAlignBP(inst.A, inst.B, inst.L) as h:
        Sp = rng.normal(size=h.s)
        yp, zp = rng.normal(size=h.m), rng.normal(size=h.m)
        h.set_state(yp, zp, Sp, 3)
        g = h.get_state()
        assert np.array_equal(g["Sp"], Sp) and np.array_equal(g["yp"], yp) and g["p"] == 3


# ------------------------------------------------------------ a7: matching
@pytest.mark.parametrize("seed", range(12))
@pytest.mark.parametrize("weights", ["ties", "ties_signed", "uniform"])
@pytest.mark.parametrize("schedule", ["suitor", "rounds"])
def test_matching_bit_exact_vs_greedy(ca, seed, weights, schedule):
    rng = np.random.default_rng(seed)
    n_a, n_b = int(rng.integers(5, 300)), int(rng.integers(5, 300))
    L = random_candidates(n_a, n_b, int(rng.integers(1, 12)), rng, weights=weights)
    o = Oracle(graph_from_edges(n_a, []), graph_from_edges(n_b, []), L, 1.0, 0.0)
    want, _ = o.greedy(L.w)
    flags = ca.FLAG_MATCH_ROUNDS if schedule == "rounds" else 0
    ma, mb, rounds = ca.match(L, n_a, n_b, L.w, flags=flags)
    assert np.array_equal(ma, want)
    # mate_b consistent with mate_a
    for a in range(n_a):
        if ma[a] >= 0:
            assert mb[L.b[ma[a]]] == ma[a]
    assert np.sum(mb >= 0) == np.sum(ma >= 0)


@pytest.mark.parametrize("schedule", ["suitor", "rounds"])
def test_matching_large_random(ca, schedule):
    rng = np.random.default_rng(0)
    n_a, n_b = 20000, 15000
    L = random_candidates(n_a, n_b, 12, rng, weights="uniform")
    o = Oracle(graph_from_edges(n_a, []), graph_from_edges(n_b, []), L, 1.0, 0.0)
    flags = ca.FLAG_MATCH_ROUNDS if schedule == "rounds" else 0
    for x in (L.w, np.round(L.w * 4) / 4):  # generic and massively tied weights
        want, _ = o.greedy(x)
        ma, _, rounds = ca.match(L, n_a, n_b, x, flags=flags)
        assert np.array_equal(ma, want)


@pytest.mark.parametrize("seed", range(6))
def test_matching_b_side_proposals(ca, seed):
    """Wide A rows, thin B columns: the Suitor schedule proposes from B."""
    rng = np.random.default_rng(40 + seed)
    n_a, n_b = 12, 400
    for weights in ("ties", "uniform"):
        L = random_candidates(n_a, n_b, 60, rng, weights=weights)
        o = Oracle(graph_from_edges(n_a, []), graph_from_edges(n_b, []), L, 1.0, 0.0)
        want, _ = o.greedy(L.w)
        ma, mb, _ = ca.match(L, n_a, n_b, L.w)
        assert np.array_equal(ma, want)
        for b in range(n_b):
            if mb[b] >= 0:
                assert ma[L.a[mb[b]]] == mb[b]


def test_round_schedules_agree_on_config(ca):
    """Suitor and pointer-round schedules give the same matchings and scores."""
    inst = make_config("O", scale=0.01)
    res = []
    for flags in (0, ca.FLAG_MATCH_ROUNDS):
        with ca.CuAlignBP(inst.A, inst.B, inst.L, flags=flags) as h:
            infos = []
            for _ in range(5):
                h.iterate(1)
                infos.append(h.round())
            res.append((infos, h.get_best()[0]))
    for a, b in zip(res[0][0], res[1][0]):
        for k in ("card_y", "card_z", "overlap_y", "overlap_z", "score_y", "score_z", "best_score"):
            assert a[k] == b[k], k
    assert np.array_equal(res[0][1], res[1][1])


def test_matching_empty_and_degenerate(ca):
    L = random_candidates(4, 4, 2, np.random.default_rng(1))
    ma, mb, _ = ca.match(L, 4, 4, -np.ones(L.m))   # nothing eligible
    assert np.all(ma == -1) and np.all(mb == -1)
    from synth import Candidates
    E = Candidates(3, 3, np.zeros(0, np.int32), np.zeros(0, np.int32), np.zeros(0))
    ma, mb, _ = ca.match(E, 3, 3, np.zeros(0))
    assert np.all(ma == -1)


# ------------------------------------------------ a7 + a8: round and best
@pytest.mark.parametrize("name,n_iter", [("T", 20), ("P10", 20)])
def test_round_matches_oracle(ca, name, n_iter):
    """Rounding on the GPU's own messages vs oracle rounding on the SAME
    messages (state injected), so matchings must be bit-exact."""
    inst = INSTANCES[name]()
    o = Oracle(inst.A, inst.B, inst.L, inst.alpha, inst.beta)
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma) as h:
        for p in range(1, n_iter + 1):
            h.iterate(1)
            r = h.round()
            g = h.get_state()
            my, cy = o.greedy(g["yc"])
            mz, cz = o.greedy(g["zc"])
            ey, ez = o.evaluate(my), o.evaluate(mz)
            gy, gz = h.round_mates()
            assert np.array_equal(gy, my) and np.array_equal(gz, mz), p
            assert r["card_y"] == cy and r["card_z"] == cz
            assert r["overlap_y"] == ey["overlap"] and r["overlap_z"] == ez["overlap"]
            assert abs(r["weight_y"] - ey["weight"]) <= 1e-12 * max(1, ey["weight"])
            assert abs(r["score_z"] - ez["score"]) <= 1e-12 * max(1, ez["score"])
            assert r["iter"] == p


@pytest.mark.parametrize("name,n_iter", [("T", 20), ("P10", 20)])
def test_round_damped_matches_oracle(ca, name, n_iter):
    """Reading Z5 variant (CUALIGN_FLAG_ROUND_DAMPED): the
    rounding takes y^p, z^p.  On the GPU's own messages, every round's M_y,
    M_z equal the oracle's greedy matchings of y^p, z^p bit for bit, and the
    round info equals the oracle's evaluation of them."""
    inst = INSTANCES[name]()
    o = Oracle(inst.A, inst.B, inst.L, inst.alpha, inst.beta, oracle.ROUND_DAMPED)
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, ca.FLAG_ROUND_DAMPED) as h:
        for p in range(1, n_iter + 1):
            h.iterate(1)
            r = h.round()
            g = h.get_state(with_S=False)
            my, cy = o.greedy(g["yp"])
            mz, cz = o.greedy(g["zp"])
            gy, gz = h.round_mates()
            assert np.array_equal(gy, my) and np.array_equal(gz, mz), p
            ey, ez = o.evaluate(my), o.evaluate(mz)
            assert r["card_y"] == cy and r["card_z"] == cz
            assert r["overlap_y"] == ey["overlap"] and r["overlap_z"] == ez["overlap"]
            assert abs(r["score_y"] - ey["score"]) <= 1e-12 * max(1, ey["score"])
            assert abs(r["score_z"] - ez["score"]) <= 1e-12 * max(1, ez["score"])
            assert r["source"] == (0 if r["score_y"] >= r["score_z"] else 1)


@pytest.mark.parametrize("reading", ["undamped", "damped"])
def test_W3_on_gpu(ca, reading):
    """Worked example W3 (tests/golden/W3.json): exact dyadic values, so the
    GPU's messages, matchings, scores and best equal the golden bit for bit
    under both readings of Z5."""
    from fractions import Fraction
    g = load_golden("W3.json")
    A, B, L = golden_instance(g)
    flags = ca.FLAG_ROUND_DAMPED if reading == "damped" else 0
    with ca.CuAlignBP(A, B, L, g["alpha"], g["beta"], float(Fraction(g["gamma"])), flags) as h:
        for it in g["iterations"]:
            h.iterate(1)
            st = h.get_state()
            for key in ("d", "yc", "zc", "yp", "zp"):
                assert list(st[key]) == [float(Fraction(x)) for x in it[key]], (it["p"], key)
            r = h.round()
            want = it[reading]
            gy, gz = h.round_mates()
            assert sorted(e for e in gy if e >= 0) == want["My"], it["p"]
            assert sorted(e for e in gz if e >= 0) == want["Mz"], it["p"]
            for k in ("score_y", "score_z", "weight_y", "weight_z", "best_score"):
                assert r[k] == float(Fraction(want[k])), (it["p"], k)
            for k in ("overlap_y", "overlap_z", "source", "best_iter"):
                assert r[k] == want[k], (it["p"], k)


@pytest.mark.parametrize("name", ["T", "P10"])
def test_end_to_end_align_exact_mode(ca, name):
    inst = INSTANCES[name]()
    n_iter = 20
    o = Oracle(inst.A, inst.B, inst.L, inst.alpha, inst.beta)
    oinfos = o.align(n_iter, inst.gamma)
    mate, info, infos = ca.align(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma,
                                 n_iter=n_iter, flags=ca.FLAG_EXACT)
    for gi, oi in zip(infos, oinfos):
        for k in ("card_y", "card_z", "overlap_y", "overlap_z", "source", "improved", "best_iter",
                  "score_y", "score_z", "weight_y", "weight_z", "best_score"):
            assert gi[k] == oi[k], (gi["iter"], k, gi[k], oi[k])
    omate, obest, oit = o.get_best()
    assert np.array_equal(mate, omate) and info["best_score"] == obest and info["best_iter"] == oit


def test_end_to_end_align_fast_mode(ca):
    inst = make_config("T")
    o = Oracle(inst.A, inst.B, inst.L, inst.alpha, inst.beta)
    oinfos = o.align(inst.n_iter, inst.gamma)
    mate, info, infos = ca.align(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma,
                                 n_iter=inst.n_iter)
    omate, obest, oit = o.get_best()
    assert abs(info["best_score"] - obest) <= 1e-9 * max(1.0, abs(obest))
    if not np.array_equal(mate, omate):  # only a near-tie may flip the choice
        gaps = [abs(oi["score_y"] - oi["score_z"]) for oi in oinfos]
        assert min(gaps) < 1e-9 * max(1.0, abs(obest))


@pytest.mark.parametrize("flags_name", ["fast", "exact", "rounds"])
def test_graph_run_equals_step_by_step(ca, flags_name):
    """cualign_bp_run (CUDA-graph replay of iterate+round) gives bit-identical
    state, round infos and best matching to the eager call sequence."""
    inst = INSTANCES["P10"]()
    flags = {"fast": 0, "exact": ca.FLAG_EXACT, "rounds": ca.FLAG_MATCH_ROUNDS}[flags_name]
    n = 12
    with ca.CuAlignBP(inst.A, inst.B, inst.L, flags=flags) as h1, \
            ca.CuAlignBP(inst.A, inst.B, inst.L, flags=flags) as h2:
        for _ in range(n):
            h1.iterate(1)
            h1.round(sync=False)
        h2.run(5)
        h2.set_timing(True)
        h2.run(4)               # timed graph variant
        h2.set_timing(False)
        h2.run(n - 9)
        s1, s2 = h1.get_state(), h2.get_state()
        assert_state_equal(s2, s1)
        assert s1["p"] == s2["p"] == n
        m1, i1 = h1.get_best()
        m2, i2 = h2.get_best()
        assert np.array_equal(m1, m2)
        for k in ("iter", "best_score", "best_iter", "score_y", "score_z", "overlap_y", "card_z"):
            assert i1[k] == i2[k], k
        st = h2.stats()
        assert st["class_ms"]["square"] > 0 and st["class_launches"]["square"] >= n


def test_graph_run_matches_oracle_exact(ca):
    inst = make_config("T")
    o = Oracle(inst.A, inst.B, inst.L, inst.alpha, inst.beta)
    oinfos = o.align(inst.n_iter, inst.gamma)
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, ca.FLAG_EXACT) as h:
        h.run(inst.n_iter)
        mate, info = h.get_best()
        assert_state_equal(h.get_state(), o.get_state())
    omate, obest, oit = o.get_best()
    assert np.array_equal(mate, omate) and info["best_score"] == obest and info["best_iter"] == oit
    assert info["iter"] == inst.n_iter and info["score"] == oinfos[-1]["score"]


# ------------------------------------------------------------ golden W1/W2
def test_W1_on_gpu(ca):
    from fractions import Fraction
    g = load_golden("W1.json")
    A, B, L = golden_instance(g)
    with ca.CuAlignBP(A, B, L, g["alpha"], g["beta"], float(Fraction(g["gamma"]))) as h:
        rp, col = h.get_S()
        for it in g["iterations"]:
            h.iterate(1)
            st = h.get_state()
            for key in ("d", "yc", "zc", "yp", "zp"):
                assert list(st[key]) == [float(Fraction(x)) for x in it[key]], (it["p"], key)
            vals = []
            for e, f in g["S_pairs"]:
                row = list(col[rp[e]:rp[e + 1]])
                vals.append(st["Sp"][rp[e] + row.index(f)])
            assert vals == [float(Fraction(x)) for x in it["Sp"]]
            r = h.round()
            assert r["score"] == 3.5 and r["overlap_y"] == 1
        _, info = h.get_best()
        assert info["best_score"] == 3.5 and info["best_iter"] == 1


@pytest.mark.parametrize("literal", [False, True])
def test_W2_on_gpu(ca, literal):
    g = load_golden("W2.json")
    A, B, L = golden_instance(g)
    flags = ca.FLAG_OTHERMAX_LITERAL if literal else 0
    with ca.CuAlignBP(A, B, L, g["alpha"], g["beta"], 1.0, flags) as h:
        for it in g["literal" if literal else "maxplus"]:
            h.iterate(1)
            st = h.get_state()
            assert list(st["yc"]) == [float(x) for x in it["yc"]]
            assert list(st["zc"]) == [float(x) for x in it["zc"]]
            h.round()
        _, info = h.get_best()
        assert info["best_score"] == 5 and info["best_iter"] == 1


# --------------------------------------------------------------- edge cases
def test_empty_L_and_edgeless_graphs(ca):
    from synth import Candidates
    A = graph_from_edges(3, [])
    B = graph_from_edges(4, [])
    E = Candidates(3, 4, np.zeros(0, np.int32), np.zeros(0, np.int32), np.zeros(0))
    with ca.CuAlignBP(A, B, E) as h:
        h.iterate(3)
        r = h.round()
        assert r["card_y"] == 0 and r["score"] == 0.0
        assert h.sizes()["s"] == 0


def test_n_a_differs_from_n_b(ca):
    inst = make_config("O", scale=0.002)
    assert inst.A.n != inst.B.n
    o = Oracle(inst.A, inst.B, inst.L, 1.0, 2.0)
    oinfos = o.align(5, 0.99)
    mate, info, infos = ca.align(inst.A, inst.B, inst.L, 1.0, 2.0, 0.99, n_iter=5, flags=ca.FLAG_EXACT)
    assert info["best_score"] == o.get_best()[1]


@pytest.mark.parametrize("bad", ["unsorted", "duplicate", "range", "asym", "selfloop", "nan", "alpha", "gamma"])
def test_validation_rejects_bad_inputs(ca, bad):
    inst = make_config("T", scale=0.2)
    A, B, L = inst.A, inst.B, inst.L
    kw = dict(alpha=1.0, beta=2.0, gamma=0.9)
    import copy
    L2 = copy.deepcopy(L)
    A2 = copy.deepcopy(A)
    if bad == "unsorted":
        L2.a, L2.b = L2.a[::-1].copy(), L2.b[::-1].copy()
    elif bad == "duplicate":
        L2.a[1], L2.b[1] = L2.a[0], L2.b[0]
    elif bad == "range":
        L2.b[-1] = B.n + 5
    elif bad == "asym":
        A2.col = A2.col.copy()
        i = int(np.argmax(np.diff(A2.rowptr) > 1))
        A2.col[A2.rowptr[i]] = (A2.col[A2.rowptr[i]] + 1) % A2.n  # breaks symmetry/order somewhere
    elif bad == "selfloop":
        A2.col = A2.col.copy()
        A2.col[A2.rowptr[0]] = 0
    elif bad == "nan":
        L2.w = L2.w.copy()
        L2.w[3] = np.nan
    elif bad == "alpha":
        kw["alpha"] = -1.0
    elif bad == "gamma":
        kw["gamma"] = 1.5
    with pytest.raises(ca.CuAlignError) as ei:
        ca.CuAlignBP(A2, B, L2, **kw)
    assert ei.value.status == -1
