"""Parity at BASELINE.json's full size (config O: m = 5.0e6 L edges, s = 1.0e8),
in the launch configuration bench.py times (the CUDA-graph step), checked on
outputs the oracle computes one by one:
  * S rows of sampled edges against the definition (oracle/sample.py);
  * one BP iteration from an injected seeded state at sampled edges (every
    output at the edge: d, y^c, z^c, y^p, z^p and the whole S^p row);
  * the matching of the full y^c against the C oracle's greedy (bit-exact,
    all 3e5 A vertices), and the round's overlap / cardinality against the
    definition of overlapped edges counted directly.
Inputs are seeded: S^p is a function of the (e, f) pair (synth/state.py), so
neither side's layout feeds the other."""
import numpy as np
import pytest

from oracle import LightOracle, gamma_power
from oracle.sample import SampledProblem
from synth import make_config
from synth.state import sp_value, edge_values

pytestmark = pytest.mark.gpu

TOL = 1e-12


@pytest.fixture(scope="module")
def full_O():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_xiangkfah23_b200 as ca
    ca.load_library()
    inst = make_config("O")
    stream = torch.cuda.Stream()
    h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=stream)
    yield ca, inst, h
    h.close()


def _close(a, b, scale):
    return abs(a - b) <= TOL * max(1.0, abs(scale))


def test_full_O_S_rows_sampled(full_O):
    ca, inst, h = full_O
    rowptr, col = h.get_S()
    assert rowptr[-1] == col.shape[0] == h.sizes()["s"]
    sp = SampledProblem(inst.A, inst.B, inst.L)
    rng = np.random.default_rng(11)
    sample = np.concatenate([rng.choice(inst.L.m, 150, replace=False),
                             [0, inst.L.m - 1, int(np.argmax(np.diff(rowptr)))]])
    for e in sample:
        assert list(col[rowptr[e]:rowptr[e + 1]]) == sp.S_row(int(e)), e


def test_full_O_one_step_from_injected_state(full_O):
    ca, inst, h = full_O
    rowptr, col = h.get_S()
    m = inst.L.m
    rows = np.repeat(np.arange(m, dtype=np.int64), np.diff(rowptr))
    Sp = sp_value(rows, col, seed=7)
    del rows
    yp, zp = edge_values(m, 8), edge_values(m, 9)
    p = 7
    h.set_state(yp, zp, Sp, p)
    del Sp
    h.run(1, with_round=False)  # the bench's graph step (iterate part)
    st = h.get_state()
    g = gamma_power(inst.gamma, p + 1)
    sp = SampledProblem(inst.A, inst.B, inst.L)
    rng = np.random.default_rng(12)
    sample = np.concatenate([rng.choice(m, 120, replace=False), [int(np.argmax(np.diff(rowptr)))]])
    fn = lambda a, b: sp_value(a, b, seed=7)
    for e in sample:
        e = int(e)
        r = sp.step(e, inst.alpha, inst.beta, g, 1.0 - g, yp, zp, fn)
        for k in ("d", "yc", "zc", "yp", "zp"):
            assert _close(st[k][e], r[k], r[k]), (e, k, st[k][e], r[k])
        got = st["Sp"][rowptr[e]:rowptr[e + 1]]
        for a, b in zip(got, r["Sp"]):
            assert _close(a, b, b), (e, a, b)


def test_full_O_matching_and_round(full_O):
    ca, inst, h = full_O
    h.run(2)  # iterate + round through the graph
    st = h.get_state(with_S=False)
    r = h.round()
    x = st["yc"]
    want, card = LightOracle(inst.L).greedy(x)
    got, _, _ = ca.match(inst.L, inst.L.n_a, inst.L.n_b, x)
    assert np.array_equal(got, want)
    assert r["card_y"] == card
    # overlap by the definition: A edges {i, j} with (M(i), M(j)) in E_B
    mb = np.full(inst.A.n, -1, dtype=np.int64)
    sel = want >= 0
    mb[sel] = inst.L.b[want[sel]]
    u, v = inst.A.edge_pairs()
    both = (mb[u] >= 0) & (mb[v] >= 0)
    bu, bv = mb[u][both], mb[v][both]
    keyB = np.sort(np.repeat(np.arange(inst.B.n, dtype=np.int64), np.diff(inst.B.rowptr)) * inst.B.n
                   + inst.B.col.astype(np.int64))
    k = bu * inst.B.n + bv
    pos = np.searchsorted(keyB, k)
    pos[pos >= keyB.shape[0]] = 0
    overlap = int(np.sum(keyB[pos] == k))
    assert r["overlap_y"] == overlap
    weight = float(np.sum(inst.L.w[want[sel]]))
    assert abs(r["weight_y"] - weight) <= 1e-12 * weight


# ------------------------------------------------ configs S and R, one step
# SURVEY §8(c) parity contract: one-step parity (bound 1e-12 of the vector's
# max norm) on O, S and R.  S^p of these instances (10^9 nonzeros) does not
# fit a host round trip, so the GPU's OWN state after 5 graph steps is the
# input: y^p, z^p in full (get_state) and S^p on the squares touching a
# sample of edges (cualign_bp_sample_squares); one more iteration of the
# bench's graph step; every output at the sampled edges (d, y^c, z^c, y^p,
# z^p and the whole new S^p row) against oracle/sample.py.  The sample holds
# random edges, the edges with the largest deg_A(a) deg_B(b) (longest rows),
# and edges of the highest-degree A and B vertices (R-MAT hub rows / columns).
ONE_STEP_TOL = 1e-12


def _sample_edges(inst, n_rand=150, seed=21):
    L, A, B = inst.L, inst.A, inst.B
    rng = np.random.default_rng(seed)
    dA, dB = np.diff(A.rowptr), np.diff(B.rowptr)
    prod = dA[L.a].astype(np.float64) * dB[L.b]
    long_rows = np.argsort(prod)[-20:]
    a_hub = int(np.argmax(np.bincount(L.a, minlength=L.n_a) * (dA > 0) + dA))  # A hub with candidates
    arow = np.searchsorted(L.a, [a_hub, a_hub + 1])
    hub_row = np.arange(arow[0], min(arow[1], arow[0] + 10))
    b_hub = int(np.argmax(dB))
    hub_col = np.nonzero(L.b == b_hub)[0][:10]
    s = np.concatenate([rng.choice(L.m, n_rand, replace=False), long_rows, hub_row, hub_col, [0, L.m - 1]])
    return np.unique(s.astype(np.int64))


def _one_step_large(name, **kw):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_xiangkfah23_b200 as ca
    ca.load_library()
    inst = make_config(name, **kw)
    stream = torch.cuda.Stream()
    sample = _sample_edges(inst)
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, stream=stream) as h:
        h.run(5)
        pre = h.get_state(with_S=False)
        sq0 = h.sample_squares(sample)
        h.run(1, with_round=False)
        post = h.get_state(with_S=False)
        sq1 = h.sample_squares(sample)
    assert (pre["p"], post["p"]) == (5, 6)
    val0, val1 = {}, {}
    for sq, val in ((sq0, val0), (sq1, val1)):
        for e, f, vef, vfe in zip(sq["e"], sq["f"], sq["v_ef"], sq["v_fe"]):
            val[(int(e), int(f))] = float(vef)
            val[(int(f), int(e))] = float(vfe)
    g = gamma_power(inst.gamma, 6)
    sp = SampledProblem(inst.A, inst.B, inst.L)
    scale = {k: max(float(np.max(np.abs(post[k]))), 1.0) for k in ("d", "yc", "zc", "yp", "zp")}
    sp_scale = max(max((abs(v) for v in val1.values()), default=0.0), 1.0)
    worst = 0.0
    for e in sample:
        e = int(e)
        r = sp.step(e, inst.alpha, inst.beta, g, 1.0 - g, pre["yp"], pre["zp"], lambda a, b: val0[(a, b)], vec=True)
        # structure: the squares touching e are exactly the S row by definition
        assert sorted(f for (a, f) in val1 if a == e) == r["row"], e
        for k in ("d", "yc", "zc", "yp", "zp"):
            err = abs(post[k][e] - r[k]) / scale[k]
            worst = max(worst, err)
            assert err <= ONE_STEP_TOL, (name, e, k, post[k][e], r[k])
        for f, want in zip(r["row"], r["Sp"]):
            err = abs(val1[(e, f)] - want) / sp_scale
            worst = max(worst, err)
            assert err <= ONE_STEP_TOL, (name, e, f, val1[(e, f)], want)
    return worst, len(sample)


@pytest.mark.slow
def test_config_S_one_step_sampled():
    worst, n = _one_step_large("S")
    assert n >= 150


@pytest.mark.slow
@pytest.mark.parametrize("k", [5, 50])
def test_config_R_one_step_sampled(k):
    worst, n = _one_step_large("R", k=k)
    assert n >= 150
