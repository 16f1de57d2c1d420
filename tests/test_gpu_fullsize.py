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
