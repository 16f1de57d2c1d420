"""Pin the sampled oracle (oracle/sample.py) to the full C oracle: on whole
instances it must reproduce S rows and one BP iteration bit for bit."""
import numpy as np
import pytest

import oracle
from oracle import Oracle, LightOracle
from oracle.sample import SampledProblem
from synth import make_config
from synth.state import sp_value, edge_values


@pytest.mark.parametrize("name,scale,literal", [("T", 1.0, False), ("T", 1.0, True), ("O", 0.002, False)])
def test_sampled_step_equals_full_oracle(name, scale, literal):
    inst = make_config(name, scale=scale)
    alpha, beta, g = 1.0, 2.0, 0.99 ** 7
    h = 1.0 - g
    o = Oracle(inst.A, inst.B, inst.L, alpha, beta, oracle.OTHERMAX_LITERAL if literal else 0)
    rowptr, col, _ = o.get_S()
    rows = np.repeat(np.arange(o.m), np.diff(rowptr))
    Sp = sp_value(rows, col, seed=5)
    yp, zp = edge_values(o.m, 3), edge_values(o.m, 4)
    o.set_state(yp, zp, Sp, 6)
    o.step(g, h)
    full = o.get_state()
    sp = SampledProblem(inst.A, inst.B, inst.L)
    rng = np.random.default_rng(0)
    for e in rng.choice(o.m, size=min(o.m, 60), replace=False):
        r = sp.step(int(e), alpha, beta, g, h, yp, zp, lambda a, b: sp_value(a, b, seed=5), literal)
        assert r["row"] == list(col[rowptr[e]:rowptr[e + 1]])
        for k in ("d", "yc", "zc", "yp", "zp"):
            assert r[k] == full[k][e], (e, k)
        assert r["Sp"] == list(full["Sp"][rowptr[e]:rowptr[e + 1]])


def test_light_oracle_greedy_equals_full():
    inst = make_config("T")
    o = Oracle(inst.A, inst.B, inst.L, 1.0, 2.0)
    lo = LightOracle(inst.L)
    x = np.random.default_rng(1).normal(size=inst.L.m)
    assert np.array_equal(o.greedy(x)[0], lo.greedy(x)[0])


def test_sp_value_is_a_function_of_the_pair():
    e = np.array([1, 5, 1, 9], dtype=np.int64)
    f = np.array([2, 3, 2, 9], dtype=np.int64)
    v = sp_value(e, f, seed=3)
    assert v[0] == v[2] and v[0] != v[1]
    assert np.all(v >= -4.0) and np.all(v < 2.0)
    assert sp_value(e, f, seed=4)[0] != v[0]


@pytest.mark.parametrize("name,scale", [("T", 1.0), ("O", 0.002), ("R", 1 / 256)])
def test_vectorised_S_row_equals_definition_loops(name, scale):
    inst = make_config(name, scale=scale, **({"k": 20} if name == "R" else {}))
    sp = SampledProblem(inst.A, inst.B, inst.L)
    o = Oracle(inst.A, inst.B, inst.L, 1.0, 2.0)
    rowptr, col, _ = o.get_S()
    rng = np.random.default_rng(3)
    deg = np.diff(inst.A.rowptr)[inst.L.a] * np.diff(inst.B.rowptr)[inst.L.b]
    sample = np.concatenate([rng.choice(inst.L.m, 80, replace=False), np.argsort(deg)[-10:]])
    for e in sample:
        want = list(col[rowptr[e]:rowptr[e + 1]])
        assert sp.S_row_vec(int(e)) == want == sp.S_row(int(e)), e
