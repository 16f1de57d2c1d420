"""NEXT-3: fp32 storage of the square messages S^p (CUALIGN_FLAG_FP32_S).

Bar (BASELINE.json:north_star): "within 1e-4 relative if an fp32 mode is
offered".  Arithmetic stays fp64; only S^p is rounded to fp32 when stored, so
  * one step from an injected state whose S^p is fp32-representable: every
    fp64 output (d, y^c, z^c, y^p, z^p) equals the oracle within 1e-12, and
    every stored S^p is the oracle's value rounded to fp32 (|err| <= 2^-24 |v|);
  * whole trajectories stay within 1e-4 relative of the fp64 oracle;
  * the sharded fp32 run equals the unsharded fp32 run bit for bit;
  * the rounding of fp32 messages gives the same matching as the oracle's
    greedy on the very same (GPU) message vector (bit-exact given identical
    messages)."""
import numpy as np
import pytest

from oracle import Oracle, LightOracle
from synth import make_config

pytestmark = pytest.mark.gpu

TOL32 = 1e-4


@pytest.fixture(scope="module")
def ca():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_xiangkfah23_b200 as ca
    ca.load_library()
    return ca


def _rel(got, want):
    scale = max(float(np.max(np.abs(want))) if want.size else 0.0, 1.0)
    return float(np.max(np.abs(got - want))) / scale if want.size else 0.0


def test_fp32_rejected_with_exact(ca):
    inst = make_config("T")
    with pytest.raises(Exception):
        ca.CuAlignBP(inst.A, inst.B, inst.L, flags=ca.FLAG_FP32_S | ca.FLAG_EXACT)


@pytest.mark.parametrize("name", ["P10", "O005"])
def test_fp32_one_step_from_fp32_state(ca, name):
    inst = make_config("P", scale=0.1) if name == "P10" else make_config("O", scale=0.005)
    o = Oracle(inst.A, inst.B, inst.L, inst.alpha, inst.beta)
    rng = np.random.default_rng(21)
    m, s = o.m, o.s
    yp, zp = rng.normal(size=m) * 3, rng.normal(size=m) * 3
    Sp = (rng.normal(size=s) * 2).astype(np.float32).astype(np.float64)
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, ca.FLAG_FP32_S) as h:
        o.set_state(yp, zp, Sp, 5)
        h.set_state(yp, zp, Sp, 5)
        assert np.array_equal(h.get_state()["Sp"], Sp)  # fp32-representable: stored exactly
        o.step_gamma(inst.gamma)
        h.iterate(1)
        g, oo = h.get_state(), o.get_state()
        for k in ("d", "yc", "zc", "yp", "zp"):
            assert _rel(g[k], oo[k]) <= 1e-12, k
        want32 = oo["Sp"].astype(np.float32).astype(np.float64)
        # the GPU's fp64 S^p may differ from the oracle's in the last bits (row-sum
        # order), so the fp32 rounding may land one fp32 ulp away
        err = np.abs(g["Sp"] - oo["Sp"])
        assert np.all(err <= 2.0 ** -23 * np.maximum(np.abs(oo["Sp"]), 1e-300) + 1e-12)
        assert np.mean(g["Sp"] == want32) > 0.99


@pytest.mark.parametrize("name,n_iter", [("T", 20), ("P10", 20), ("O005", 10)])
def test_fp32_trajectory_within_1e4(ca, name, n_iter):
    inst = {"T": lambda: make_config("T"), "P10": lambda: make_config("P", scale=0.1),
            "O005": lambda: make_config("O", scale=0.005)}[name]()
    o = Oracle(inst.A, inst.B, inst.L, inst.alpha, inst.beta)
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, ca.FLAG_FP32_S) as h:
        for p in range(1, n_iter + 1):
            o.step_gamma(inst.gamma)
            h.iterate(1)
            g, oo = h.get_state(), o.get_state()
            for k in ("d", "yc", "zc", "yp", "zp", "Sp"):
                e = _rel(g[k], oo[k])
                assert e <= TOL32, f"{name} p={p} {k}: {e:.3e}"
            # matching of the GPU's own fp32-mode messages: bit-exact vs greedy
            r = h.round()
            want, card = LightOracle(inst.L).greedy(g["yc"])
            assert r["card_y"] == card


@pytest.mark.parametrize("world", [2, 3])
def test_fp32_virtual_shards_bitwise(ca, world):
    inst = make_config("O", scale=0.01)
    f = ca.FLAG_FP32_S
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, f) as h1, \
            ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, f, world=world) as hs:
        for p in range(1, 7):
            h1.iterate(1)
            hs.iterate(1)
            a, b = h1.get_state(with_S=False), hs.get_state(with_S=False)
            for k in ("yc", "zc", "yp", "zp", "d"):
                assert np.array_equal(a[k], b[k]), (p, k)
            r1, rs = h1.round(), hs.round()
            for k in ("score_y", "overlap_y", "card_y", "best_score", "best_iter"):
                assert r1[k] == rs[k], (p, k)
        assert np.array_equal(h1.get_best()[0], hs.get_best()[0])


def test_fp32_graph_run_equals_step_by_step(ca):
    inst = make_config("P", scale=0.1)
    f = ca.FLAG_FP32_S
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, f) as h1, \
            ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, f) as h2:
        for _ in range(6):
            h1.iterate(1)
            h1.round()
        h2.run(6)
        a, b = h1.get_state(), h2.get_state()
        for k in ("yc", "zc", "yp", "zp", "d", "Sp"):
            assert np.array_equal(a[k], b[k]), k
        assert np.array_equal(h1.get_best()[0], h2.get_best()[0])
