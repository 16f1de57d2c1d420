"""Order-independence of the square layout and the step pipeline.

* Square tiles: the squares are reordered into
  (e block, f block) tiles at init.  Every result is order-independent
  (integer fixed-point F sums, per-square arithmetic), so a run with tiny
  blocks (many tiles, cualign_params.square_tile_log) must equal the
  default run bit for bit.
* Step pipeline: run(n) overlaps the rounding of
  iteration k with iteration k+1 through double-buffered y^c, z^c; for every
  n (1, even, odd) and interleaved with eager calls the state, the last round
  and the best matching equal the eager sequence bit for bit.
"""
import os

import numpy as np
import pytest

from synth import make_config

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def ca():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_xiangkfah23_b200 as ca
    ca.load_library()
    return ca


def _run_tiles(ca, tile_log):
    inst = make_config("P", scale=0.1)
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma,
                      square_tile_log=tile_log) as h:
        h.run(7)
        st = h.get_state()
        rp, col = h.get_S()
        mate, info = h.get_best()
        out = {k: np.asarray(st[k]).view(np.uint64) for k in ("yc", "zc", "yp", "zp", "d", "Sp")}
        out["S"] = np.concatenate([rp, col])
        out["mate"] = np.asarray(mate)
        out["best"] = np.asarray([info["best_score"], info["best_iter"]])
    return out


def test_square_tiles_bitwise_invariant(ca):
    base = _run_tiles(ca, -1)      # plain (e, f) order
    tiled = _run_tiles(ca, 6)      # blocks of 64 edges: hundreds of tiles on P10
    default = _run_tiles(ca, 0)    # default block size
    for k in base:
        assert np.array_equal(base[k], tiled[k]), k
        assert np.array_equal(base[k], default[k]), k


def test_packed_square_chunks_across_f_blocks(ca):
    """m > 2^21 edges: the packed square stream cuts its chunks at 2^21-edge
    f blocks (and falls back to the int2 stream when an untiled order would
    make them tiny); every layout gives the same bits (DESIGN.md §5 "Packed
    square indices")."""
    inst = make_config("R", scale=0.5, k=5)
    assert inst.L.m > (1 << 21)
    outs = []
    for tile_log in (-1, 0, 12):
        with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma,
                          square_tile_log=tile_log) as h:
            h.run(4)
            st = h.get_state(with_S=False)
            outs.append({k: np.asarray(st[k]).view(np.uint64) for k in ("yc", "zc", "yp", "zp", "d")})
            outs[-1]["best"] = np.asarray([h.get_best()[1]["best_score"]])
    for o in outs[1:]:
        for k in outs[0]:
            assert np.array_equal(outs[0][k], o[k]), k


def _eager(ca, inst, n):
    h = ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma)
    infos = []
    for _ in range(n):
        h.iterate(1)
        infos.append(h.round())
    return h, infos


@pytest.mark.parametrize("n,schedule", [(1, 0), (2, 0), (5, 0), (6, 0), (21, 0), (24, 0), (40, 0),
                                        (7, 1), (7, 2), (7, 3), (40, 1), (40, 2), (40, 3)])
def test_pipelined_run_equals_eager(ca, n, schedule):
    """Every step schedule (cualign_params.schedule: 0 = the library's
    choice, 1 pipelined, 2 serial, 3 forked) for short and long runs."""
    inst = make_config("P", scale=0.1)
    h1, infos = _eager(ca, inst, n)
    with h1, ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, schedule=schedule) as h2:
        h2.run(n)
        s1, s2 = h1.get_state(), h2.get_state()
        for k in ("yc", "zc", "yp", "zp", "d", "Sp"):
            assert np.array_equal(s1[k], s2[k]), k
        m1, i1 = h1.get_best()
        m2, i2 = h2.get_best()
        assert np.array_equal(m1, m2)
        for k in ("iter", "best_score", "best_iter", "score_y", "score_z", "overlap_y", "overlap_z", "card_y",
                  "card_z", "source", "improved"):
            assert i1[k] == i2[k], (k, i1[k], i2[k])
        assert i2["iter"] == n


def test_pipelined_runs_interleaved_with_eager_calls(ca):
    inst = make_config("T")
    h1, _ = _eager(ca, inst, 9)
    with h1, ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma) as h2:
        h2.run(3)
        h2.iterate(1)
        h2.round()
        h2.run(1)
        h2.run(4)
        s1, s2 = h1.get_state(), h2.get_state()
        for k in ("yc", "zc", "yp", "zp", "d", "Sp"):
            assert np.array_equal(s1[k], s2[k]), k
        m1, i1 = h1.get_best()
        m2, i2 = h2.get_best()
        assert np.array_equal(m1, m2) and i1["best_score"] == i2["best_score"] and i1["iter"] == i2["iter"] == 9


@pytest.mark.parametrize("mode", ["pipelined", "damped", "shards3"])
def test_run_trace_infos_equal_step_by_step(ca, mode):
    """cualign_bp_run_trace (the e2e loop): every step's round info, copied to
    the host without a per-step synchronisation, equals the info of the
    eager iterate(1) + round() sequence; the final state is identical."""
    inst = make_config("P", scale=0.05)
    flags = ca.FLAG_ROUND_DAMPED if mode == "damped" else 0
    kw = {"world": 3} if mode == "shards3" else {}
    n = 23
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, flags) as h1, \
            ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, flags, **kw) as h2:
        eager = []
        for _ in range(n):
            h1.iterate(1)
            h1.round()
            eager.append(h1.get_best(with_mate=False)[1])
        traced = h2.run_trace(n)
        assert len(traced) == n
        for k in range(n):
            for key in ("iter", "score", "score_y", "score_z", "overlap_y", "overlap_z", "card_y", "card_z",
                        "source", "best_score", "best_iter"):
                assert eager[k][key] == traced[k][key], (k, key, eager[k][key], traced[k][key])
        m1, _ = h1.get_best()
        m2, _ = h2.get_best()
        assert np.array_equal(m1, m2)


def test_default_schedule_rule(ca):
    """cualign_params.schedule = 0: the library's rule (DESIGN.md §6 "Step
    graph and schedule"): pipelined whenever the rounding can be evaluated one
    step later (Suitor proposal rounds) -- small, dense (s/m = 20) and sparse
    (s/m = 5) instances alike; reported by cualign_sizes.schedule after a
    run."""
    small = make_config("T")
    dense = make_config("O", scale=0.2)
    sparse = make_config("R", scale=0.5, k=5)
    for inst in (small, dense, sparse):
        with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma) as h:
            h.run(3)
            assert h.sizes()["schedule"] == 1


@pytest.mark.parametrize("field,value", [("schedule", 4), ("schedule", -1), ("square_tile_log", 31),
                                         ("square_tile_log", -2)])
def test_tuning_params_validated(ca, field, value):
    inst = make_config("T", scale=0.2)
    with pytest.raises(ca.CuAlignError) as ei:
        ca.CuAlignBP(inst.A, inst.B, inst.L, **{field: value})
    assert ei.value.status == -1


def test_round_mates_and_sample_squares_contracts(ca):
    """get_round_mates before any rounding is ESTATE; sample_squares returns
    exactly the squares touching the sampled edges (S by its definition) on
    single and virtual-shard handles, and EINVAL on an id out of range."""
    from oracle.sample import SampledProblem
    inst = make_config("P", scale=0.05)
    sp = SampledProblem(inst.A, inst.B, inst.L)
    rng = np.random.default_rng(3)
    sample = rng.choice(inst.L.m, 40, replace=False).astype(np.int32)
    for kw in ({}, {"world": 3}):
        with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, **kw) as h:
            with pytest.raises(ca.CuAlignError) as ei:
                h.round_mates()
            assert ei.value.status == -5
            h.iterate(2)
            h.round()
            my, mz = h.round_mates()
            assert my.shape == (inst.A.n,) and mz.shape == (inst.A.n,)
            sq = h.sample_squares(sample)
            assert np.all(sq["e"] < sq["f"])
            for e in sample:
                got = sorted([int(f) for a, f in zip(sq["e"], sq["f"]) if a == e] +
                             [int(a) for a, f in zip(sq["e"], sq["f"]) if f == e])
                assert got == sp.S_row(int(e)), (kw, e)
            with pytest.raises(ca.CuAlignError) as ei:
                h.sample_squares(np.array([inst.L.m], np.int32))
            assert ei.value.status == -1
