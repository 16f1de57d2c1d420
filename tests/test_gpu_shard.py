"""Sharded path on one GPU: `world` virtual shards in one handle
exchange through device copies exactly where process shards use NCCL.  The
sharded run must equal the unsharded run BIT FOR BIT (integer F sums, exact
max merges, replicated deterministic rounding)."""
import numpy as np
import pytest

from synth import make_config
from oracle import Oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ca():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_xiangkfah23_b200 as ca
    ca.load_library()
    return ca


def _compare_runs(ca, inst, world, n_iter, flags=0):
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, flags) as h1, \
            ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, flags, world=world) as hs:
        rp1, col1 = h1.get_S()
        rps, cols = hs.get_S()
        assert np.array_equal(rp1, rps) and np.array_equal(col1, cols)
        for p in range(1, n_iter + 1):
            h1.iterate(1)
            hs.iterate(1)
            a, b = h1.get_state(with_S=False), hs.get_state(with_S=False)
            for k in ("yc", "zc", "yp", "zp", "d"):
                bad = np.nonzero(a[k] != b[k])[0]
                assert bad.size == 0, f"world={world} p={p} {k}: {bad.size} differ"
            r1, rs = h1.round(), hs.round()
            for k in ("score_y", "score_z", "overlap_y", "overlap_z", "card_y", "card_z", "best_score",
                      "best_iter", "source", "iter"):
                assert r1[k] == rs[k], (p, k)
        m1, _ = h1.get_best()
        ms, _ = hs.get_best()
        assert np.array_equal(m1, ms)
        sz = hs.sizes()
        assert sz["world"] == world and sz["s"] == h1.sizes()["s"]


@pytest.mark.parametrize("world", [2, 3, 4])
def test_virtual_shards_bitwise_T(ca, world):
    _compare_runs(ca, make_config("T"), world, 12)


@pytest.mark.parametrize("world", [2, 5])
def test_virtual_shards_bitwise_O_small(ca, world):
    _compare_runs(ca, make_config("O", scale=0.01), world, 8)


def test_virtual_shards_literal_and_damped(ca):
    inst = make_config("P", scale=0.05)
    _compare_runs(ca, inst, 3, 6, ca.FLAG_OTHERMAX_LITERAL | ca.FLAG_ROUND_DAMPED)


def test_virtual_shards_more_shards_than_rows(ca):
    """Tiny instance, many shards: some shards own no edge at all."""
    from tests.util import load_golden, golden_instance
    g = load_golden("W1.json")
    A, B, L = golden_instance(g)
    inst = make_config("T", scale=0.05)
    _compare_runs(ca, inst, 8, 5)


def test_virtual_shards_match_oracle(ca):
    inst = make_config("T")
    o = Oracle(inst.A, inst.B, inst.L, inst.alpha, inst.beta)
    o.align(inst.n_iter, inst.gamma)
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, world=4) as hs:
        hs.run(inst.n_iter)
        mate, info = hs.get_best()
    omate, obest, _ = o.get_best()
    assert abs(info["best_score"] - obest) <= 1e-9 * max(1.0, obest)


def test_shard_partition_whole_rows(ca):
    inst = make_config("O", scale=0.01)
    with ca.CuAlignBP(inst.A, inst.B, inst.L, world=3) as hs:
        sz = hs.sizes()
        assert sz["rank"] == -1 and sz["edge_begin"] == 0 and sz["edge_end"] == inst.L.m


def test_sharded_rejects_exact_and_set_state(ca):
    inst = make_config("T", scale=0.2)
    with pytest.raises(ca.CuAlignError):
        ca.CuAlignBP(inst.A, inst.B, inst.L, flags=ca.FLAG_EXACT, world=2)
    with ca.CuAlignBP(inst.A, inst.B, inst.L, world=2) as hs:
        with pytest.raises(ca.CuAlignError) as ei:
            hs.set_state(np.zeros(inst.L.m), np.zeros(inst.L.m), np.zeros(hs.s), 0)
        assert ei.value.status == -5


@pytest.mark.parametrize("world", [3, 8])
def test_sharded_rounding_merge_rounds(ca, world):
    """NEXT-1: rounding sharded by A rows (proposals local, B suitors merged by
    all-reduce MAX/MIN per round) equals the single-GPU greedy matching bit for
    bit, after several merge rounds on an instance with cross-shard conflicts."""
    inst = make_config("O", scale=0.02)
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma) as h1, \
            ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, world=world) as hs:
        for p in range(1, 6):
            h1.iterate(1)
            hs.iterate(1)
            r1, rs = h1.round(), hs.round()
            for k in ("card_y", "card_z", "overlap_y", "overlap_z", "score_y", "score_z", "best_score"):
                assert r1[k] == rs[k], (p, k)
            assert hs.sizes()["merge_rounds"] >= 2
            assert h1.sizes()["merge_rounds"] == 0
        st = hs.get_state(with_S=False)
        from oracle import LightOracle
        want, card = LightOracle(inst.L).greedy(st["yc"])
        got, _, _ = ca.match(inst.L, inst.L.n_a, inst.L.n_b, st["yc"])
        assert np.array_equal(got, want)
        assert np.array_equal(h1.get_best()[0], hs.get_best()[0])


@pytest.mark.parametrize("world", [2, 5])
@pytest.mark.parametrize("damped", [False, True])
def test_sharded_round_mates_equal_oracle_greedy(ca, world, damped):
    """NEXT-1 against the oracle directly: every round's sharded M_y and M_z
    (the replicated result of the merge rounds) equal the oracle's greedy
    matching (readings Z6/Z7) of the y^c, z^c (y^p, z^p
    under ROUND_DAMPED, reading Z5) gathered from the shards, and the round's
    cardinalities / overlaps equal the oracle's evaluation of them."""
    from oracle import LightOracle
    inst = make_config("O", scale=0.02)
    flags = ca.FLAG_ROUND_DAMPED if damped else 0
    lo = LightOracle(inst.L)
    o = Oracle(inst.A, inst.B, inst.L, inst.alpha, inst.beta)
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, flags, world=world) as hs:
        for p in range(1, 6):
            hs.iterate(1)
            r = hs.round()
            st = hs.get_state(with_S=False)
            my, mz = hs.round_mates()
            wy, cy = lo.greedy(st["yp" if damped else "yc"])
            wz, cz = lo.greedy(st["zp" if damped else "zc"])
            assert np.array_equal(my, wy), (p, "M_y")
            assert np.array_equal(mz, wz), (p, "M_z")
            assert r["card_y"] == cy and r["card_z"] == cz
            ey, ez = o.evaluate(wy), o.evaluate(wz)
            assert r["overlap_y"] == ey["overlap"] and r["overlap_z"] == ez["overlap"], p


def test_exchange_accounting_virtual_shards(ca):
    """Bytes the shards receive per iteration: the B-side
    top-2 all-gather, (w-1)·n_B·16 per shard, plus the square-pass halo (u_f
    of the remote f a shard's squares touch, and their F sums back to the
    owners) -- strictly less than all-gathering u and reducing full F-sum
    vectors, (w-1)·16·m summed over the shards."""
    inst = make_config("O", scale=0.01)
    w = 3
    with ca.CuAlignBP(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, world=w) as h:
        h.stats(reset=True)
        h.iterate(2)
        st = h.stats(reset=True)
        m, nB = inst.L.m, inst.B.n
        top2 = 2 * w * (w - 1) * nB * 16
        halo = st["comm_bytes_in"] - top2
        assert 0 < halo < 2 * (w - 1) * 16 * m
        assert halo % 16 == 0  # every halo entry moves once each way (8 B u + 8 B F sum)
        assert st["comm_calls"] > 0
