"""NEXT-4 quality harness on the GPU (cualign_quality_eval through the C ABI)
against the quality oracle (oracle/quality.py): integer counts bit-exact,
ratios equal (same integers, same IEEE divisions)."""
import numpy as np
import pytest

from oracle.quality import quality as oracle_quality
from synth import make_config
from tests.util import graph_from_edges, load_golden

pytestmark = pytest.mark.gpu

KEYS_INT = ("n_a", "n_b", "edges_a", "edges_b", "aligned", "truth_total", "correct", "conserved", "induced")
KEYS_F = ("nc", "ec", "ics", "s3", "ncv", "gs3", "ncv_gs3")


@pytest.fixture(scope="module")
def ca():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_xiangkfah23_b200 as ca
    ca.load_library()
    return ca


def _same(g, o):
    for k in KEYS_INT:
        assert g[k] == o[k], (k, g[k], o[k])
    for k in KEYS_F:
        assert g[k] == pytest.approx(o[k], rel=1e-15, abs=0), k


def test_Q1_on_gpu(ca):
    g = load_golden("Q1.json")
    A = graph_from_edges(g["A"]["n"], g["A"]["edges"])
    B = graph_from_edges(g["B"]["n"], g["B"]["edges"])
    mp, tr = np.array(g["map"], np.int32), np.array(g["truth"], np.int32)
    _same(ca.quality(A, B, mp, tr), oracle_quality(A, B, mp, tr))


@pytest.mark.parametrize("name", ["T", "P10", "O005"])
def test_best_alignment_quality(ca, name):
    inst = {"T": lambda: make_config("T"), "P10": lambda: make_config("P", scale=0.1),
            "O005": lambda: make_config("O", scale=0.005)}[name]()
    mate, info, _ = ca.align(inst.A, inst.B, inst.L, inst.alpha, inst.beta, inst.gamma, n_iter=10)
    mp = ca.alignment_map(mate, inst.L)
    truth = np.asarray(inst.truth, dtype=np.int32)
    g = ca.quality(inst.A, inst.B, mp, truth)
    _same(g, oracle_quality(inst.A, inst.B, mp, truth))
    # the engine's best score is alpha w(M) + beta overlap(M) with overlap = conserved (Eq. 1, :68)
    sel = mate >= 0
    wsum = float(np.sum(inst.L.w[mate[sel]]))
    assert info["best_score"] == pytest.approx(inst.alpha * wsum + inst.beta * g["conserved"], rel=1e-12)


@pytest.mark.parametrize("seed", range(4))
def test_random_injective_maps(ca, seed):
    inst = make_config("P", scale=0.05)
    rng = np.random.default_rng(seed)
    k = int(rng.integers(0, inst.A.n + 1))
    mp = np.full(inst.A.n, -1, dtype=np.int32)
    mp[rng.choice(inst.A.n, k, replace=False)] = rng.choice(inst.B.n, k, replace=False)
    _same(ca.quality(inst.A, inst.B, mp, None), oracle_quality(inst.A, inst.B, mp, None))


def test_device_tensors(ca):
    import torch
    inst = make_config("T")
    mp = np.asarray(inst.truth, dtype=np.int32)

    class G:
        pass

    def dev(g):
        d = G()
        d.n, d.rowptr, d.col = g.n, torch.from_numpy(g.rowptr).cuda(), torch.from_numpy(g.col).cuda()
        return d

    g = ca.quality(dev(inst.A), dev(inst.B), torch.from_numpy(mp).cuda(), torch.from_numpy(mp).cuda())
    _same(g, oracle_quality(inst.A, inst.B, mp, mp))


def test_empty_and_invalid(ca):
    A = graph_from_edges(4, [[0, 1], [2, 3]])
    B = graph_from_edges(4, [[0, 1]])
    none = np.full(4, -1, dtype=np.int32)
    _same(ca.quality(A, B, none), oracle_quality(A, B, none))
    with pytest.raises(ca.CuAlignError):
        ca.quality(A, B, np.array([0, 0, -1, -1], np.int32))      # not injective
    with pytest.raises(ca.CuAlignError):
        ca.quality(A, B, np.array([0, 9, -1, -1], np.int32))      # out of range
    E = graph_from_edges(0, [])
    q = ca.quality(E, E, np.zeros(0, np.int32))
    assert q["aligned"] == 0 and q["ncv_gs3"] == 0.0
