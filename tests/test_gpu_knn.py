"""NEXT-2: kNN sparsification on the tensor cores (cualign_knn, tcgen05 +
TMEM + bulk copies) against oracle/knn.py.

The similarity is a float decision input, so the comparison follows the
"several results are correct" rule: every GPU weight equals the oracle's exact
similarity of the same pair within the fp32 accumulation bound TOL; the GPU
row set contains every B vertex the oracle ranks clearly inside the top-k
(> kth + 2 TOL) and nothing clearly outside (< kth - 2 TOL); rows are k
distinct B vertices in ascending order.  Exact cases (one-hot, duplicates,
zero rows) are compared bit for bit."""
import numpy as np
import pytest

from oracle.knn import similarity_bf16, knn as oracle_knn

pytestmark = pytest.mark.gpu

TOL = 2e-5   # |fp32 accumulation - exact| for d <= 256 unit bf16 vectors


@pytest.fixture(scope="module")
def ca():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_xiangkfah23_b200 as ca
    ca.load_library()
    return ca


def check(L, YA, YB, k):
    n_a, n_b = YA.shape[0], YB.shape[0]
    S = similarity_bf16(YA, YB)
    a, b, w = np.asarray(L.a), np.asarray(L.b), np.asarray(L.w)
    assert a.shape[0] == n_a * k
    assert np.array_equal(a, np.repeat(np.arange(n_a), k))
    B = b.reshape(n_a, k)
    W = w.reshape(n_a, k)
    assert np.all(np.diff(B, axis=1) > 0), "rows must be strictly ascending in b"
    assert np.all((B >= 0) & (B < n_b))
    got = S[np.arange(n_a)[:, None], B]
    assert np.max(np.abs(W - got)) <= TOL
    kth = -np.partition(-S, k - 1, axis=1)[:, k - 1]
    assert np.all(got >= kth[:, None] - 2 * TOL), "selected a pair clearly outside the top-k"
    inside = S > kth[:, None] + 2 * TOL
    sel = np.zeros_like(inside)
    sel[np.arange(n_a)[:, None], B] = True
    assert not np.any(inside & ~sel), "missed a pair clearly inside the top-k"
    return sel


@pytest.mark.parametrize("n_a,n_b,d,k", [(300, 1000, 64, 10), (129, 257, 100, 7), (500, 700, 128, 32),
                                         (64, 300, 256, 5), (200, 5000, 128, 1), (1, 33, 3, 32)])
def test_knn_random(ca, n_a, n_b, d, k):
    rng = np.random.default_rng(n_a + n_b + d + k)
    YA = rng.normal(size=(n_a, d)).astype(np.float32)
    YB = rng.normal(size=(n_b, d)).astype(np.float32)
    check(ca.knn(YA, YB, k), YA, YB, k)


def test_knn_one_hot_exact(ca):
    n, d = 300, 256
    rng = np.random.default_rng(7)
    perm = rng.permutation(n)
    YA = np.zeros((n, d), np.float32)
    YB = np.zeros((n, d), np.float32)
    YA[np.arange(n), perm % d] = rng.uniform(0.5, 4, n)
    YB[perm, perm % d] = rng.uniform(0.5, 4, n)
    L = ca.knn(YA, YB, 1)
    # collisions of perm % d share a direction: the lowest B index among them wins
    want_b = np.array([np.flatnonzero((np.arange(n) % d) == (perm[u] % d)).min() for u in range(n)])
    assert np.array_equal(L.b, want_b) and np.all(L.w == 1.0)
    a, b, w = oracle_knn(YA, YB, 1)
    assert np.array_equal(L.b, b) and np.array_equal(L.w, w)


def test_knn_ties_and_zero_rows(ca):
    rng = np.random.default_rng(8)
    x = rng.normal(size=64).astype(np.float32)
    YB = rng.normal(size=(600, 64)).astype(np.float32)
    YB[[5, 300, 301, 599]] = x                 # four identical B rows
    YA = np.stack([x, 2 * x, np.zeros(64, np.float32)])
    L = ca.knn(YA, YB, 3)
    B = np.asarray(L.b).reshape(3, 3)
    assert list(B[0]) == [5, 300, 301] and list(B[1]) == [5, 300, 301]
    assert list(B[2]) == [0, 1, 2] and np.all(np.asarray(L.w).reshape(3, 3)[2] == 0.0)


def test_knn_many_splits(ca):
    """Enough columns that every row block is split across many CTAs."""
    rng = np.random.default_rng(9)
    YA = rng.normal(size=(256, 128)).astype(np.float32)
    YB = rng.normal(size=(40000, 128)).astype(np.float32)
    check(ca.knn(YA, YB, 16), YA, YB, 16)


def test_knn_device_tensors_and_align(ca):
    import torch
    from synth import make_config
    inst = make_config("T")
    rng = np.random.default_rng(10)
    # embeddings of a noisy copy: A's rows near their images' rows in B
    YB = rng.normal(size=(inst.B.n, 32)).astype(np.float32)
    YA = (YB[inst.truth] + 0.3 * rng.normal(size=(inst.A.n, 32))).astype(np.float32)
    Lh = ca.knn(YA, YB, 8)
    Ld = ca.knn(torch.from_numpy(YA).cuda(), torch.from_numpy(YB).cuda(), 8)
    assert np.array_equal(Ld.b.cpu().numpy(), Lh.b) and np.array_equal(Ld.w.cpu().numpy(), Lh.w)
    mate, info, _ = ca.align(inst.A, inst.B, Lh, 1.0, 2.0, 0.99, n_iter=10)
    q = ca.quality(inst.A, inst.B, ca.alignment_map(mate, Lh), np.asarray(inst.truth, np.int32))
    assert q["nc"] > 0.5


def test_knn_rejects_bad_args(ca):
    Y = np.ones((4, 8), np.float32)
    with pytest.raises(ca.CuAlignError):
        ca.knn(Y, Y, 5)            # k > n_b
    with pytest.raises(ca.CuAlignError):
        ca.knn(np.ones((4, 300), np.float32), np.ones((4, 300), np.float32), 2)   # d > 256
    Z = Y.copy()
    Z[1, 3] = np.nan
    with pytest.raises(ca.CuAlignError):
        ca.knn(Z, Y, 2)
