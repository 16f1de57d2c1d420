"""NEXT-2: kNN sparsification on the tensor cores (cualign_knn, tcgen05 +
TMEM + bulk copies) against oracle/knn.py -- the paper's cosine similarity
(Alg. 1 l.9) in fp64.

The kernel multiplies unit vectors rounded to bf16 (unit roundoff 2^-8) and
accumulates in fp32 (2^-24); oracle.knn.dot_error_bound gives the rigorous
per-pair bound eps(u, v) on that computation's distance from the fp64 cosine.
The similarity decides a selection, so the comparison follows the "several
results are correct" rule: every GPU weight is within eps of the fp64 cosine
of its pair; with E = the row's largest eps, the GPU row contains every B
vertex whose cosine exceeds the row's k-th largest by more than 2E and
nothing below it by more than 2E; rows are k distinct B vertices in
ascending order.  Exactly representable cases (one-hot, duplicates, zero
rows) are compared bit for bit."""
import numpy as np
import pytest

from oracle.knn import cosine_fp64, dot_error_bound, knn as oracle_knn

pytestmark = pytest.mark.gpu

BF16_U, FP32_U = 2.0 ** -8, 2.0 ** -24


@pytest.fixture(scope="module")
def ca():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_sc_xiangkfah23_b200 as ca
    ca.load_library()
    return ca


def check_rows(rows, B, W, YA, YB, k):
    """rows: A vertex ids; B, W: the GPU's k neighbours / weights of them."""
    n_b = YB.shape[0]
    C = cosine_fp64(YA[rows], YB)
    eps = dot_error_bound(YA[rows], YB, BF16_U, FP32_U)
    assert np.all(np.diff(B, axis=1) > 0), "rows must be strictly ascending in b"
    assert np.all((B >= 0) & (B < n_b))
    r = np.arange(len(rows))[:, None]
    got = C[r, B]
    assert np.all(np.abs(W - got) <= eps[r, B]), float(np.max(np.abs(W - got) - eps[r, B]))
    E = eps.max(axis=1)[:, None]
    kth = -np.partition(-C, k - 1, axis=1)[:, k - 1][:, None]
    assert np.all(got >= kth - 2 * E), "selected a pair clearly outside the top-k"
    inside = C > kth + 2 * E
    sel = np.zeros_like(inside)
    sel[r, B] = True
    assert not np.any(inside & ~sel), "missed a pair clearly inside the top-k"
    return sel


def check(L, YA, YB, k):
    n_a = YA.shape[0]
    a, b, w = np.asarray(L.a), np.asarray(L.b), np.asarray(L.w)
    assert a.shape[0] == n_a * k
    assert np.array_equal(a, np.repeat(np.arange(n_a), k))
    return check_rows(np.arange(n_a), b.reshape(n_a, k), w.reshape(n_a, k), YA, YB, k)


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


def test_knn_full_size_sampled(ca):
    """The bench's kNN workload (n_A = n_B = 65536, d = 128, top-20, N(0,1)
    embeddings, device tensors) -- every row checked structurally, 64 sampled
    rows (incl. the first and last row blocks' edges) against the fp64
    cosine."""
    import torch
    n, d, k = 65536, 128, 20
    g = torch.Generator(device="cuda").manual_seed(20231112)
    YA = torch.randn(n, d, device="cuda", generator=g)
    YB = torch.randn(n, d, device="cuda", generator=g)
    L = ca.knn(YA, YB, k)
    a = L.a.cpu().numpy()
    b = L.b.cpu().numpy().reshape(n, k)
    w = L.w.cpu().numpy().reshape(n, k)
    assert np.array_equal(a, np.repeat(np.arange(n), k))
    assert np.all(np.diff(b, axis=1) > 0) and b.min() >= 0 and b.max() < n
    rng = np.random.default_rng(5)
    rows = np.unique(np.concatenate([[0, 127, 128, n - 129, n - 1], rng.choice(n, 59, replace=False)]))
    YAh, YBh = YA.cpu().double().numpy(), YB.cpu().double().numpy()
    check_rows(rows, b[rows], w[rows], YAh, YBh, k)
