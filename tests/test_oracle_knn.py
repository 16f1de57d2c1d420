"""Pins of the kNN oracle (oracle/knn.py, NEXT-2; Alg. 1 l.7-14, PAPER.md:121,
:133-140): closed forms (unit norms, one-hot and planar-angle embeddings),
scale invariance, the library routine (scikit-learn brute-force cosine kNN)
where neighbours are well separated, and the error bound used to judge a
low-precision implementation: it holds for bf16-rounded inputs with fp32
accumulation (torch CPU) and is attained to within a small factor (not
vacuous)."""
import math

import numpy as np
import pytest
import torch

from oracle.knn import (unit_rows, cosine_fp64, dot_error_bound, knn_from_similarity, knn)


def test_unit_rows_closed_form():
    Y = np.array([[3.0, 4.0], [0.0, 0.0], [-2.0, 0.0]])
    U = unit_rows(Y)
    assert np.array_equal(U, [[0.6, 0.8], [0.0, 0.0], [-1.0, 0.0]])
    rng = np.random.default_rng(1)
    Z = rng.normal(size=(20, 7))
    assert np.allclose(np.linalg.norm(unit_rows(Z), axis=1), 1.0, atol=1e-15)


def test_one_hot_embeddings_recover_permutation():
    n, d = 12, 16
    rng = np.random.default_rng(2)
    perm = rng.permutation(n)
    YA = np.zeros((n, d))
    YB = np.zeros((n, d))
    for u in range(n):
        YA[u, perm[u]] = rng.uniform(0.5, 4.0)       # scale does not matter
        YB[perm[u], perm[u]] = rng.uniform(0.5, 4.0)
    S = cosine_fp64(YA, YB)
    assert np.array_equal(S, (np.arange(n)[None, :] == perm[:, None]).astype(float))
    a, b, w = knn(YA, YB, 1)
    assert np.array_equal(a, np.arange(n)) and np.array_equal(b, perm) and np.all(w == 1.0)


def test_planar_angles_closed_form():
    th_a = np.array([0.0, 1.0, 2.5])
    th_b = np.array([0.1, 0.9, 2.0, 3.0, -0.5])
    YA = np.stack([np.cos(th_a), np.sin(th_a)], 1) * 3.0
    YB = np.stack([np.cos(th_b), np.sin(th_b)], 1) * 0.5
    C = cosine_fp64(YA, YB)
    assert np.allclose(C, np.cos(th_a[:, None] - th_b[None, :]), atol=1e-15)
    a, b, _ = knn_from_similarity(C, 2)
    # nearest angles: 0.0 -> {0.1, -0.5}; 1.0 -> {0.9, 0.1}; 2.5 -> {2.0, 3.0}
    assert [list(b[a == u]) for u in range(3)] == [[0, 4], [0, 1], [2, 3]]


def test_ties_go_to_lower_index_and_canonical_order():
    S = np.array([[0.5, 0.9, 0.5, 0.9, 0.1]])
    a, b, w = knn_from_similarity(S, 3)
    assert list(b) == [0, 1, 3] and list(w) == [0.5, 0.9, 0.9]


def test_scale_invariance_power_of_two():
    rng = np.random.default_rng(3)
    YA, YB = rng.normal(size=(15, 8)), rng.normal(size=(30, 8))
    s = 2.0 ** rng.integers(-5, 6, size=(15, 1))
    assert np.array_equal(cosine_fp64(YA, YB), cosine_fp64(YA * s, YB))


def test_against_sklearn_cosine_knn():
    from sklearn.neighbors import NearestNeighbors
    rng = np.random.default_rng(4)
    n_b, d, k = 200, 32, 5
    YB = rng.normal(size=(n_b, d))
    # queries close to chosen B rows so that the k nearest are well separated
    YA = YB[rng.choice(n_b, 40, replace=False)] + 0.01 * rng.normal(size=(40, d))
    nn = NearestNeighbors(n_neighbors=k, metric="cosine", algorithm="brute").fit(YB)
    _, idx = nn.kneighbors(YA)
    for S in (cosine_fp64(YA, YB),):
        a, b, _ = knn_from_similarity(S, k)
        for u in range(40):
            assert set(b[a == u]) == set(idx[u]), u


@pytest.mark.parametrize("d", [3, 64, 128, 256])
def test_dot_error_bound_holds_for_bf16_fp32(d):
    """The bound of dot_error_bound (unit roundoff 2^-8 inputs, 2^-24
    accumulation) covers bf16-rounded unit vectors multiplied with fp32
    accumulation, and is within 2^5 of the observed worst error."""
    rng = np.random.default_rng(d)
    YA, YB = rng.normal(size=(60, d)), rng.normal(size=(90, d))
    C = cosine_fp64(YA, YB)
    bound = dot_error_bound(YA, YB, 2.0 ** -8, 2.0 ** -24)
    ua = torch.from_numpy(unit_rows(YA)).to(torch.bfloat16).to(torch.float32)
    ub = torch.from_numpy(unit_rows(YB)).to(torch.bfloat16).to(torch.float32)
    got = (ua @ ub.T).double().numpy()
    err = np.abs(got - C)
    assert np.all(err <= bound)
    assert np.max(err / bound) > 2.0 ** -5


def test_dot_error_bound_exact_inputs():
    """One-hot rows are exact in any format: the bound is tiny but positive."""
    Y = np.eye(4)
    b = dot_error_bound(Y, Y, 2.0 ** -8, 2.0 ** -24)
    assert np.all(b > 0) and np.all(b[~np.eye(4, dtype=bool)] <= 1e-15 + 1e-18)
