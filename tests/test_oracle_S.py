"""Pins P1-P4 for the oracle's S construction (§2; Alg. 3 :185-197).

P1 brute force over all (e, f) pairs with dense adjacency (oracle/brute.py).
P2 complete L => S = A (x) B (Kronecker, scipy.sparse.kron), s = nnz(A) nnz(B).
P3 general L => S = (A (x) B)[idx, idx] with idx = a*n_B + b; row counts = (A L B)_{a,b}.
P4 S symmetric ("structurally symmetric"), zero diagonal, tau an
   involution, raw overlap counts even.
"""
import numpy as np
import pytest
import scipy.sparse as sp

from oracle import Oracle
from oracle.brute import S_dense
from synth import complete_candidates, make_config
from tests.util import tiny_instance, S_from_csr


def _adj(g):
    return sp.csr_matrix((np.ones(g.col.shape[0]), g.col, g.rowptr), shape=(g.n, g.n))


@pytest.mark.parametrize("seed", range(8))
def test_P1_S_matches_definition_bruteforce(seed):
    A, B, L, _ = tiny_instance(seed, n=6, n_edges=8, k=3, n_b=5 + seed % 3)
    o = Oracle(A, B, L, 1.0, 2.0)
    rowptr, col, _ = o.get_S()
    assert np.array_equal(S_from_csr(rowptr, col, L.m), S_dense(A, B, L))
    # rows list f in strictly ascending order
    for e in range(L.m):
        assert np.all(np.diff(col[rowptr[e]:rowptr[e + 1]]) > 0)


@pytest.mark.parametrize("seed", range(4))
def test_P2_complete_L_is_kronecker(seed):
    rng = np.random.default_rng(100 + seed)
    from synth import er_graph
    A = er_graph(5 + seed, 6 + seed, rng)
    B = er_graph(4 + seed, 5 + seed, rng)
    L = complete_candidates(A.n, B.n, rng=rng)
    o = Oracle(A, B, L, 1.0, 1.0)
    rowptr, col, _ = o.get_S()
    K = sp.kron(_adj(A), _adj(B)).toarray().astype(np.int8)
    assert np.array_equal(S_from_csr(rowptr, col, L.m), K)
    assert o.s == A.col.shape[0] * B.col.shape[0]


@pytest.mark.parametrize("name,scale", [("T", 1.0), ("P", 0.1)])
def test_P3_general_L_submatrix_of_kronecker(name, scale):
    inst = make_config(name, scale=scale)
    A, B, L = inst.A, inst.B, inst.L
    o = Oracle(A, B, L, 1.0, 2.0)
    rowptr, col, _ = o.get_S()
    # row counts: nnz(S row (i,i')) = (A Lmat B)_{i,i'}
    Lmat = sp.csr_matrix((np.ones(L.m), (L.a, L.b)), shape=(A.n, B.n))
    ALB = (_adj(A) @ Lmat @ _adj(B)).tocsr()
    counts = np.asarray(ALB[L.a, L.b]).ravel()
    assert np.array_equal(np.diff(rowptr), counts.astype(np.int64))
    # entries: S = (A kron B)[idx, idx], idx = a*n_B + b; test on sampled rows
    idx = L.a.astype(np.int64) * B.n + L.b
    pos_of = {int(v): e for e, v in enumerate(idx)}
    Aad, Bad = _adj(A).tolil(), _adj(B).tolil()
    rng = np.random.default_rng(7)
    for e in rng.choice(L.m, size=min(L.m, 200), replace=False):
        i, ip = int(L.a[e]), int(L.b[e])
        want = sorted(pos_of[j * B.n + jp] for j in Aad.rows[i] for jp in Bad.rows[ip]
                      if j * B.n + jp in pos_of)
        assert list(col[rowptr[e]:rowptr[e + 1]]) == want


@pytest.mark.parametrize("seed", range(6))
def test_P4_symmetry_tau_involution(seed):
    A, B, L, _ = tiny_instance(seed, n=7, n_edges=10, k=4)
    o = Oracle(A, B, L, 1.0, 2.0)
    rowptr, col, tau = o.get_S()
    S = S_from_csr(rowptr, col, L.m)
    assert np.array_equal(S, S.T)
    assert np.all(np.diag(S) == 0)
    assert np.array_equal(tau[tau], np.arange(o.s))
    rows = np.repeat(np.arange(L.m), np.diff(rowptr))
    assert np.array_equal(col[tau], rows)
    # raw overlap count of any matching is even
    for x_seed in range(5):
        x = np.random.default_rng(x_seed).random(L.m)
        mate, _ = o.greedy(x)
        assert o.evaluate(mate)["raw"] % 2 == 0


def test_P4_edges_sharing_an_endpoint_never_overlap():
    """Consequence of Z14 (simple graphs, no self loops): S never couples two L
    edges that share an A or a B vertex."""
    inst = make_config("T")
    o = Oracle(inst.A, inst.B, inst.L, 1.0, 2.0)
    rowptr, col, _ = o.get_S()
    rows = np.repeat(np.arange(inst.L.m), np.diff(rowptr))
    assert not np.any(inst.L.a[rows] == inst.L.a[col])
    assert not np.any(inst.L.b[rows] == inst.L.b[col])
