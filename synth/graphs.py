"""Seeded graph-pair and candidate-graph generators (no method arithmetic).

Workload shape (§6.1): "For each graph A, we created a matching
pair B = P(A), by applying a random permutation P on the vertices of A".
Table 1 gives average degrees of 6-16 for the inputs.
Candidates L follow Alg. 1: k candidates per A vertex
with a similarity weight (honest kNN on structural features for the small
configs; a locality proxy for the large ones).

All arrays are numpy; graphs are symmetric CSR with int64 row pointers and
int32 sorted columns, no self loops, no duplicates (reading Z14).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass
class Graph:
    """Undirected simple graph as symmetric CSR (int64 rowptr, int32 col)."""
    n: int
    rowptr: np.ndarray
    col: np.ndarray

    @property
    def n_edges(self) -> int:
        return int(self.col.shape[0]) // 2

    def degrees(self) -> np.ndarray:
        return np.diff(self.rowptr)

    def edge_pairs(self):
        """Each undirected edge once as (u < v)."""
        u = np.repeat(np.arange(self.n, dtype=np.int64), self.degrees())
        v = self.col.astype(np.int64)
        keep = u < v
        return u[keep], v[keep]


@dataclass
class Candidates:
    """Bipartite candidate graph L: strictly increasing (a, b), weights w."""
    n_a: int
    n_b: int
    a: np.ndarray  # int32 [m]
    b: np.ndarray  # int32 [m]
    w: np.ndarray  # float64 [m]

    @property
    def m(self) -> int:
        return int(self.a.shape[0])


def _unique(x) -> np.ndarray:
    """Sorted distinct values of an int64 array (same result as np.unique;
    a plain sort: numpy's hash-based unique is ~10x slower at 10^8 keys)."""
    x = np.sort(np.asarray(x, dtype=np.int64).ravel())
    if x.shape[0] == 0:
        return x
    keep = np.empty(x.shape[0], dtype=bool)
    keep[0] = True
    np.not_equal(x[1:], x[:-1], out=keep[1:])
    return x[keep]


def _union(a, b) -> np.ndarray:
    return _unique(np.concatenate([np.asarray(a, dtype=np.int64), np.asarray(b, dtype=np.int64)]))


def _setdiff(a, b) -> np.ndarray:
    """Sorted distinct values of a that are not in b (as np.setdiff1d)."""
    a = _unique(a)
    b = _unique(b)
    pos = np.searchsorted(b, a)
    pos[pos >= b.shape[0]] = 0
    hit = (b.shape[0] > 0) & (b[pos] == a) if b.shape[0] else np.zeros(a.shape[0], dtype=bool)
    return a[~hit]


def csr_from_pairs(n: int, u, v) -> Graph:
    """Symmetrise, drop self loops and duplicates, return sorted CSR."""
    u = np.asarray(u, dtype=np.int64)
    v = np.asarray(v, dtype=np.int64)
    keep = u != v
    u, v = u[keep], v[keep]
    src = np.concatenate([u, v])
    dst = np.concatenate([v, u])
    key = _unique(src * n + dst)
    src = key // n
    dst = key % n
    rowptr = np.zeros(n + 1, dtype=np.int64)
    np.add.at(rowptr, src + 1, 1)
    rowptr = np.cumsum(rowptr).astype(np.int64)
    return Graph(n=n, rowptr=rowptr, col=dst.astype(np.int32))


def _dedupe_undirected(n, u, v):
    lo = np.minimum(u, v)
    hi = np.maximum(u, v)
    keep = lo != hi
    key = _unique(lo[keep] * n + hi[keep])
    return key


def er_graph(n: int, n_edges: int, rng: np.random.Generator) -> Graph:
    """Erdos-Renyi G(n, M): M distinct undirected edges chosen uniformly."""
    max_edges = n * (n - 1) // 2
    if n_edges > max_edges:
        raise ValueError("too many edges for ER graph")
    keys = np.zeros(0, dtype=np.int64)
    while keys.shape[0] < n_edges:
        need = n_edges - keys.shape[0]
        u = rng.integers(0, n, size=2 * need + 8)
        v = rng.integers(0, n, size=2 * need + 8)
        keys = _union(keys, _dedupe_undirected(n, u, v))
    keys = rng.permutation(keys)[:n_edges]
    return csr_from_pairs(n, keys // n, keys % n)


def chung_lu_graph(n: int, n_edges: int, tau: float, rng: np.random.Generator,
                   max_deg_frac: float = 0.02) -> Graph:
    """Chung-Lu power-law graph with exponent tau and ~n_edges distinct edges.

    Expected-degree weights w_i ∝ (i + i0)^(-1/(tau-1)); i0 is chosen so that
    the expected maximum degree is about max_deg_frac * n (keeps hubs bounded,
    like the PPI inputs of Table 1)."""
    gamma = 1.0 / (tau - 1.0)
    mean_deg = 2.0 * n_edges / n
    target_max = max(mean_deg * 2, max_deg_frac * n)
    i0 = 1.0
    for _ in range(60):  # bisection-free fixed point on the shift
        idx = np.arange(n, dtype=np.float64) + i0
        wts = idx ** (-gamma)
        ratio = wts[0] / wts.mean()
        if ratio * mean_deg <= target_max:
            break
        i0 *= 1.5
    prob = wts / wts.sum()
    keys = np.zeros(0, dtype=np.int64)
    while keys.shape[0] < n_edges:
        need = n_edges - keys.shape[0]
        u = rng.choice(n, size=int(need * 1.3) + 16, p=prob)
        v = rng.choice(n, size=int(need * 1.3) + 16, p=prob)
        keys = _union(keys, _dedupe_undirected(n, u, v))
    keys = rng.permutation(keys)[:n_edges]
    # random relabel so that hubs are not the low ids
    relabel = rng.permutation(n).astype(np.int64)
    return csr_from_pairs(n, relabel[keys // n], relabel[keys % n])


def rmat_graph(scale: int, edge_factor: int, probs, rng: np.random.Generator) -> Graph:
    """R-MAT (Graph500-style) graph: symmetrised, deduplicated, relabelled."""
    n = 1 << scale
    n_draw = edge_factor * n
    a, b, c, _ = probs
    u = np.zeros(n_draw, dtype=np.int64)
    v = np.zeros(n_draw, dtype=np.int64)
    for level in range(scale):
        r = rng.random(n_draw)
        right = (r >= a) & (r < a + b) | (r >= a + b + c)
        down = r >= a + b
        u |= down.astype(np.int64) << level
        v |= right.astype(np.int64) << level
    relabel = rng.permutation(n).astype(np.int64)
    return csr_from_pairs(n, relabel[u], relabel[v])


def induced_subgraph(g: Graph, keep: np.ndarray) -> Graph:
    """Subgraph induced on vertex set `keep` (relabelled 0..len(keep)-1 in that order)."""
    new_id = np.full(g.n, -1, dtype=np.int64)
    new_id[keep] = np.arange(keep.shape[0])
    u, v = g.edge_pairs()
    nu, nv = new_id[u], new_id[v]
    ok = (nu >= 0) & (nv >= 0)
    return csr_from_pairs(int(keep.shape[0]), nu[ok], nv[ok])


def permuted_noisy_copy(g: Graph, rng: np.random.Generator, noise: float = 0.05):
    """B = P(g) with ⌊noise·|E|⌋ edges deleted and as many random non-edges added.

    Returns (B, perm) with perm[v] = image of v in B."""
    n = g.n
    perm = rng.permutation(n).astype(np.int64)
    u, v = g.edge_pairs()
    pu, pv = perm[u], perm[v]
    n_e = u.shape[0]
    n_noise = int(np.floor(noise * n_e))
    keep = np.ones(n_e, dtype=bool)
    if n_noise > 0:
        keep[rng.choice(n_e, size=n_noise, replace=False)] = False
    lo = np.minimum(pu[keep], pv[keep])
    hi = np.maximum(pu[keep], pv[keep])
    existing = lo * n + hi
    all_existing = _union(existing, np.minimum(pu, pv) * n + np.maximum(pu, pv))
    added = np.zeros(0, dtype=np.int64)
    max_edges = n * (n - 1) // 2
    n_add = min(n_noise, max_edges - all_existing.shape[0])
    while added.shape[0] < n_add:
        need = n_add - added.shape[0]
        x = rng.integers(0, n, size=2 * need + 8)
        y = rng.integers(0, n, size=2 * need + 8)
        cand = _dedupe_undirected(n, x, y)
        cand = _setdiff(cand, all_existing)
        added = _union(added, cand)
    if added.shape[0] > n_add:
        added = rng.permutation(added)[:n_add]
    keys = np.concatenate([existing, added])
    return csr_from_pairs(n, keys // n, keys % n), perm


# ----------------------------------------------------------------------------
# candidate graphs L
# ----------------------------------------------------------------------------

def _finish_candidates(n_a, n_b, a, b, w) -> Candidates:
    a = np.asarray(a, dtype=np.int64)
    b = np.asarray(b, dtype=np.int64)
    order = np.lexsort((b, a))
    a, b, w = a[order], b[order], np.asarray(w, dtype=np.float64)[order]
    key = a * n_b + b
    if key.shape[0] > 1 and np.any(np.diff(key) <= 0):
        raise ValueError("duplicate candidate edges")
    return Candidates(n_a=n_a, n_b=n_b, a=a.astype(np.int32), b=b.astype(np.int32), w=w)


def _uniform01_open_low(rng, size):
    """U(0, 1]."""
    return 1.0 - rng.random(size)


def complete_candidates(n_a: int, n_b: int, w: np.ndarray | None = None,
                        rng: np.random.Generator | None = None) -> Candidates:
    """Complete bipartite L (canonical id = a*n_b + b)."""
    a = np.repeat(np.arange(n_a), n_b)
    b = np.tile(np.arange(n_b), n_a)
    if w is None:
        w = _uniform01_open_low(rng, n_a * n_b)
    return _finish_candidates(n_a, n_b, a, b, w)


def random_candidates(n_a: int, n_b: int, k: int, rng: np.random.Generator,
                      weights: str = "uniform", truth: np.ndarray | None = None) -> Candidates:
    """k distinct uniform candidates per A vertex (plus truth[a] if given)."""
    k = min(k, n_b)
    rows_a, rows_b = [], []
    for a in range(n_a):
        bs = rng.choice(n_b, size=k, replace=False)
        if truth is not None and truth[a] >= 0 and truth[a] not in bs:
            bs[0] = truth[a]
        rows_a.append(np.full(k, a))
        rows_b.append(bs)
    a = np.concatenate(rows_a)
    b = np.concatenate(rows_b)
    if weights == "uniform":
        w = _uniform01_open_low(rng, a.shape[0])
    elif weights == "ties":
        w = rng.integers(0, 4, size=a.shape[0]).astype(np.float64)
    elif weights == "ties_signed":
        w = rng.integers(-2, 4, size=a.shape[0]).astype(np.float64)
    elif weights == "int":
        w = rng.integers(1, 5, size=a.shape[0]).astype(np.float64)
    else:
        raise ValueError(weights)
    return _finish_candidates(n_a, n_b, a, b, w)


def _structural_features(g: Graph) -> np.ndarray:
    """Permutation-equivariant per-vertex features (log deg, mean log nbr deg,
    log 2-hop size, log triangles), standardised."""
    import scipy.sparse as sp
    n = g.n
    deg = g.degrees().astype(np.float64)
    adj = sp.csr_matrix((np.ones(g.col.shape[0]), g.col, g.rowptr), shape=(n, n))
    logdeg = np.log1p(deg)
    nbr_logdeg = np.zeros(n)
    nz = deg > 0
    nbr_logdeg[nz] = (adj @ logdeg)[nz] / deg[nz]
    a2 = adj @ adj
    a2.data[:] = 1.0
    two_hop = np.asarray(a2.sum(axis=1)).ravel()
    tri = np.asarray((adj.multiply(adj @ adj)).sum(axis=1)).ravel() / 2.0
    feats = np.stack([logdeg, nbr_logdeg, np.log1p(two_hop), np.log1p(tri)], axis=1)
    mu = feats.mean(axis=0)
    sd = feats.std(axis=0)
    sd[sd == 0] = 1.0
    return (feats - mu) / sd


def knn_candidates(ga: Graph, gb: Graph, k: int, rng: np.random.Generator,
                   jitter: float = 1e-3) -> Candidates:
    """Honest kNN (Alg. 1 l.7-14; reading Z19: top-k
    most similar per A vertex): full n_A x n_B cosine similarity of structural
    features (+ a tiny seeded jitter to break exact feature ties), top-k per A
    vertex, w = similarity clipped to (0, 1]."""
    fa = _structural_features(ga)
    fb = _structural_features(gb)
    fa = fa + jitter * rng.standard_normal(fa.shape)
    fb = fb + jitter * rng.standard_normal(fb.shape)
    fa /= np.maximum(np.linalg.norm(fa, axis=1, keepdims=True), 1e-12)
    fb /= np.maximum(np.linalg.norm(fb, axis=1, keepdims=True), 1e-12)
    k = min(k, gb.n)
    a_out, b_out, w_out = [], [], []
    chunk = max(1, int(2e7 // max(gb.n, 1)))
    for lo in range(0, ga.n, chunk):
        hi = min(ga.n, lo + chunk)
        sim = fa[lo:hi] @ fb.T
        idx = np.argpartition(-sim, k - 1, axis=1)[:, :k]
        rows = np.repeat(np.arange(lo, hi), k)
        cols = idx.ravel()
        vals = sim[np.arange(hi - lo)[:, None], idx].ravel()
        a_out.append(rows)
        b_out.append(cols)
        w_out.append(vals)
    w = np.clip(np.concatenate(w_out), 1e-6, 1.0)
    return _finish_candidates(ga.n, gb.n, np.concatenate(a_out), np.concatenate(b_out), w)


def proxy_candidates(gb: Graph, anchor: np.ndarray, k: float, lam: float,
                     rng: np.random.Generator, two_hop: float = 0.5) -> Candidates:
    """Locality-proxy candidates for the large configs.

    For each A vertex a: the anchor (the ground-truth image if defined, else a
    uniform B vertex) plus distinct draws that, with probability `lam`, come
    from the <=2-hop B-neighbourhood of the anchor and otherwise are uniform.
    k may be fractional: each row gets floor(k) or ceil(k) candidates.
    w ~ U(0, 1]."""
    n_a = anchor.shape[0]
    n_b = gb.n
    anchor = anchor.astype(np.int64).copy()
    undef = anchor < 0
    anchor[undef] = rng.integers(0, n_b, size=int(undef.sum()))
    k_lo = int(np.floor(k))
    k_row = k_lo + (rng.random(n_a) < (k - k_lo)).astype(np.int64)
    k_row = np.minimum(k_row, n_b)
    deg_b = np.diff(gb.rowptr)
    n_draw = int(np.ceil(k)) * 2 + 4
    a_rep = np.repeat(np.arange(n_a, dtype=np.int64), n_draw)
    anc = np.repeat(anchor, n_draw)
    local = rng.random(a_rep.shape[0]) < lam
    # one hop: random neighbour of the anchor
    d0 = deg_b[anc]
    has = local & (d0 > 0)
    pick = np.zeros(a_rep.shape[0], dtype=np.int64)
    off = (rng.random(a_rep.shape[0]) * np.maximum(d0, 1)).astype(np.int64)
    hop1 = np.where(has, gb.col[np.minimum(gb.rowptr[anc] + off, gb.col.shape[0] - 1)], 0)
    # optional second hop
    d1 = deg_b[hop1]
    second = has & (rng.random(a_rep.shape[0]) < two_hop) & (d1 > 0)
    off2 = (rng.random(a_rep.shape[0]) * np.maximum(d1, 1)).astype(np.int64)
    hop2 = gb.col[np.minimum(gb.rowptr[hop1] + off2, gb.col.shape[0] - 1)]
    pick = np.where(second, hop2, hop1)
    uni = rng.integers(0, n_b, size=a_rep.shape[0])
    b_draw = np.where(has, pick, uni)
    # anchors get top priority, then draws in random priority order
    all_a = np.concatenate([np.arange(n_a, dtype=np.int64), a_rep])
    all_b = np.concatenate([anchor, b_draw])
    prio = np.concatenate([np.full(n_a, -1.0), rng.random(a_rep.shape[0])])
    key = all_a * n_b + all_b
    order = np.lexsort((prio, key))
    key_s = key[order]
    first = np.ones(key_s.shape[0], dtype=bool)
    first[1:] = key_s[1:] != key_s[:-1]
    sel = order[first]
    u_a, u_b, u_p = all_a[sel], all_b[sel], prio[sel]
    order2 = np.lexsort((u_p, u_a))
    u_a, u_b = u_a[order2], u_b[order2]
    starts = np.searchsorted(u_a, np.arange(n_a))
    rank = np.arange(u_a.shape[0]) - starts[u_a]
    keep = rank < k_row[u_a]
    a_out, b_out = u_a[keep], u_b[keep]
    # top up rows that are short (tiny B neighbourhoods) with uniform draws
    cnt = np.bincount(a_out, minlength=n_a)
    short = np.nonzero(cnt < k_row)[0]
    if short.shape[0]:
        extra_a, extra_b = [], []
        have = set((a_out[np.isin(a_out, short)] * n_b + b_out[np.isin(a_out, short)]).tolist())
        for a in short.tolist():
            need = int(k_row[a] - cnt[a])
            while need > 0:
                bb = int(rng.integers(0, n_b))
                if a * n_b + bb not in have:
                    have.add(a * n_b + bb)
                    extra_a.append(a)
                    extra_b.append(bb)
                    need -= 1
        a_out = np.concatenate([a_out, np.asarray(extra_a, dtype=np.int64)])
        b_out = np.concatenate([b_out, np.asarray(extra_b, dtype=np.int64)])
    w = _uniform01_open_low(rng, a_out.shape[0])
    return _finish_candidates(n_a, n_b, a_out, b_out, w)


def small_world_power_law(n: int, h: int, n_random: int, tau: float,
                          rng: np.random.Generator, max_deg_frac: float = 0.01) -> Graph:
    """Clustered power-law graph: a ring lattice (each vertex joined to its h
    nearest ring neighbours on each side: high clustering, like the local
    structure of ontology / PPI networks) plus a Chung-Lu power-law layer of
    n_random edges (hubs).  Vertices are relabelled randomly."""
    base = np.arange(n, dtype=np.int64)
    us, vs = [], []
    for d in range(1, h + 1):
        us.append(base)
        vs.append((base + d) % n)
    ring_u = np.concatenate(us) if us else np.zeros(0, dtype=np.int64)
    ring_v = np.concatenate(vs) if vs else np.zeros(0, dtype=np.int64)
    if n_random > 0:
        cl = chung_lu_graph(n, n_random, tau, rng, max_deg_frac=max_deg_frac)
        cu, cv = cl.edge_pairs()
    else:
        cu = cv = np.zeros(0, dtype=np.int64)
    relabel = rng.permutation(n).astype(np.int64)
    u = relabel[np.concatenate([ring_u, cu])]
    v = relabel[np.concatenate([ring_v, cv])]
    return csr_from_pairs(n, u, v)
