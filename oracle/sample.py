"""Sampled oracle: one BP iteration evaluated edge by edge -- TEST
INFRASTRUCTURE ONLY (full-size parity on sampled outputs).

For a sampled L edge e, everything iteration p+1 produces at e follows from
the previous state and the definitions, without building S:
  S row e       by its definition (Alg. 3 :185-197): f = (j, j')
                with j in N_A(i), j' in N_B(i') ascending, (j, j') in L;
  F_ef          = bound_{0,beta}(beta + S^p_fe)          (Alg. 2 l.9, :162)
  d_e           = alpha w_e + sum_f F_ef, summed in ascending f from 0.0 (l.10, Z10)
  omc, omr      othermax of z^p over e's B column, of y^p over its A row (l.11-12, :203, Z4)
  y^c, z^c      = d - omc, d - omr
  S^c_ef        = (y^c + z^c - d) - F_ef                  (l.13)
  damping       y^p' = g y^c + h y^p, S^p'_ef = g S^c_ef + h S^p_ef (l.14-16)
in the same order of operations as oracle/cualign_oracle.c (Python floats are
IEEE doubles, no FMA), pinned against it in tests/test_oracle_sample.py.
S^p values come from a function sp(e, f) of the pair (synth/state.py).
"""
from __future__ import annotations

import numpy as np


class SampledProblem:
    def __init__(self, A, B, L):
        self.A, self.B, self.L = A, B, L
        self.key = L.a.astype(np.int64) * L.n_b + L.b.astype(np.int64)  # sorted (canonical order)
        self.arow = np.searchsorted(L.a, np.arange(L.n_a + 1))
        order = np.argsort(L.b, kind="stable")
        self.bedge = order
        self.bcol = np.searchsorted(L.b[order], np.arange(L.n_b + 1))

    def edge_id(self, j, jp):
        k = int(j) * self.L.n_b + int(jp)
        pos = int(np.searchsorted(self.key, k))
        return pos if pos < self.key.shape[0] and self.key[pos] == k else -1

    def S_row(self, e):
        """Row e of S by the definition (ascending f)."""
        i, ip = int(self.L.a[e]), int(self.L.b[e])
        A, B = self.A, self.B
        out = []
        for j in A.col[A.rowptr[i]:A.rowptr[i + 1]]:
            for jp in B.col[B.rowptr[ip]:B.rowptr[ip + 1]]:
                f = self.edge_id(j, jp)
                if f >= 0:
                    out.append(f)
        return out

    def S_row_vec(self, e):
        """Row e of S by the same definition, vectorised over the candidate
        pairs (for hub rows with 10^5-10^8 pairs): f = (j, j') in L with
        j in N_A(i) and j' in N_B(i'), ascending f (= ascending (j, j'), the
        canonical order).  Pinned against S_row (tests/test_oracle_sample.py)."""
        i, ip = int(self.L.a[e]), int(self.L.b[e])
        A, B = self.A, self.B
        J = A.col[A.rowptr[i]:A.rowptr[i + 1]].astype(np.int64)
        NB = B.col[B.rowptr[ip]:B.rowptr[ip + 1]].astype(np.int64)
        if J.shape[0] == 0 or NB.shape[0] == 0:
            return []
        lo, hi = self.arow[J], self.arow[J + 1]
        cnt = hi - lo
        f = np.repeat(lo - np.concatenate([[0], np.cumsum(cnt)[:-1]]), cnt) + np.arange(int(cnt.sum()))
        bf = self.L.b[f].astype(np.int64)
        hit = np.isin(bf, NB)
        return sorted(int(x) for x in f[hit])

    def othermax(self, edges, e, v, literal):
        others = [float(v[f]) for f in edges if f != e]
        if literal:
            om, found = 0.0, False
            for x in others:
                if not found or x > om:
                    om, found = x, True
            return om
        om = 0.0
        for x in others:
            if x > om:
                om = x
        return om

    def step(self, e, alpha, beta, g, h, yp, zp, sp, literal=False, vec=False):
        """Iteration outputs at edge e.  sp(e, f) -> S^p value of nonzero (e, f).
        vec: build the S row with S_row_vec (hub rows)."""
        L = self.L
        row = self.S_row_vec(e) if vec else self.S_row(e)
        F = []
        t = 0.0
        for f in row:
            val = beta + float(sp(f, e))
            if val < 0.0:
                val = 0.0
            if val > beta:
                val = beta
            F.append(val)
            t = t + val
        d = alpha * float(L.w[e]) + t
        a, b = int(L.a[e]), int(L.b[e])
        colB = [int(x) for x in self.bedge[self.bcol[b]:self.bcol[b + 1]]]
        rowA = list(range(int(self.arow[a]), int(self.arow[a + 1])))
        omc = self.othermax(colB, e, zp, literal)
        omr = self.othermax(rowA, e, yp, literal)
        yc = d - omc
        zc = d - omr
        u = (yc + zc) - d
        ypn = g * yc + h * float(yp[e])
        zpn = g * zc + h * float(zp[e])
        spn = [g * (u - F[k]) + h * float(sp(e, f)) for k, f in enumerate(row)]
        return dict(row=row, d=d, yc=yc, zc=zc, yp=ypn, zp=zpn, Sp=spn)
