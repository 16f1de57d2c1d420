"""Alg. 2 written in the matrix notation of the paper, on DENSE m x m matrices --
a second formulation used only to pin the oracle (tests only).

It follows PAPER.md:162-169 literally: F = bound_{0,beta}[beta*S + S^p^T] on the
whole matrix (entries off S's pattern come out 0 automatically: beta*0 + 0 = 0),
d = alpha*w + F e, y = d - othermaxcol(z^p), z = d - othermaxrow(y^p),
S^c = diag(y + z - d) S - F, damping.  No CSR, no transpose map: a transposed
index or a row/column mix-up in the sparse oracle disagrees with this.  Works on
Python Fractions (exact rationals) or floats.
"""
from __future__ import annotations

from fractions import Fraction


def othermax_by_group(v, group, literal=False):
    """om(e) over the other members of e's group (reading Z4)."""
    out = []
    for e in range(len(v)):
        others = [v[f] for f in range(len(v)) if f != e and group[f] == group[e]]
        if literal:
            out.append(max(others) if others else 0)
        else:
            out.append(max([0] + others))
    return out


def step(S, w, a, b, alpha, beta, g, h, state, literal=False):
    """One Alg. 2 iteration on dense lists-of-lists.  state = dict(yp, zp, Sp)."""
    m = len(w)
    Sp = state["Sp"]
    F = [[min(max(beta * S[e][f] + Sp[f][e], 0), beta) for f in range(m)] for e in range(m)]
    d = [alpha * w[e] + sum(F[e]) for e in range(m)]
    omc = othermax_by_group(state["zp"], b, literal)   # column = shared B vertex
    omr = othermax_by_group(state["yp"], a, literal)   # row = shared A vertex
    yc = [d[e] - omc[e] for e in range(m)]
    zc = [d[e] - omr[e] for e in range(m)]
    Sc = [[(yc[e] + zc[e] - d[e]) * S[e][f] - F[e][f] for f in range(m)] for e in range(m)]
    yp = [g * yc[e] + h * state["yp"][e] for e in range(m)]
    zp = [g * zc[e] + h * state["zp"][e] for e in range(m)]
    Spn = [[g * Sc[e][f] + h * Sp[e][f] for f in range(m)] for e in range(m)]
    return dict(F=F, d=d, yc=yc, zc=zc, yp=yp, zp=zp, Sp=Spn)


def zero_state(m, zero=Fraction(0)):
    return dict(yp=[zero] * m, zp=[zero] * m, Sp=[[zero] * m for _ in range(m)])
