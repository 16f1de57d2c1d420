"""Quality measures of an alignment -- TEST INFRASTRUCTURE ONLY (oracle for the
NEXT-4 harness; only tests/ and bench/tools may import it).

The paper scores alignments with NCV-GS^3 "which measures how well the edges
are conserved between two networks (i.e., overlaps) normalized by the sizes of
the networks" (definitions in its refs [18, 20]) against the
ground-truth permutation P of B = P(A).  Written out plainly,
for an alignment M: V_A -> V_B (partial, one-to-one):

  conserved  = #{ {i,j} in E_A : M(i), M(j) defined and {M(i), M(j)} in E_B }
               (the overlap of PAPER.md:60)
  induced    = #{ {u,v} in E_B : u, v both in M(V_A) }
  NC   = #{i : M(i) = P(i)} / #{i : P(i) defined}
  EC   = conserved / |E_A|
  ICS  = conserved / induced
  S3   = conserved / (|E_A| + induced - conserved)
  NCV  = (|M(V_A)| + |V_A aligned|) / (|V_A| + |V_B|) = 2|M| / (|V_A| + |V_B|)
  GS3  = S3 (for a one-to-one alignment the generalised score reduces to S3)
  NCV-GS3 = sqrt(NCV * GS3)
A ratio with a zero denominator is 0.  Pure Python over edge sets: obviously
correct, slow; pinned in tests/test_oracle_quality.py.
"""
from __future__ import annotations

import math


def _edges(g):
    """Undirected edge set {(i, j) : i < j} of a CSR graph."""
    out = set()
    for i in range(int(g.n)):
        for x in range(int(g.rowptr[i]), int(g.rowptr[i + 1])):
            j = int(g.col[x])
            if i < j:
                out.add((i, j))
    return out


def _ratio(a, b):
    return a / b if b > 0 else 0.0


def quality(A, B, map_ab, truth=None):
    EA, EB = _edges(A), _edges(B)
    M = {i: int(map_ab[i]) for i in range(int(A.n)) if int(map_ab[i]) >= 0}
    image = set(M.values())
    if len(image) != len(M):
        raise ValueError("alignment not one-to-one")
    conserved = 0
    for (i, j) in EA:
        if i in M and j in M:
            u, v = M[i], M[j]
            if (min(u, v), max(u, v)) in EB:
                conserved += 1
    induced = sum(1 for (u, v) in EB if u in image and v in image)
    truth_total = correct = 0
    if truth is not None:
        for i in range(int(A.n)):
            t = int(truth[i])
            if t >= 0:
                truth_total += 1
                if M.get(i, -1) == t:
                    correct += 1
    q = dict(n_a=int(A.n), n_b=int(B.n), edges_a=len(EA), edges_b=len(EB), aligned=len(M),
             truth_total=truth_total, correct=correct, conserved=conserved, induced=induced)
    q["nc"] = _ratio(correct, truth_total)
    q["ec"] = _ratio(conserved, len(EA))
    q["ics"] = _ratio(conserved, induced)
    q["s3"] = _ratio(conserved, len(EA) + induced - conserved)
    q["ncv"] = _ratio(2 * len(M), int(A.n) + int(B.n))
    q["gs3"] = q["s3"]
    q["ncv_gs3"] = math.sqrt(q["ncv"] * q["gs3"])
    return q
