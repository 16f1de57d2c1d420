"""Seeded synthetic inputs shared by the oracle tests, the GPU tests and bench.py.

This package holds NO arithmetic of the alignment method (no S, no BP, no
matching).  It only draws graph pairs (A, B = P(A) + noise) and candidate
bipartite graphs L with the shapes of the paper's workloads
(§6.1, Table 1; recipe in DESIGN.md "Input recipe").
Both the oracle (`oracle/`) and the CUDA path consume its arrays; neither
imports the other.
"""
from .graphs import (Graph, Candidates, csr_from_pairs, er_graph, chung_lu_graph, small_world_power_law,
                     rmat_graph, permuted_noisy_copy, induced_subgraph,
                     knn_candidates, proxy_candidates, complete_candidates,
                     random_candidates)
from .configs import CONFIGS, make_config, Instance, O_full_work

__all__ = ["Graph", "Candidates", "csr_from_pairs", "er_graph", "chung_lu_graph",
           "rmat_graph", "permuted_noisy_copy", "induced_subgraph", "knn_candidates",
           "proxy_candidates", "complete_candidates", "random_candidates",
           "CONFIGS", "make_config", "Instance"]
