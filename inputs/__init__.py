"""Seeded synthetic inputs shared by `oracle/` and the CUDA path.

Holds none of the method's arithmetic: graphs (CSR), BFS roots and queue-bench
item ids. See DESIGN.md "Input recipe".
"""
from .graphs import (CSR, csr_from_adjacency, edge_weights, edges_to_csr, grid_csr, grid_edges,
                     hash2, kronecker_csr, kronecker_edges, permute_ids, sample_roots,
                     tree4_csr, tree4_edges)
from .items import fingerprint, item_of

__all__ = [
    "CSR", "csr_from_adjacency", "edge_weights", "edges_to_csr", "grid_csr", "grid_edges", "hash2",
    "kronecker_csr", "kronecker_edges", "permute_ids", "sample_roots", "tree4_csr",
    "tree4_edges", "fingerprint", "item_of",
]
