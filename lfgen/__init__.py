"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

This module holds NONE of the method's arithmetic (no proposal, no confirmation,
no scan): it only builds sparse matrices in CSR form (symmetric, and for SURVEY.md §8(f)
f3 general non-symmetric ones) whose graphs are
shaped like the paper's workloads (Table 3 and the ANISO
stencils), following the recipes of SURVEY.md §8(d) "Concrete synthetic inputs".
Both `oracle/` and the product path consume its output; neither is imported here.

CSR layout: int64 rowptr[N+1], int32 col[Z], float32 val[Z],
columns ascending inside each row, diagonal stored, no duplicates.
"""
from .graphs import (  # noqa: F401
    CSR,
    splitmix64,
    edge_hash_u,
    csr_from_edges,
    grid2d_5pt,
    aniso2d,
    grid3d_7pt_aniso,
    grid3d_7pt_aniso_rows,
    fem27_bricks,
    chung_lu,
    grid3d_27pt,
    grid3d_27pt_slab_edges,
    grid3d_27pt_rows,
    grid3d_27pt_big,
    grid27_nnz,
    random_graph,
    directed_hash_u,
    nonsymmetric,
    config,
    CONFIG_NAMES,
)
