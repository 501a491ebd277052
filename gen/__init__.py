"""Seeded synthetic input generators shared by the CUDA path's tests/bench and the oracle.

This module holds NONE of the method's arithmetic (no SpGEMM, SpMV, format
conversion, casting or V-cycle).  It only produces input matrices in CSR and
input vectors, with the shapes and structure of the workloads in
BASELINE.json `configs` (recipes: DESIGN.md "Input recipe").

  * stencils   — Dirichlet-eliminated Laplacians, lexicographic order, x fastest
                 (SURVEY §8(c) R27): 2D 5-point (4/-1), 3D 7-point (6/-1),
                 3D 27-point (26/-1); optional symmetric random SPD values.
  * aggregation— fixed piecewise-constant aggregation P and R = P^T built directly
                 from the grid (2x2x2 in 3D, 2x2 in 2D).
  * irregular  — power-law block-sparse matrix built at 4x4-tile level and
                 emitted as CSR (config 4).
  * vectors    — seeded x / b vectors.
  * random_csr — small random CSR matrices for brute-force pins.

Every generator is deterministic for a given seed.  Stencil generators are
written with torch integer ops so they run identically on CPU or CUDA.
"""
from .csr import CSR  # noqa: F401
from .stencils import laplacian_5pt, laplacian_7pt, laplacian_27pt, stencil  # noqa: F401
from .aggregation import aggregation_P, aggregation_R, aggregation_hierarchy  # noqa: F401
from .irregular import irregular_block_sparse  # noqa: F401
from .vectors import uniform_vector, integer_vector  # noqa: F401
from .random_csr import random_csr  # noqa: F401
from . import configs, partition  # noqa: F401
