"""Small random CSR matrices for brute-force pins and edge cases."""
from __future__ import annotations

import numpy as np
import torch

from .csr import CSR


def random_csr(m: int, n: int, density: float, seed: int, integer: bool = False,
               empty_rows: int = 0, zero_frac: float = 0.0, positive: bool = False) -> CSR:
    """Random pattern with given density.  Options: some forced-empty rows, a fraction
    of explicit (structural) zeros, integer values in {-3..3}\\{0}, or positive values."""
    rng = np.random.default_rng(seed)
    mask = rng.random((m, n)) < density
    if empty_rows and m:
        mask[rng.choice(m, size=min(empty_rows, m), replace=False), :] = False
    rows, cols = np.nonzero(mask)  # row-major -> sorted by (row, col)
    nnz = rows.size
    if integer:
        v = rng.integers(1, 4, size=nnz).astype(np.float64)
        if not positive:
            v *= np.where(rng.random(nnz) < 0.5, -1.0, 1.0)
    else:
        v = rng.random(nnz) + (0.25 if positive else -0.5)
    if zero_frac > 0:
        v[rng.random(nnz) < zero_frac] = 0.0
    row_ptr = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(rows, minlength=m), out=row_ptr[1:])
    return CSR(m, n, torch.from_numpy(row_ptr), torch.from_numpy(cols.astype(np.int32)), torch.from_numpy(v))
