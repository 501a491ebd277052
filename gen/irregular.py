"""Irregular power-law block-sparse matrix (config 4), emitted as CSR.

Recipe (built at 4x4-tile level, then every structurally present entry is emitted
as a CSR triplet; no format conversion code is involved — the generator decides
which entries exist):
  * BR = BC block rows/cols (default 2^18, i.e. 1,048,576 scalar rows);
  * tiles in block row I: k_I = min(cap, floor(u^(-1/(a-1)))), a = 2, u ~ U(0,1];
  * tile columns uniform in [0, BC), duplicates removed (so k_I is an upper bound);
  * per tile, popcount ~ U{1..16} with uniformly random bit positions;
  * values U[-1, 1) (or integers U{-3..3}\\{0} with integer=True).
"""
from __future__ import annotations

import numpy as np
import torch

from .csr import CSR


def irregular_block_sparse(BR: int = 1 << 18, BC: int | None = None, seed: int = 20240917,
                           cap: int = 8192, a: float = 2.0, integer: bool = False) -> CSR:
    if BC is None:
        BC = BR
    cap = min(cap, BC)
    rng = np.random.default_rng(seed)
    u = 1.0 - rng.random(BR)  # (0, 1]
    k = np.minimum(cap, np.floor(u ** (-1.0 / (a - 1.0)))).astype(np.int64)
    k = np.maximum(k, 1)
    rows_rep = np.repeat(np.arange(BR, dtype=np.int64), k)
    cols = rng.integers(0, BC, size=rows_rep.size, dtype=np.int64)
    key = np.unique(rows_rep * BC + cols)  # sorted by (row, col), unique
    trow = key // BC
    tcol = key % BC
    T = key.size
    pc = rng.integers(1, 17, size=T)
    ranks = rng.random((T, 16)).argsort(axis=1).argsort(axis=1)
    present = ranks < pc[:, None]  # (T, 16) bool, bit b = 4*r + c
    del ranks
    t_idx, bit = np.nonzero(present)
    del present
    rows = 4 * trow[t_idx] + bit // 4
    cols_s = 4 * tcol[t_idx] + bit % 4
    n_cols = 4 * BC
    order = np.argsort(rows * n_cols + cols_s, kind="stable")
    rows = rows[order]
    cols_s = cols_s[order]
    nnz = rows.size
    if integer:
        v = rng.integers(-3, 3, size=nnz)  # -3..2
        v = np.where(v >= 0, v + 1, v).astype(np.float64)  # {-3..-1, 1..3}
    else:
        v = rng.random(nnz) * 2.0 - 1.0
    counts = np.bincount(rows, minlength=4 * BR)
    row_ptr = np.zeros(4 * BR + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    return CSR(4 * BR, n_cols, torch.from_numpy(row_ptr), torch.from_numpy(cols_s.astype(np.int32)),
               torch.from_numpy(v))
