"""Fixed piecewise-constant aggregation operators.

Fine grid dims (x fastest).  Each coarse point aggregates a 2x2(x2) box of fine
points: fine (x, y, z) -> coarse (x//2, y//2, z//2) on a ceil(N/2) grid.
P is n_fine x n_coarse with exactly one entry (value alpha) per row; R = P^T is
emitted directly (coarse row c lists its fine points in ascending order).
alpha = 1/2 in 3D (keeps 27-point coarse values inside FP16 range), 1 in 2D.
"""
from __future__ import annotations

import itertools

import torch

from .csr import CSR


def _coarse_dims(dims):
    return tuple((d + 1) // 2 for d in dims)


def _lin(coords, dims):
    out = torch.zeros_like(coords[0])
    s = 1
    for c, d in zip(coords, dims):
        out = out + c * s
        s *= d
    return out


def default_alpha(dims) -> float:
    return 0.5 if len(dims) == 3 else 1.0


def aggregation_P(dims, alpha: float | None = None, device="cpu", rows=None) -> CSR:
    """rows=(r0, r1): only fine rows r0..r1-1 (global coarse column indices)."""
    dims = tuple(int(d) for d in dims)
    if alpha is None:
        alpha = default_alpha(dims)
    cd = _coarse_dims(dims)
    n = 1
    for d in dims:
        n *= d
    nc = 1
    for d in cd:
        nc *= d
    r0, r1 = (0, n) if rows is None else (int(rows[0]), int(rows[1]))
    idx = torch.arange(r0, r1, dtype=torch.int64, device=device)
    coords, rem = [], idx
    for d in dims:
        coords.append(rem % d)
        rem = rem // d
    ccol = _lin([c // 2 for c in coords], cd)
    m = r1 - r0
    row_ptr = torch.arange(m + 1, dtype=torch.int64, device=device)
    return CSR(m, nc, row_ptr, ccol.to(torch.int32), torch.full((m,), float(alpha), dtype=torch.float64, device=device))


def aggregation_R(dims, alpha: float | None = None, device="cpu") -> CSR:
    dims = tuple(int(d) for d in dims)
    if alpha is None:
        alpha = default_alpha(dims)
    cd = _coarse_dims(dims)
    nd = len(dims)
    nc = 1
    for d in cd:
        nc *= d
    n = 1
    for d in dims:
        n *= d
    cidx = torch.arange(nc, dtype=torch.int64, device=device)
    ccoords, rem = [], cidx
    for d in cd:
        ccoords.append(rem % d)
        rem = rem // d
    # children in ascending fine linear order: iterate offsets with the slowest dim outermost
    child_offsets = [tuple(reversed(o)) for o in itertools.product((0, 1), repeat=nd)]
    valids, fines = [], []
    count = torch.zeros(nc, dtype=torch.int64, device=device)
    for o in child_offsets:
        fc = [ccoords[k] * 2 + o[k] for k in range(nd)]
        v = torch.ones(nc, dtype=torch.bool, device=device)
        for k in range(nd):
            v &= fc[k] < dims[k]
        valids.append(v)
        fines.append(_lin(fc, dims))
        count += v
    row_ptr = torch.zeros(nc + 1, dtype=torch.int64, device=device)
    row_ptr[1:] = torch.cumsum(count, 0)
    nnz = int(row_ptr[-1])
    col = torch.empty(nnz, dtype=torch.int32, device=device)
    fill = row_ptr[:-1].clone()
    for v, f in zip(valids, fines):
        col[fill[v]] = f[v].to(torch.int32)
        fill += v
    return CSR(nc, n, row_ptr, col, torch.full((nnz,), float(alpha), dtype=torch.float64, device=device))


def aggregation_hierarchy(dims, nlev: int, alpha: float | None = None, device="cpu"):
    """[(P_1, R_1), ..., (P_{nlev-1}, R_{nlev-1})] for geometric 2x coarsening."""
    out = []
    d = tuple(int(x) for x in dims)
    for _ in range(nlev - 1):
        out.append((aggregation_P(d, alpha, device), aggregation_R(d, alpha, device)))
        d = _coarse_dims(d)
    return out
