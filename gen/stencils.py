"""Dirichlet-eliminated finite-difference Laplacians on regular grids.

Ordering is lexicographic with x fastest: point (x, y, z) -> x + Nx*(y + Ny*z).
Columns within a row are emitted in ascending order.  Works on any torch device.

Symmetric random SPD variant (config 2): off-diagonal (i, j) gets
-(0.5 + u(min(i,j), max(i,j))) with u a counter-based uniform in [0, 1) keyed by the
unordered pair and the seed; the diagonal is the sum of |off-diagonals| + 1.
"""
from __future__ import annotations

import itertools

import torch

from .csr import CSR

_MASK64 = (1 << 64) - 1


def _to_i64(c: int) -> int:
    c &= _MASK64
    return c - (1 << 64) if c >= (1 << 63) else c


def _lsr(x: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of int64 tensors (torch >> is arithmetic)."""
    return (x >> k) & ((1 << (64 - k)) - 1)


def splitmix64(x: torch.Tensor) -> torch.Tensor:
    """Counter-based 64-bit mixer (int64 wraparound arithmetic)."""
    x = x + _to_i64(0x9E3779B97F4A7C15)
    x = (x ^ _lsr(x, 30)) * _to_i64(0xBF58476D1CE4E5B9)
    x = (x ^ _lsr(x, 27)) * _to_i64(0x94D049BB133111EB)
    return x ^ _lsr(x, 31)


def pair_uniform(i: torch.Tensor, j: torch.Tensor, seed: int) -> torch.Tensor:
    """Uniform [0,1) float64 keyed by the unordered pair {i, j} and seed."""
    lo = torch.minimum(i, j).long()
    hi = torch.maximum(i, j).long()
    h = splitmix64(splitmix64(lo * _to_i64(0x100000001B3) + _to_i64(seed * 0x9E37 + 1)) ^ hi)
    return _lsr(h, 11).to(torch.float64) * (2.0 ** -53)


def stencil(dims, offsets, center: float, off: float, device="cpu", spd_seed: int | None = None,
            rows=None) -> CSR:
    """Generic constant-coefficient stencil matrix on a grid of `dims` (x fastest).
    rows=(r0, r1): generate only rows r0..r1-1 (global column indices kept)."""
    dims = tuple(int(d) for d in dims)
    nd = len(dims)
    strides = [1]
    for d in dims[:-1]:
        strides.append(strides[-1] * d)
    n = 1
    for d in dims:
        n *= d
    # sort offsets by linear offset -> ascending column order within a row
    offs = sorted(offsets, key=lambda o: sum(o[k] * strides[k] for k in range(nd)))
    r0, r1 = (0, n) if rows is None else (int(rows[0]), int(rows[1]))
    idx = torch.arange(r0, r1, dtype=torch.int64, device=device)
    m = r1 - r0
    coords = []
    rem = idx
    for k in range(nd):
        coords.append(rem % dims[k])
        rem = rem // dims[k]
    valids = []
    count = torch.zeros(m, dtype=torch.int64, device=device)
    for o in offs:
        v = torch.ones(m, dtype=torch.bool, device=device)
        for k in range(nd):
            if o[k] != 0:
                c = coords[k] + o[k]
                v &= (c >= 0) & (c < dims[k])
        valids.append(v)
        count += v
    row_ptr = torch.zeros(m + 1, dtype=torch.int64, device=device)
    row_ptr[1:] = torch.cumsum(count, 0)
    nnz = int(row_ptr[-1])
    col = torch.empty(nnz, dtype=torch.int32, device=device)
    val = torch.empty(nnz, dtype=torch.float64, device=device)
    fill = row_ptr[:-1].clone()
    for o, v in zip(offs, valids):
        lin = sum(o[k] * strides[k] for k in range(nd))
        rows = idx[v]
        pos = fill[v]
        col[pos] = (rows + lin).to(torch.int32)
        if lin == 0:
            val[pos] = center
        else:
            if spd_seed is None:
                val[pos] = off
            else:
                val[pos] = -(0.5 + pair_uniform(rows, rows + lin, spd_seed))
        fill += v
    del valids
    if spd_seed is not None:
        # diagonal = sum |off-diagonals| + 1 (strictly diagonally dominant -> SPD)
        rows_all = torch.repeat_interleave(idx, count)
        is_diag = col.long() == rows_all
        absoff = torch.where(is_diag, torch.zeros_like(val), val.abs())
        rowsum = torch.zeros(m, dtype=torch.float64, device=device).index_add_(0, rows_all - r0, absoff)
        val[is_diag] = rowsum + 1.0
    return CSR(m, n, row_ptr, col, val)


OFFS_5PT = [(0, 0), (1, 0), (-1, 0), (0, 1), (0, -1)]
OFFS_7PT = [(0, 0, 0), (1, 0, 0), (-1, 0, 0), (0, 1, 0), (0, -1, 0), (0, 0, 1), (0, 0, -1)]
OFFS_27PT = list(itertools.product((-1, 0, 1), repeat=3))


def laplacian_5pt(N: int, device="cpu", spd_seed=None, rows=None) -> CSR:
    return stencil((N, N), OFFS_5PT, 4.0, -1.0, device, spd_seed, rows)


def laplacian_7pt(N: int, device="cpu", spd_seed=None, rows=None, dims=None) -> CSR:
    """7-point Laplacian on N^3 (or on `dims` = (Nx, Ny, Nz))."""
    return stencil(dims or (N, N, N), OFFS_7PT, 6.0, -1.0, device, spd_seed, rows)


def laplacian_27pt(N: int, device="cpu", spd_seed=None, rows=None, dims=None) -> CSR:
    return stencil(dims or (N, N, N), OFFS_27PT, 26.0, -1.0, device, spd_seed, rows)
