"""Synthetic matrices shaped like the paper's Table II (§8(f) NEXT-3): the
16 SuiteSparse matrices are not available here, so each is replaced by a seeded symmetric
M-matrix with exactly the printed order and number of nonzeros (TSOPF_RS_b300_c3: one fewer —
its printed nnz - order is odd, which no symmetric pattern with a full diagonal reaches).

Recipe: K positive diagonal offsets — the first half consecutive
(1, 2, ...: mesh-neighbour couplings), the rest spread geometrically up to n^(2/3) (the plane
stride of a cube of n points: the long-range couplings of 3D meshes and FE models) — with K the smallest count whose full symmetric pattern
reaches the printed nnz; the last offset's diagonal is cut short so the count is exact.
Off-diagonal values -(0.5 + u), u uniform per unordered pair (seeded); diagonal = sum |off| +
1e-3 (strictly diagonally dominant, SPD, and PDE-like: row sums ~1e-4 of the diagonal, so AMG's
max_row_sum rule (L300) does not cut the strong couplings of the coarse levels).  No method arithmetic: structure and values only.
"""
from __future__ import annotations

import torch

from .csr import CSR
from .stencils import pair_uniform

# (group, matrix, #orders, #nonzeros) as printed in Table II
TABLE2 = [
    ("GHS_indef", "spmsrtls", 29995, 229947),
    ("Schmid", "thermal 1", 82654, 574458),
    ("ACUSIM", "Pres_Poisson", 14822, 715804),
    ("Chevron", "Chevron2", 90249, 803173),
    ("Simon", "venkat25", 62424, 1717792),
    ("Boeing", "bcsstk39", 46772, 2089294),
    ("Williams", "mc2depi", 525825, 2100225),
    ("Norris", "stomach", 213360, 3021648),
    ("Wissgott", "parabolic_fem", 525825, 3674625),
    ("Williams", "cant", 62451, 4007383),
    ("TSOPF", "TSOPF_RS_b300_c3", 42138, 4413449),
    ("Schenk_AFE", "af_shell4", 504855, 17588875),
    ("INPRO", "msdoor", 415863, 20240935),
    ("Janna", "CoupCons3D", 416800, 22322336),
    ("ND", "nd24k", 72000, 28715634),
    ("GHS psdef", "ldoor", 952203, 46522475),
]
BY_NAME = {m: (g, m, n, z) for g, m, n, z in TABLE2}
SHIFT = 1e-3  # diagonal = sum |off| + SHIFT


def _offsets(n: int, K: int):
    K1 = (K + 1) // 2
    offs = list(range(1, K1 + 1))
    K2 = K - K1
    if K2 > 0:  # geometric in (K1, n^(2/3)]: the plane stride of a cube of n points at the top
        lo = K1 + 1
        top = max(lo + K2, int(round(n ** (2.0 / 3.0))))
        for t in range(1, K2 + 1):
            offs.append(max(int(round(lo * (top / lo) ** (t / K2))), offs[-1] + 1))
    return [o for o in offs if o < n]


def plan(name: str):
    """(n, offsets, cut): the diagonals used (ascending offsets, the smallest K whose full
    symmetric pattern reaches the printed nnz) and how many entries of the last one are kept so
    that the pattern has exactly the printed nnz (minus one when nnz - n is odd)."""
    _, _, n, nnz = BY_NAME[name]
    target = nnz - ((nnz - n) & 1)
    for K in range(1, n):
        offs = _offsets(n, K)
        if n + 2 * sum(n - o for o in offs) < target:
            continue
        tot = n
        for t, o in enumerate(offs):
            if tot + 2 * (n - o) >= target:
                return n, offs[:t + 1], (target - tot) // 2
            tot += 2 * (n - o)
    raise ValueError(name)


def realised_nnz(name: str) -> int:
    n, offs, cut = plan(name)
    return n + 2 * sum(n - o for o in offs[:-1]) + 2 * cut


def table2_matrix(name: str, seed: int = 2024, device="cpu") -> CSR:
    """The Table II-shaped synthetic matrix `name` (CSR, float64, sorted unique columns)."""
    n, offs, cut = plan(name)
    rows, cols = [torch.arange(n, dtype=torch.int64, device=device)], [torch.arange(n, dtype=torch.int64, device=device)]
    for t, o in enumerate(offs):
        cnt = (n - o) if t + 1 < len(offs) else cut
        i = torch.arange(cnt, dtype=torch.int64, device=device)
        rows += [i, i + o]
        cols += [i + o, i]
    r = torch.cat(rows)
    c = torch.cat(cols)
    off = r != c
    v = torch.zeros(r.numel(), dtype=torch.float64, device=device)
    v[off] = -(0.5 + pair_uniform(r[off], c[off], seed))
    diag = torch.zeros(n, dtype=torch.float64, device=device).index_add_(0, r[off], v[off].abs())
    v[~off] = diag[r[~off]] + SHIFT
    key = r * n + c
    order = torch.argsort(key)
    r, c, v = r[order], c[order], v[order]
    row_ptr = torch.zeros(n + 1, dtype=torch.int64, device=device)
    row_ptr[1:] = torch.cumsum(torch.bincount(r, minlength=n), 0)
    return CSR(n, n, row_ptr, c.to(torch.int32), v)
