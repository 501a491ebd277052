"""Row-slab inputs for the distributed path: each rank generates only its own rows
(global column indices) of A_1 and of every P_k.  z-slabs of the lexicographic grid,
split by whole planes; planes of every level stay 4-row aligned while the coarse grid
keeps >= 2x2 points per plane."""
from __future__ import annotations

from .aggregation import _coarse_dims, aggregation_P
from .stencils import OFFS_5PT, OFFS_7PT, OFFS_27PT, stencil

STENCILS = {"7pt": (OFFS_7PT, 6.0), "27pt": (OFFS_27PT, 26.0), "5pt": (OFFS_5PT, 4.0)}


def slab_ranges(n_planes: int, plane: int, size: int):
    """Rank r owns planes [r*n/size, (r+1)*n/size) -> rows [z0*plane, z1*plane)."""
    return [((r * n_planes) // size * plane, ((r + 1) * n_planes) // size * plane) for r in range(size)]


def level_dims(dims, nlev):
    out = [tuple(dims)]
    for _ in range(nlev - 1):
        out.append(_coarse_dims(out[-1]))
    return out


def slab_inputs(kind: str, dims, nlev: int, rank: int, size: int, alpha=None, device="cpu", spd_seed=None):
    """(A_rows, (rb, re), n, [P_rows per level]) for this rank.  The slab of every level is
    the same z-range (halved per level), so aggregates never straddle ranks."""
    offs, center = STENCILS[kind]
    ld = level_dims(dims, nlev)
    plane0 = ld[0][0] * ld[0][1]
    n0 = plane0 * ld[0][2]
    z = [((rank * ld[0][2]) // size, ((rank + 1) * ld[0][2]) // size)]
    for k in range(1, nlev):  # coarse z-range = halved fine range
        z.append(((z[-1][0] + 1) // 2, (z[-1][1] + 1) // 2))
    rows0 = (z[0][0] * plane0, z[0][1] * plane0)
    A = stencil(ld[0], offs, center, -1.0, device, spd_seed, rows0)
    Ps = []
    for k in range(nlev - 1):
        pk = ld[k][0] * ld[k][1]
        Ps.append(aggregation_P(ld[k], alpha, device, rows=(z[k][0] * pk, z[k][1] * pk)))
    return A, rows0, n0, Ps
