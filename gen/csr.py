"""A plain CSR container (row_ptr int64[m+1], col int32[nnz], val float64[nnz]).

Arrays are torch tensors (CPU or CUDA).  `.numpy()` gives zero-copy numpy views
for CPU tensors (what the oracle consumes).
"""
from __future__ import annotations

from dataclasses import dataclass

import torch


@dataclass
class CSR:
    m: int
    n: int
    row_ptr: torch.Tensor  # int64 [m+1]
    col: torch.Tensor      # int32 [nnz], sorted and unique within each row
    val: torch.Tensor      # float64 [nnz]

    @property
    def nnz(self) -> int:
        return int(self.col.numel())

    @property
    def device(self) -> torch.device:
        return self.row_ptr.device

    def to(self, device) -> "CSR":
        return CSR(self.m, self.n, self.row_ptr.to(device), self.col.to(device), self.val.to(device))

    def numpy(self):
        """(row_ptr, col, val) as contiguous numpy arrays (copies to host if needed)."""
        c = self.to("cpu")
        return (c.row_ptr.contiguous().numpy(), c.col.contiguous().numpy(), c.val.contiguous().numpy())

    def with_values(self, val: torch.Tensor) -> "CSR":
        return CSR(self.m, self.n, self.row_ptr, self.col, val)

    def to_dense(self) -> torch.Tensor:
        """Dense float64 copy (small matrices only; used by pins)."""
        c = self.to("cpu")
        rows = torch.repeat_interleave(torch.arange(c.m, dtype=torch.int64), c.row_ptr.diff())
        d = torch.zeros(c.m, c.n, dtype=torch.float64)
        d.index_put_((rows, c.col.long()), c.val, accumulate=True)
        return d

    def structure_dense(self) -> torch.Tensor:
        """Dense bool pattern (structural nonzeros, explicit zeros included)."""
        c = self.to("cpu")
        rows = torch.repeat_interleave(torch.arange(c.m, dtype=torch.int64), c.row_ptr.diff())
        d = torch.zeros(c.m, c.n, dtype=torch.bool)
        d[rows, c.col.long()] = True
        return d


def csr_from_coo_sorted(m: int, n: int, rows: torch.Tensor, cols: torch.Tensor, vals: torch.Tensor) -> CSR:
    """Build CSR from COO triplets that are already sorted by (row, col) and unique."""
    counts = torch.bincount(rows.long(), minlength=m)
    row_ptr = torch.zeros(m + 1, dtype=torch.int64, device=rows.device)
    row_ptr[1:] = torch.cumsum(counts, 0)
    return CSR(m, n, row_ptr, cols.to(torch.int32).contiguous(), vals.to(torch.float64).contiguous())
