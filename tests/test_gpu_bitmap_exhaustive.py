"""Exhaustive BITMAPMULTIPLY (reading R4/R5; Alg. 3, Alg. 4): every one of the
65,535 x 65,535 pairs of nonzero 4x4 tile bitmaps goes through the GPU symbolic SpGEMM, whose C
structure and bitmaps must equal the boolean 4x4 matrix product (a C tile exists iff the
product is nonzero, R5; its bitmap is the product, bit 4r+c = entry (r, c), R1).

A = 65,535 block rows, block row I one tile at block column 0 with bitmap I+1; B = one block row
of 256 tiles whose bitmaps walk 1..65,535 in 256 batches.  Expected bitmaps are the definition
of the boolean product written row-wise — row r of C is the OR of the rows k of B selected by
row r of A — evaluated with torch integer ops (not the library); that formulation is itself
checked against numpy 4x4 boolean matmuls on random pairs.
"""
import numpy as np
import pytest
import torch

import gen

pytestmark = pytest.mark.gpu

NB = 256


def _amgt():
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    return amgt


def _csr_col_tiles(maps: np.ndarray) -> gen.CSR:
    """Block rows I = 0..len-1, one tile each at block column 0 with bitmap maps[I]."""
    bits = ((maps[:, None].astype(np.int64) >> np.arange(16)) & 1).astype(bool)
    I, k = np.nonzero(bits)  # row-major: block row, then bit = 4r + c -> sorted (row, col)
    rows, cols = 4 * I + k // 4, k % 4
    m = 4 * len(maps)
    rp = np.zeros(m + 1, dtype=np.int64)
    rp[1:] = np.cumsum(np.bincount(rows, minlength=m))
    return gen.CSR(m, 4, torch.from_numpy(rp), torch.from_numpy(cols.astype(np.int32)),
                   torch.ones(len(cols), dtype=torch.float64))


def _csr_row_tiles(maps: np.ndarray) -> gen.CSR:
    """One block row, tile J at block column J with bitmap maps[J]."""
    bits = ((maps[:, None].astype(np.int64) >> np.arange(16)) & 1).astype(bool).reshape(-1, 4, 4)  # [J, r, c]
    r, J, c = np.nonzero(bits.transpose(1, 0, 2))  # sorted by row, then column 4J + c
    rp = np.zeros(5, dtype=np.int64)
    rp[1:] = np.cumsum(np.bincount(r, minlength=4))
    return gen.CSR(4, 4 * len(maps), torch.from_numpy(rp), torch.from_numpy((4 * J + c).astype(np.int32)),
                   torch.ones(len(J), dtype=torch.float64))


def _product_rowwise(a: torch.Tensor, b: torch.Tensor) -> torch.Tensor:
    """C[I, J] bitmaps: row r of C = OR over k in row r of A of row k of B."""
    rowB = [(b >> (4 * k)) & 0xF for k in range(4)]
    T = torch.zeros(16, b.numel(), dtype=torch.int64, device=b.device)
    for nib in range(16):
        for k in range(4):
            if (nib >> k) & 1:
                T[nib] |= rowB[k]
    C = torch.zeros(a.numel(), b.numel(), dtype=torch.int64, device=b.device)
    for r in range(4):
        C |= T[(a >> (4 * r)) & 0xF] << (4 * r)
    return C


def test_rowwise_product_is_boolean_matmul():
    rng = np.random.default_rng(7)
    a = rng.integers(1, 1 << 16, 4000)
    b = rng.integers(1, 1 << 16, 4000)
    C = _product_rowwise(torch.from_numpy(a), torch.from_numpy(b)).numpy()
    for i in range(4000):
        A = ((a[i] >> np.arange(16)) & 1).reshape(4, 4)
        B = ((b[i] >> np.arange(16)) & 1).reshape(4, 4)
        D = ((A @ B) > 0).reshape(16)
        assert C[i, i] == int((D.astype(np.int64) << np.arange(16)).sum())


def test_symbolic_bitmaps_exhaustive():
    amgt = _amgt()
    a_maps = np.arange(1, 1 << 16, dtype=np.int64)
    A = amgt.from_csr(_csr_col_tiles(a_maps), "f16")
    a_dev = torch.from_numpy(a_maps).cuda()
    pairs = 0
    for b0 in range(1, 1 << 16, NB):
        b_maps = np.arange(b0, min(b0 + NB, 1 << 16), dtype=np.int64)
        B = amgt.from_csr(_csr_row_tiles(b_maps), "f16")
        C = amgt.spgemm_symbolic(A, B)
        exp = _product_rowwise(a_dev, torch.from_numpy(b_maps).cuda())
        nz = exp != 0
        cnt = nz.sum(1)
        assert torch.equal(C.blc_ptr.diff(), cnt), b0
        Jexp = torch.nonzero(nz)[:, 1].to(torch.int32)  # row-major: ascending J within each row
        assert torch.equal(C.blc_idx, Jexp), b0
        assert torch.equal(C.map_u16().to(torch.int64), exp[nz]), b0
        pairs += a_maps.size * b_maps.size
        C.free()
        B.free()
    assert pairs == 65535 * 65535
