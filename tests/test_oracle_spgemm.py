"""Pins for oracle O1 (structural Gustavson SpGEMM) — SURVEY §8(c) P1, P2, P10.

None of these re-derive the oracle's loop: they compare against dense products,
closed forms of the 5-point Laplacian, and scipy's SMMP on positive data.
"""
import numpy as np
import pytest
import scipy.sparse as sp

import gen
import oracle


def _dense_pattern_product(A, B):
    return (A.pattern().astype(np.int64) @ B.pattern().astype(np.int64)) > 0


@pytest.mark.parametrize("m,k,n,dens,seed", [(1, 1, 1, 1.0, 0), (5, 7, 3, 0.4, 1), (13, 9, 17, 0.3, 2),
                                             (33, 31, 30, 0.15, 3), (64, 61, 63, 0.08, 4), (10, 10, 10, 0.0, 5)])
def test_p1_bruteforce_dense_integer(m, k, n, dens, seed):
    """P1: integer data -> the dense FP64 product is exact; structure = boolean product
    (keeps cancelled entries, reading R3/R5); empty rows/cols, m,n not multiples of 4."""
    A = oracle.as_csr(gen.random_csr(m, k, dens, seed, integer=True, empty_rows=min(2, m)))
    B = oracle.as_csr(gen.random_csr(k, n, dens, seed + 100, integer=True, zero_frac=0.1))
    C, Cabs = oracle.spgemm(A, B, with_abs=True)
    assert np.array_equal(C.pattern(), _dense_pattern_product(A, B))
    assert np.array_equal(C.dense(), A.dense() @ B.dense())
    # columns strictly increasing per row
    for i in range(C.m):
        assert np.all(np.diff(C.col[C.row_ptr[i]:C.row_ptr[i + 1]]) > 0)
    # |A||B| scale on C's pattern
    absd = np.abs(A.dense()) @ np.abs(B.dense())
    rows = np.repeat(np.arange(C.m), np.diff(C.row_ptr))
    assert np.array_equal(Cabs, absd[rows, C.col])


def test_p1_cancellation_kept():
    """A structural entry whose value cancels to 0 stays in C (reading R3)."""
    A = oracle.Csr(1, 2, np.array([0, 2]), np.array([0, 1], np.int32), np.array([1.0, 1.0]))
    B = oracle.Csr(2, 1, np.array([0, 1, 2]), np.array([0, 0], np.int32), np.array([1.0, -1.0]))
    C = oracle.spgemm(A, B)
    assert C.nnz == 1 and C.val[0] == 0.0


@pytest.mark.parametrize("N", [4, 8, 17, 64])
def test_p2_5pt_square_closed_form(N):
    """P2: nnz(A^2) = 13N^2 - 20N + 4 for the 5-point Laplacian; scalar products = sum deg^2."""
    A = oracle.as_csr(gen.laplacian_5pt(N))
    C = oracle.spgemm(A, A)
    assert C.nnz == 13 * N * N - 20 * N + 4
    deg = np.diff(A.row_ptr)
    if N == 64:
        assert int((deg * deg).sum()) == 100_104
        M = oracle.csr_to_mbsr(C)
        assert M.blc_num == 10_724


def test_p10_scipy_positive():
    """P10: on positive data (no cancellation) O1 equals scipy's SMMP product exactly
    (integer values -> exact regardless of summation order)."""
    A = oracle.as_csr(gen.random_csr(70, 50, 0.1, 7, integer=True, positive=True))
    B = oracle.as_csr(gen.random_csr(50, 90, 0.1, 8, integer=True, positive=True))
    C = oracle.spgemm(A, B)
    S = (sp.csr_matrix((A.val, A.col, A.row_ptr), shape=(A.m, A.n)) @
         sp.csr_matrix((B.val, B.col, B.row_ptr), shape=(B.m, B.n))).tocsr()
    S.sort_indices()
    assert np.array_equal(C.row_ptr, S.indptr) and np.array_equal(C.col, S.indices)
    assert np.array_equal(C.val, S.data)


def test_p10_scipy_positive_float():
    """Random positive floats: values agree with scipy to rounding (1e-14 relative)."""
    A = oracle.as_csr(gen.random_csr(60, 60, 0.2, 9, positive=True))
    C = oracle.spgemm(A, A)
    Sd = (sp.csr_matrix((A.val, A.col, A.row_ptr), shape=(A.m, A.n)) ** 2).toarray()
    assert np.allclose(C.dense(), Sd, rtol=1e-14, atol=0)


def test_thread_count_invariance():
    A = oracle.as_csr(gen.random_csr(300, 300, 0.05, 11))
    C1 = oracle.spgemm(A, A, nthreads=1)
    C4 = oracle.spgemm(A, A, nthreads=4)
    assert np.array_equal(C1.col, C4.col) and np.array_equal(C1.val, C4.val)
