"""Pins for oracle O3 (CSR SpMV) and O4 (transpose) — SURVEY §8(c) P1, P2, P10."""
import numpy as np
import pytest
import scipy.sparse as sp

import gen
import oracle


@pytest.mark.parametrize("m,n,dens,seed", [(1, 1, 1.0, 0), (17, 13, 0.3, 1), (64, 100, 0.05, 2), (10, 10, 0.0, 3)])
def test_dense_matvec_integer(m, n, dens, seed):
    A = oracle.as_csr(gen.random_csr(m, n, dens, seed, integer=True, empty_rows=1))
    x = gen.integer_vector(n, seed).numpy()
    assert np.array_equal(oracle.spmv(A, x), A.dense() @ x)
    assert np.array_equal(oracle.spmv_abs(A, x), np.abs(A.dense()) @ np.abs(x))


def test_p2_5pt_rowsums():
    """P2: A*1 for the 5-point 64x64 Laplacian has 3,844 zeros, 248 ones and 4 twos."""
    y = oracle.spmv(gen.laplacian_5pt(64), np.ones(4096))
    assert (y == 0).sum() == 3844 and (y == 1).sum() == 248 and (y == 2).sum() == 4


@pytest.mark.parametrize("N", [5, 12])
def test_7pt_rowsums(N):
    """7-point A*1 = number of missing neighbours: (N-2)^3 zeros, 6(N-2)^2 ones,
    12(N-2) twos, 8 threes."""
    y = oracle.spmv(gen.laplacian_7pt(N), np.ones(N ** 3))
    counts = [(y == v).sum() for v in range(4)]
    assert counts == [(N - 2) ** 3, 6 * (N - 2) ** 2, 12 * (N - 2), 8]


def test_scipy_random_float():
    A = oracle.as_csr(gen.random_csr(200, 150, 0.05, 4))
    x = gen.uniform_vector(150, 4).numpy()
    S = sp.csr_matrix((A.val, A.col, A.row_ptr), shape=(A.m, A.n))
    np.testing.assert_allclose(oracle.spmv(A, x), S @ x, rtol=1e-13, atol=1e-15)


def test_transpose_dense_and_aggregation():
    A = oracle.as_csr(gen.random_csr(23, 41, 0.2, 5))
    T = oracle.transpose(A)
    assert np.array_equal(T.dense(), A.dense().T)
    P = gen.aggregation_P((6, 6, 6))
    R = oracle.as_csr(gen.aggregation_R((6, 6, 6)))
    PT = oracle.transpose(P)
    assert np.array_equal(PT.row_ptr, R.row_ptr) and np.array_equal(PT.col, R.col)
    assert np.array_equal(PT.val, R.val)
