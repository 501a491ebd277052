"""Pins for the NEXT-2 oracle steps: O8 strength-of-connection filter and
O9 interpolation through one SpGEMM call (Alg. 1 line 4, L54; [35], L385), reading R31
(smoothed aggregation: P = (I - w D_F^-1 A_F) Pt, classical strength with str_thr = theta, L300).

Pins independent of the oracle's own loops:
  * a hand-derived 4x4 worked example of the filter (expected arrays written out below);
  * lumping preserves row sums (exact on integer data) and A_F is a sub-pattern of A;
  * a constant-coefficient stencil keeps every connection (A_F = A for theta <= 1);
  * the 1D Poisson closed form of smoothed aggregation with pair aggregates and w = 2/3:
    interior rows (1/3, 2/3 | 2/3, 1/3), boundary rows 2/3;
  * dense brute force (numpy dense products) for P on random matrices;
  * a zero-row-sum (Neumann) operator: P reproduces the constant (P 1 = 1);
  * RAP with the SA P is symmetric, and the SA V-cycle converges faster than the
    tentative-P V-cycle on the 7-point Laplacian (a sign or scale error would not)."""
import numpy as np
import pytest

import gen
import oracle


def _csr(dense):
    d = np.asarray(dense, dtype=np.float64)
    m, n = d.shape
    rows, cols = np.nonzero(d)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.add.at(rp, rows + 1, 1)
    return oracle.Csr(m, n, np.cumsum(rp), cols.astype(np.int32), d[rows, cols].copy())


def test_strength_worked_example():
    # theta = 0.25.  Row 0: off-diagonals -2, -0.4 -> m = 2, threshold 0.5: -0.4 is weak,
    # lumped: diag 4 - 0.4 = 3.6.  Row 1: -2, -1, +1 -> m = 2: -2, -1 strong (>= 0.5), +1 weak
    # (positive), diag 5 + 1 = 6.  Row 2: -0.4, -3 -> m = 3, thr 0.75: -0.4 weak, diag 7 - 0.4.
    # Row 3: +1, -0.1 -> m = 0.1, thr 0.025: -0.1 strong, +1 weak, diag 2 + 1 = 3.
    A = [[4.0, -2.0, -0.4, 0.0],
         [-2.0, 5.0, -1.0, 1.0],
         [-0.4, 0.0, 7.0, -3.0],
         [0.0, 1.0, 0.0, 2.0]]
    A[3][2] = -0.1
    AF = oracle.strength_filter(_csr(A), 0.25)
    expect = np.array([[3.6, -2.0, 0.0, 0.0],
                       [-2.0, 6.0, -1.0, 0.0],
                       [0.0, 0.0, 6.6, -3.0],
                       [0.0, 0.0, -0.1, 3.0]])
    np.testing.assert_allclose(AF.dense(), expect, rtol=0, atol=1e-15)
    assert AF.nnz == 9  # structure: the 3 dropped entries removed (12 -> 9)


def test_strength_row_sums_and_subpattern():
    rng = np.random.default_rng(5)
    n = 60
    d = np.zeros((n, n))
    for i in range(n):
        cols = rng.choice(n, 6, replace=False)
        d[i, cols] = rng.integers(-9, 4, 6)
        d[i, i] = 40
    A = _csr(d)
    for theta in (0.1, 0.25, 0.5, 0.9):
        AF = oracle.strength_filter(A, theta)
        assert np.array_equal(AF.dense().sum(1), d.sum(1))  # lumping keeps row sums (integers: exact)
        assert not np.any(AF.pattern() & ~A.pattern())
        assert np.all(np.diag(AF.dense()) != 0)
    # theta -> larger keeps fewer entries
    assert oracle.strength_filter(A, 0.9).nnz <= oracle.strength_filter(A, 0.1).nnz


@pytest.mark.parametrize("mk", [lambda: gen.laplacian_7pt(6), lambda: gen.laplacian_27pt(5), lambda: gen.laplacian_5pt(9)])
def test_strength_constant_stencil_keeps_everything(mk):
    A = oracle.as_csr(mk())
    for theta in (0.25, 1.0):
        AF = oracle.strength_filter(A, theta)
        assert np.array_equal(AF.row_ptr, A.row_ptr) and np.array_equal(AF.col, A.col)
        assert np.array_equal(AF.val, A.val)


def _pairs_P(n):
    Pt = np.zeros((n, n // 2))
    for i in range(n):
        Pt[i, i // 2] = 1.0
    return Pt


def test_sa_1d_poisson_closed_form():
    n = 8
    A = np.diag(np.full(n, 2.0)) - np.diag(np.ones(n - 1), 1) - np.diag(np.ones(n - 1), -1)
    P = oracle.sa_interp(_csr(A), _csr(_pairs_P(n)), theta=0.25, omega=2.0 / 3.0).dense()
    expect = np.zeros((n, n // 2))
    for j in range(n // 2):
        expect[2 * j, j] = expect[2 * j + 1, j] = 2.0 / 3.0
        if j > 0:
            expect[2 * j, j - 1] = 1.0 / 3.0
        if j + 1 < n // 2:
            expect[2 * j + 1, j + 1] = 1.0 / 3.0
    np.testing.assert_allclose(P, expect, rtol=0, atol=1e-15)


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_sa_dense_brute_force(seed):
    rng = np.random.default_rng(seed)
    m, nc = 23, 7
    d = np.where(rng.random((m, m)) < 0.25, -rng.random((m, m)) * 2, 0.0)
    d = d + np.where(rng.random((m, m)) < 0.05, rng.random((m, m)), 0.0)
    np.fill_diagonal(d, np.abs(d).sum(1) + 1.0)
    agg = rng.integers(0, nc, m)
    agg[:nc] = np.arange(nc)
    Pt = np.zeros((m, nc))
    Pt[np.arange(m), agg] = 1.0
    theta, w = 0.3, 2.0 / 3.0
    AF = oracle.strength_filter(_csr(d), theta)
    P = oracle.sa_interp(_csr(d), _csr(Pt), theta, w)
    F = AF.dense()
    expect = Pt - (w / np.diag(F))[:, None] * (F @ Pt)
    np.testing.assert_allclose(P.dense(), expect, rtol=0, atol=1e-14)
    # structure = boolean product of the patterns (cancelled entries kept, R3)
    assert np.array_equal(P.pattern(), (AF.pattern().astype(int) @ (Pt != 0).astype(int)) > 0)


def test_sa_reproduces_constant_for_zero_row_sums():
    n = 16
    A = np.diag(np.full(n, 2.0)) - np.diag(np.ones(n - 1), 1) - np.diag(np.ones(n - 1), -1)
    A[0, 0] = A[-1, -1] = 1.0  # Neumann ends: A 1 = 0
    P = oracle.sa_interp(_csr(A), _csr(_pairs_P(n)), 0.25, 2.0 / 3.0).dense()
    np.testing.assert_allclose(P @ np.ones(n // 2), np.ones(n), rtol=0, atol=1e-15)


def test_sa_hierarchy_symmetric_and_faster():
    N, nlev = 16, 3
    A = gen.laplacian_7pt(N)
    PR = gen.aggregation_hierarchy((N, N, N), nlev)
    As, PRs = oracle.build_hierarchy_sa(A, [P for P, _ in PR], theta=0.25, omega=2.0 / 3.0)
    for Ak in As[1:]:
        D = Ak.dense()
        np.testing.assert_allclose(D, D.T, rtol=0, atol=1e-12 * np.abs(D).max())
    # the SA interpolation is denser than the tentative one (it came out of a SpGEMM)
    assert PRs[0][0].nnz > oracle.as_csr(PR[0][0]).nnz
    b = gen.uniform_vector(A.m, 3).numpy()
    _, res_sa, calls_sa = oracle.vcycle(As, PRs, b, ncycles=6)
    _, res_t, _ = oracle.vcycle(oracle.build_hierarchy(A, PR), PR, b, ncycles=6)
    assert calls_sa == 1 + 6 * (5 * (nlev - 1) + 1)
    assert res_sa[-1] < 0.5 * res_t[-1], (res_sa, res_t)
