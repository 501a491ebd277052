"""Pins for oracle O6 (V-cycle, Alg. 2 L68-82) — SURVEY §8(c) P8, P9.

The expected residual history comes from the dense error-propagation operator of
the V-cycle, built recursively with numpy:
    S_k = I - w D_k^-1 A_k,   E_M = 0 (exact coarsest solve),
    E_k = S_k^nu2 (I - P_k (I - E_{k+1}) A_{k+1}^-1 R_k A_k) S_k^nu1,
    x_c = x* - E_1 (x* - x_{c-1}),  x* = A^-1 b.
"""
import numpy as np
import pytest

import gen
import oracle


def _dense_levels(A, PR):
    As = [oracle.as_csr(A).dense()]
    Ps, Rs = [], []
    for P, R in PR:
        Pd, Rd = oracle.as_csr(P).dense(), oracle.as_csr(R).dense()
        Ps.append(Pd)
        Rs.append(Rd)
        As.append(Rd @ As[-1] @ Pd)
    return As, Ps, Rs


def _E(k, As, Ps, Rs, w, nu1, nu2, l1=False):
    n = As[k].shape[0]
    I = np.eye(n)
    if k == len(As) - 1:
        return np.zeros((n, n))
    D = np.abs(As[k]).sum(axis=1) if l1 else np.diag(As[k])  # L1-Jacobi: l1 row norms (L300)
    S = I - w * np.diag(1.0 / D) @ As[k]
    Ec = _E(k + 1, As, Ps, Rs, w, nu1, nu2, l1)
    Bc = (np.eye(As[k + 1].shape[0]) - Ec) @ np.linalg.inv(As[k + 1])
    return np.linalg.matrix_power(S, nu2) @ (I - Ps[k] @ Bc @ Rs[k] @ As[k]) @ np.linalg.matrix_power(S, nu1)


@pytest.mark.parametrize("kind,N,nlev,nu", [("7pt", 8, 3, 1), ("27pt", 8, 2, 1), ("7pt", 8, 3, 2), ("5pt", 16, 3, 1)])
def test_p8_error_propagation(kind, N, nlev, nu):
    A = {"7pt": gen.laplacian_7pt, "27pt": gen.laplacian_27pt, "5pt": gen.laplacian_5pt}[kind](N)
    dims = (N, N) if kind == "5pt" else (N, N, N)
    PR = gen.aggregation_hierarchy(dims, nlev)
    n = A.m
    b = gen.uniform_vector(n, 3).numpy()
    As_o = oracle.build_hierarchy(A, PR)
    x, res, calls = oracle.vcycle(As_o, PR, b, ncycles=6, nu1=nu, nu2=nu)
    As, Ps, Rs = _dense_levels(A, PR)
    for k in range(nlev):
        assert np.array_equal(As_o[k].dense(), As[k])
    E = _E(0, As, Ps, Rs, 2.0 / 3.0, nu, nu)
    xs = np.linalg.solve(As[0], b)
    xc = np.zeros(n)
    exp = [np.linalg.norm(b - As[0] @ xc)]
    for _ in range(6):
        xc = xs - E @ (xs - xc)
        exp.append(np.linalg.norm(b - As[0] @ xc))
    np.testing.assert_allclose(res, exp, rtol=1e-9, atol=1e-13 * exp[0])
    np.testing.assert_allclose(x, xc, rtol=0, atol=1e-10 * np.abs(xs).max())
    # P9: SpMV calls = ncycles*((nu1+nu2+3)(L-1)+1)+1 (= 5(L-1)+1 per cycle at nu=1, L308)
    assert calls == 6 * ((2 * nu + 3) * (nlev - 1) + 1) + 1
    # convergence
    assert res[-1] < 0.2 * res[0]


@pytest.mark.parametrize("omega", [1.0, 0.8])
def test_l1_jacobi_error_propagation(omega):
    """L1-Jacobi smoother (NEXT-3, L300): S = I - w D_l1^-1 A with D_l1 = diag(sum_j |a_ij|),
    on the random SPD 7-point variant (off-diagonals not all equal)."""
    N, nlev = 8, 3
    A = gen.laplacian_7pt(N, spd_seed=4)
    PR = gen.aggregation_hierarchy((N, N, N), nlev)
    b = gen.uniform_vector(A.m, 6).numpy()
    As_o = oracle.build_hierarchy(A, PR)
    x, res, calls = oracle.vcycle(As_o, PR, b, ncycles=5, omega=omega, smoother="l1_jacobi")
    As, Ps, Rs = _dense_levels(A, PR)
    E = _E(0, As, Ps, Rs, omega, 1, 1, l1=True)
    xs = np.linalg.solve(As[0], b)
    xc = np.zeros(A.m)
    exp = [np.linalg.norm(b - As[0] @ xc)]
    for _ in range(5):
        xc = xs - E @ (xs - xc)
        exp.append(np.linalg.norm(b - As[0] @ xc))
    np.testing.assert_allclose(res, exp, rtol=1e-9, atol=1e-13 * exp[0])
    # differs from weighted Jacobi with the same weight (the D really is the l1 norm)
    _, res_j, _ = oracle.vcycle(As_o, PR, b, ncycles=5, omega=omega)
    assert not np.allclose(res, res_j)


def test_l1_jacobi_diagonal_exact():
    """On a positive diagonal matrix L1-Jacobi with w = 1 is an exact solve in one sweep."""
    n = 16
    d = np.arange(1, n + 1, dtype=np.float64)
    A = gen.CSR(n, n, __import__("torch").arange(n + 1, dtype=__import__("torch").int64),
                __import__("torch").arange(n, dtype=__import__("torch").int32), __import__("torch").from_numpy(d))
    PR = gen.aggregation_hierarchy((4, 4), 2)
    b = gen.uniform_vector(n, 7).numpy()
    x, res, _ = oracle.vcycle(oracle.build_hierarchy(A, PR), PR, b, ncycles=1, omega=1.0, smoother="l1_jacobi")
    np.testing.assert_allclose(x, b / d, rtol=1e-15)


def test_alpha_invariance_bitwise():
    """P -> aP, R -> aR (a a power of 2) leaves every iterate bit-identical (R19)."""
    N = 8
    A = gen.laplacian_7pt(N)
    b = gen.uniform_vector(A.m, 5).numpy()
    out = []
    for alpha in (1.0, 0.5):
        PR = gen.aggregation_hierarchy((N, N, N), 3, alpha)
        x, res, _ = oracle.vcycle(oracle.build_hierarchy(A, PR), PR, b, ncycles=4)
        out.append((x, res))
    assert np.array_equal(out[0][0].view(np.uint64), out[1][0].view(np.uint64))
    assert np.array_equal(out[0][1], out[1][1])


def test_p9_call_count_seven_levels():
    """L308: 7 levels, 50 iterations, direct coarsest solve -> 1551 SpMV calls."""
    N = 128  # 128 -> 64 -> ... -> 2 (7 levels); only the call count is checked
    A = gen.laplacian_7pt(16)
    PR = gen.aggregation_hierarchy((16, 16, 16), 4)
    x, res, calls = oracle.vcycle(oracle.build_hierarchy(A, PR), PR, np.ones(A.m), ncycles=50)
    assert calls == 50 * (5 * 3 + 1) + 1
    assert 50 * (5 * 6 + 1) + 1 == 1551 and N == 128


def test_cholesky_dense():
    rng = np.random.default_rng(0)
    M = rng.random((20, 20))
    S = M @ M.T + 20 * np.eye(20)
    L = oracle.cholesky(S)
    assert np.allclose(np.tril(L) @ np.tril(L).T, S, rtol=1e-13, atol=1e-12)
    b = rng.random(20)
    assert np.allclose(oracle.cholesky_solve(L, b), np.linalg.solve(S, b), rtol=1e-12)
