"""Pins for the oracle PCG (NEXT-1; L92) — not against itself:
* scipy.sparse.linalg.cg (the textbook routine) with the same preconditioner gives the same
  iterates (compared through ||b - A x_k||);
* with the identity preconditioner on a small SPD system, CG terminates in <= n steps;
* successive preconditioned residuals are M-orthogonal: r_i . M r_j = 0 (i != j);
* the V-cycle preconditioner beats plain V-cycle iteration (same number of V-cycles)."""
import numpy as np
import pytest
import scipy.sparse as sp
import scipy.sparse.linalg as spla

import gen
import oracle


def _setup(N=8, nlev=3, spd_seed=3):
    A = gen.laplacian_7pt(N, spd_seed=spd_seed)
    PR = gen.aggregation_hierarchy((N, N, N), nlev)
    As = oracle.build_hierarchy(A, PR)
    b = gen.uniform_vector(A.m, 11).numpy()
    return A, PR, As, b


def _scipy(A):
    Ao = oracle.as_csr(A)
    return sp.csr_matrix((Ao.val, Ao.col, Ao.row_ptr), shape=(Ao.m, Ao.n))


def test_pcg_matches_scipy_cg():
    A, PR, As, b = _setup()
    M = oracle.vcycle_preconditioner(As, PR)
    x, res = oracle.pcg(A, b, M, maxit=8)
    As_ = _scipy(A)
    xs_hist = []
    spla.cg(As_, b, x0=np.zeros(A.m), rtol=1e-300, atol=0.0, maxiter=8,
            M=spla.LinearOperator(As_.shape, matvec=M), callback=lambda xk: xs_hist.append(xk.copy()))
    true_res = [np.linalg.norm(b - As_ @ xk) for xk in xs_hist]
    np.testing.assert_allclose(res[1:len(true_res) + 1], true_res, rtol=1e-6, atol=1e-12 * res[0])
    assert res[-1] < 1e-6 * res[0]


def test_cg_finite_termination_identity_preconditioner():
    rng = np.random.default_rng(1)
    n = 12
    Q = rng.standard_normal((n, n))
    S = Q @ Q.T + n * np.eye(n)
    Sd = sp.csr_matrix(S)
    Acsr = gen.CSR(n, n, __import__("torch").from_numpy(Sd.indptr.astype(np.int64)),
                   __import__("torch").from_numpy(Sd.indices.astype(np.int32)), __import__("torch").from_numpy(Sd.data))
    b = rng.standard_normal(n)
    x, res = oracle.pcg(Acsr, b, lambda r: r.copy(), maxit=n)
    assert res[-1] <= 1e-9 * res[0]
    np.testing.assert_allclose(x, np.linalg.solve(S, b), rtol=1e-8)


def test_preconditioned_residuals_m_orthogonal():
    A, PR, As, b = _setup(N=8, nlev=2)
    M = oracle.vcycle_preconditioner(As, PR)
    Ao = oracle.as_csr(A)
    # re-run the recurrence keeping r_k and z_k (the oracle's own steps)
    x = np.zeros(Ao.m)
    r = b - oracle.spmv(Ao, x)
    z = M(r)
    p, rz = z.copy(), r @ z
    rs, zs = [r.copy()], [z.copy()]
    for _ in range(5):
        q = oracle.spmv(Ao, p)
        alpha = rz / (p @ q)
        x, r = x + alpha * p, r - alpha * q
        z = M(r)
        rz_new = r @ z
        p, rz = z + (rz_new / rz) * p, rz_new
        rs.append(r.copy())
        zs.append(z.copy())
    for i in range(len(rs)):
        for j in range(len(rs)):
            if i != j:
                scale = np.sqrt(abs(rs[i] @ zs[i]) * abs(rs[j] @ zs[j]))
                assert abs(rs[i] @ zs[j]) <= 1e-8 * scale, (i, j)


def test_pcg_beats_vcycle_iteration():
    A, PR, As, b = _setup(N=16, nlev=4)
    _, res_v, _ = oracle.vcycle(As, PR, b, ncycles=6)
    _, res_p = oracle.pcg(A, b, oracle.vcycle_preconditioner(As, PR), maxit=6)
    assert res_p[-1] < res_v[-1]
