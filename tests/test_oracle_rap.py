"""Pins for oracle O5 (RAP) — SURVEY §8(c) P3, P4, P5.

The expected coarse operators come from Kronecker identities of the stencils, built
with numpy.kron (independent of the oracle's SpGEMM loop):
  7-point:  A = 6I - sum_d T0_d,  T0 = tridiag(1,0,1);  p^T p = 2I, p^T T0 p = tridiag(1,2,1)
            => R A P = 4 A_7(N/2) at alpha = 1, A_7(N/2) at alpha = 1/2.
  27-point: A = 27I - T (x) T (x) T,  T = tridiag(1,1,1);  p^T T p = tridiag(1,4,1)
            => R A P = 216 I - tridiag(1,4,1)^(x)3 at alpha = 1 (diag 152, face -16,
               edge -4, corner -1), divided by 4 at alpha = 1/2.
"""
import numpy as np
import pytest

import gen
import oracle


def _tri(n, lo, d, hi):
    return np.diag(np.full(n, float(d))) + np.diag(np.full(n - 1, float(lo)), -1) + np.diag(np.full(n - 1, float(hi)), 1)


def _kron3(a, b, c):
    # lexicographic x fastest: index = x + N y + N^2 z  ->  kron(z, kron(y, x))
    return np.kron(c, np.kron(b, a))


@pytest.mark.parametrize("N,alpha", [(8, 1.0), (8, 0.5), (16, 0.5)])
def test_p3_7pt_rap_closed_form(N, alpha):
    A = gen.laplacian_7pt(N)
    P = gen.aggregation_P((N, N, N), alpha)
    R = gen.aggregation_R((N, N, N), alpha)
    C = oracle.rap(R, A, P)
    expect = oracle.as_csr(gen.laplacian_7pt(N // 2)).dense() * (4.0 * alpha * alpha)
    assert np.array_equal(C.dense(), expect)
    assert np.array_equal(C.pattern(), expect != 0)
    AP = oracle.spgemm(A, P)
    assert AP.nnz == N ** 3 + 3 * (N - 2) * N * N
    assert oracle.csr_to_mbsr(AP).blc_num == N * N * (N - 3)


@pytest.mark.parametrize("N,alpha", [(8, 1.0), (8, 0.5)])
def test_p4_27pt_rap_closed_form(N, alpha):
    A = gen.laplacian_27pt(N)
    P = gen.aggregation_P((N, N, N), alpha)
    R = gen.aggregation_R((N, N, N), alpha)
    C = oracle.rap(R, A, P)
    n = N // 2
    t = _tri(n, 1, 4, 1)
    expect = (216.0 * np.eye(n ** 3) - _kron3(t, t, t)) * (alpha * alpha)
    assert np.array_equal(C.dense(), expect)
    d = C.dense()
    if alpha == 1.0:  # interior coarse point (1,1,1)
        i = 1 + n * (1 + n * 1)
        assert d[i, i] == 152 and d[i, i + 1] == -16 and d[i, i + 1 + n] == -4 and d[i, i + 1 + n + n * n] == -1
    assert C.nnz == (3 * n - 2) ** 3
    assert oracle.spgemm(A, P).nnz == (2 * N - 2) ** 3


def test_p5_rap_symmetry_random_spd():
    """R = P^T -> R A P symmetric (structure bit-exact; dyadic values exact)."""
    N = 12
    A = gen.laplacian_7pt(N, spd_seed=2)
    vals = A.val.numpy()
    # make values dyadic (multiples of 2^-8) while keeping symmetry of the generator
    A = A.with_values(__import__("torch").from_numpy(np.round(vals * 256) / 256))
    C = oracle.rap(gen.aggregation_R((N, N, N)), A, gen.aggregation_P((N, N, N)))
    d = C.dense()
    assert np.array_equal(C.pattern(), C.pattern().T)
    assert np.array_equal(d, d.T)


def test_rap_with_abs_scale():
    A = gen.laplacian_7pt(6)
    P = gen.aggregation_P((6, 6, 6), 0.5)
    R = gen.aggregation_R((6, 6, 6), 0.5)
    C, Cabs = oracle.rap(R, A, P, with_abs=True)
    Ad, Pd, Rd = oracle.as_csr(A).dense(), oracle.as_csr(P).dense(), oracle.as_csr(R).dense()
    full = np.abs(Rd) @ (np.abs(Ad) @ np.abs(Pd))
    rows = np.repeat(np.arange(C.m), np.diff(C.row_ptr))
    assert np.array_equal(Cabs, full[rows, C.col])
