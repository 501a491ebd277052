"""GPU parity: amgt_pcg (V-cycle-preconditioned CG, NEXT-1, L92) vs the oracle PCG
(textbook recurrence, oracle V-cycle as M).  FP64 hierarchy: residual history to 1e-7
relative while ||r_k||/||r_0|| > 1e-10; mixed precision (L266): on operators exact in every
level precision, per iteration within 1e-4 of the FP64 oracle (derivation in the test); on
random SPD data (operators rounded per level) within a factor 2 at every iteration; early stop
on rtol; SpMV call count."""
import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu


def _run(N, nlev, prec, maxit, rtol=0.0, spd_seed=3, b_seed=11):
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    A = gen.laplacian_7pt(N, spd_seed=spd_seed)
    PR = gen.aggregation_hierarchy((N, N, N), nlev)
    b = gen.uniform_vector(A.m, b_seed)
    H = amgt.Hierarchy(amgt.from_csr(A), [amgt.from_csr(P) for P, _ in PR], level_prec=prec)
    x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
    res, it, calls = H.pcg(b.cuda(), x, maxit, rtol)
    H.close()
    As = oracle.build_hierarchy(A, PR)
    xo, res_o = oracle.pcg(A, b.numpy(), oracle.vcycle_preconditioner(As, PR), maxit=maxit)
    return np.array(res), it, calls, x.cpu().numpy(), np.array(res_o), xo


@pytest.mark.parametrize("N,nlev", [(16, 3), (32, 5)])
def test_pcg_fp64_matches_oracle(N, nlev):
    res, it, calls, x, res_o, xo = _run(N, nlev, ("f64",) * 8, 10)
    assert it == 10 and len(res) == 11
    live = res_o / res_o[0] > 1e-10
    np.testing.assert_allclose(res[live], res_o[live], rtol=1e-7)
    assert calls == 1 + 10 + 11 * 5 * (nlev - 1)
    if live.all():
        np.testing.assert_allclose(x, xo, rtol=0, atol=1e-8 * np.abs(xo).max())


def test_pcg_mixed_precision_converges_like_fp64():
    res, it, calls, x, res_o, xo = _run(32, 5, ("f64", "f32", "f16", "f16", "f16"), 12)
    assert np.all(res <= 2.0 * res_o + 1e-14 * res_o[0]), (res, res_o)
    assert res[-1] < 1e-8 * res[0]


def test_pcg_mixed_precision_per_iteration():
    """Mixed precision (L266: FP64 / FP32 / FP16 levels) on the 7-point Laplacian with alpha = 1/2
    aggregation: every coarse operator is an integer stencil (A_c = A_7(N/2), P3 of SURVEY
    8(c)), exact in FP32 and FP16, so the GPU preconditioner differs from the oracle's FP64
    V-cycle only by its FP32 coarse-level vectors (unit roundoff u = 2^-24).  Tolerance: the
    preconditioned residual of CG moves by O(kappa_M u) per iteration with kappa_M (the
    V-cycle-preconditioned condition number) ~ 10 here; over 12 iterations, 1e-4 relative."""
    res, it, calls, x, res_o, xo = _run(32, 5, ("f64", "f32", "f16", "f16", "f16"), 12, spd_seed=None)
    live = res_o / res_o[0] > 1e-9
    assert live.sum() >= 6
    np.testing.assert_allclose(res[live], res_o[live], rtol=1e-4)


def test_pcg_early_stop():
    res, it, calls, x, res_o, xo = _run(16, 3, ("f64",) * 8, 50, rtol=1e-8)
    assert it < 50 and res[-1] <= 1e-8 * res[0] and res[-2] > 1e-8 * res[0]
