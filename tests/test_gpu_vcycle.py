"""GPU parity: hierarchy setup (Alg. 1 with fixed P) + V-cycle (a10, Alg. 2) vs oracle O6.
FP64 everywhere: residual history matches the oracle to 1e-9 relative.  Mixed precision
(L266): residual reduction per cycle within 1% of the oracle's (north_star), checked
while ||r_k|| / ||r_0|| > 1e-10 (reading R24).  SpMV call count = 1 + ncycles(5(L-1)+1)."""
import numpy as np
import pytest
import torch

import gen
import oracle
from gpu_helpers import assert_structure_equal

pytestmark = pytest.mark.gpu


def _amgt():
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    return amgt


def _run(kind, N, nlev, prec, ncycles, smoother="jacobi", omega=2.0 / 3.0, spd_seed=None):
    amgt = _amgt()
    mk = {"7pt": gen.laplacian_7pt, "27pt": gen.laplacian_27pt, "5pt": gen.laplacian_5pt}[kind]
    A = mk(N, spd_seed=spd_seed) if spd_seed is not None else mk(N)
    dims = (N, N) if kind == "5pt" else (N, N, N)
    PR = gen.aggregation_hierarchy(dims, nlev)
    b = gen.uniform_vector(A.m, 3)
    H = amgt.Hierarchy(amgt.from_csr(A), [amgt.from_csr(P) for P, _ in PR], level_prec=prec, smoother=smoother,
                       omega=omega)
    x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
    res, calls = H.vcycle(b.cuda(), x, ncycles)
    As = oracle.build_hierarchy(A, PR)
    xo, res_o, calls_o = oracle.vcycle(As, PR, b.numpy(), ncycles=ncycles, smoother=smoother, omega=omega)
    return H, As, np.array(res), np.array(res_o), calls, calls_o, x.cpu().numpy(), xo


@pytest.mark.parametrize("kind,N,nlev", [("7pt", 16, 3), ("27pt", 16, 4), ("5pt", 64, 5), ("7pt", 32, 5)])
def test_vcycle_fp64_matches_oracle(kind, N, nlev):
    H, As, res, res_o, calls, calls_o, x, xo = _run(kind, N, nlev, ("f64",) * 8, 8)
    assert calls == calls_o == 1 + 8 * (5 * (nlev - 1) + 1)
    np.testing.assert_allclose(res, res_o, rtol=1e-9)
    np.testing.assert_allclose(x, xo, rtol=0, atol=1e-10 * np.abs(xo).max())
    # the hierarchy's coarse operators equal the oracle's RAP, bit for bit
    for k in range(1, H.nlev):
        Ak, _, _ = H.level(k)
        assert_structure_equal(Ak, oracle.csr_to_mbsr(As[k]))
        rp, ci, v = Ak.to_csr()
        assert np.array_equal(v.cpu().numpy(), As[k].val)
    H.close()


@pytest.mark.parametrize("prec", [("f64",) * 8, ("f64", "f32", "f16", "f16", "f16")])
def test_vcycle_l1_jacobi(prec):
    """L1-Jacobi smoother (D_ii = sum_j |a_ij|, L300, w = 1 as HYPRE) on the random SPD
    7-point variant: FP64 residual history to 1e-9, mixed precision rho within 1%."""
    H, As, res, res_o, calls, calls_o, x, xo = _run("7pt", 32, 5, prec, 8, smoother="l1_jacobi", omega=1.0,
                                                    spd_seed=2)
    assert calls == calls_o
    if prec[1] == "f64":
        np.testing.assert_allclose(res, res_o, rtol=1e-9)
    else:
        rho, rho_o = res[1:] / res[:-1], res_o[1:] / res_o[:-1]
        live = res_o[1:] / res_o[0] > 1e-10
        assert np.all(np.abs(rho[live] - rho_o[live]) <= 0.01 * rho_o[live]), (rho, rho_o)
    H.close()


@pytest.mark.parametrize("kind,N,nlev", [("27pt", 32, 4), ("7pt", 32, 5)])
def test_vcycle_mixed_precision_rho_within_1pct(kind, N, nlev):
    H, As, res, res_o, calls, calls_o, x, xo = _run(kind, N, nlev, ("f64", "f32", "f16", "f16", "f16"), 12)
    assert calls == calls_o
    rho, rho_o = res[1:] / res[:-1], res_o[1:] / res_o[:-1]
    live = res_o[1:] / res_o[0] > 1e-10
    assert live.sum() >= 3
    assert np.all(np.abs(rho[live] - rho_o[live]) <= 0.01 * rho_o[live]), (rho, rho_o)
    H.close()


@pytest.mark.slow
def test_vcycle_cfg3_shape_mixed():
    """Config 3 shape at 64^3 (27-point, 5 levels, mixed precision, 10 cycles)."""
    H, As, res, res_o, calls, calls_o, x, xo = _run("27pt", 64, 5, ("f64", "f32", "f16", "f16", "f16"), 10)
    rho, rho_o = res[1:] / res[:-1], res_o[1:] / res_o[:-1]
    live = res_o[1:] / res_o[0] > 1e-10
    assert np.all(np.abs(rho[live] - rho_o[live]) <= 0.01 * rho_o[live]), (rho, rho_o)
    H.close()


def test_hierarchy_fp16_overflow_reported():
    """R18: a coarse FP16 level whose values exceed 65504 makes amgt_hierarchy_create return
    AMGT_ERR_RANGE (the FP16 range flags of the casts are read back at the hierarchy's
    coarse-level synchronisation): the 27-point operator scaled by 1e4 (diagonal 2.6e5,
    in range for the FP64 / FP32 levels, not for the FP16 ones) fails, the unscaled one
    builds."""
    amgt = _amgt()
    A = gen.laplacian_27pt(16)
    PR = gen.aggregation_hierarchy((16, 16, 16), 4)
    prec = ("f64", "f32", "f16", "f16")
    As = type(A)(A.m, A.n, A.row_ptr, A.col, A.val * 1e4)
    with pytest.raises(amgt.AmgtError) as ei:
        amgt.Hierarchy(amgt.from_csr(As), [amgt.from_csr(P) for P, _ in PR], level_prec=prec)
    assert "RANGE" in str(ei.value)
    H = amgt.Hierarchy(amgt.from_csr(A), [amgt.from_csr(P) for P, _ in PR], level_prec=prec)
    H.close()


_ZG_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import gen, paper_conf_sc_luzwflcy0c024_b200 as amgt
A = gen.laplacian_27pt(32)
PR = gen.aggregation_hierarchy((32, 32, 32), 5)
H = amgt.Hierarchy(amgt.from_csr(A), [amgt.from_csr(P) for P, _ in PR], level_prec=("f64", "f32", "f16", "f16", "f16"))
b = gen.uniform_vector(A.m, 3).cuda()
x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
res, calls = H.vcycle(b, x, 6)
np.save(sys.argv[2], x.cpu().numpy())
print(calls)
"""


def test_zero_guess_fused_bit_identical(tmp_path):
    """The coarse-level zero-guess sweep + residual in one pass (EPI_RES_X0) gives the same
    iterates, bit for bit, as k_jacobi0 followed by the residual SpMV (separate processes:
    AMGT_ZERO_GUESS_FUSED is read once per process), and the same SpMV call count."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    script = tmp_path / "zg.py"
    script.write_text(_ZG_SCRIPT)
    outs, calls = [], []
    for flag in ("1", "0"):
        out = tmp_path / f"x{flag}.npy"
        env = dict(os.environ, AMGT_ZERO_GUESS_FUSED=flag)
        p = subprocess.run([sys.executable, str(script), root, str(out)], env=env, capture_output=True, text=True,
                           timeout=300)
        assert p.returncode == 0, p.stderr[-2000:]
        calls.append(int(p.stdout.strip().splitlines()[-1]))
        outs.append(np.load(out))
    assert calls[0] == calls[1] == 1 + 6 * (5 * 4 + 1)
    assert np.array_equal(outs[0].view(np.uint64), outs[1].view(np.uint64))
