"""GPU parity: fused multi-stage sweeps (amgt_spmv_sweeps, §8(f) NEXT-1) — consecutive
Alg. 2 steps (Jacobi sweep L73/L81, residual L75) in one pass over an FP64 operator.

* every stage output is bit-identical to the separate single-SpMV kernels (same per-row
  arithmetic), and within 1e-12 (scaled, R28) of the oracle's SpMV + Alg. 2 formulas;
* the squared residual norm equals the FP64 sum of squares to 1e-12 relative;
* correctness does not depend on the wavefront knobs (minimum lag, one CTA per SM);
* the V-cycle that uses the sweeps reproduces the unfused V-cycle (AMGT_SWEEP=0) iterate
  for iterate (x bit-identical, norms to 1e-12) and the oracle's residual history."""
import os

import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu


def _amgt():
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    return amgt


MATS = [
    ("7pt_24_spd", lambda: gen.laplacian_7pt(24, spd_seed=2)),     # 13,824 rows: 54 chunks, bandwidth 2 chunks
    ("5pt_64", lambda: gen.laplacian_5pt(64)),                      # 16 chunks
    ("27pt_20", lambda: gen.laplacian_27pt(20)),
    ("7pt_7_ragged", lambda: gen.laplacian_7pt(7)),                 # 343 rows: m not a multiple of 4
    ("irregular_small", lambda: gen.irregular_block_sparse(1 << 11)),  # bandwidth ~ whole matrix
    ("rand_sq_empty", lambda: gen.random_csr(1001, 1001, 0.01, 5, empty_rows=30)),
    ("one", lambda: gen.random_csr(1, 1, 1.0, 3)),
]


def _dinv_host(Ao):
    d = np.zeros(Ao.m)
    for i in range(Ao.m):
        for p in range(Ao.row_ptr[i], Ao.row_ptr[i + 1]):
            if Ao.col[p] == i and Ao.val[p] != 0:
                d[i] = 1.0 / Ao.val[p]
    return d


def _pad(v, n):
    out = torch.zeros(n, dtype=torch.float64, device="cuda")
    out[:v.numel()] = v
    return out


@pytest.mark.parametrize("name,mk", MATS, ids=[m[0] for m in MATS])
@pytest.mark.parametrize("knobs", [{}, {"AMGT_SWEEP_LAG": "0", "AMGT_SWEEP_CTAS": "1"}], ids=["default", "minlag"])
def test_sweeps_match_separate_kernels_and_oracle(name, mk, knobs, monkeypatch):
    amgt = _amgt()
    for k, v in knobs.items():
        monkeypatch.setenv(k, v)
    A = mk()
    Ao = oracle.as_csr(A)
    M = amgt.from_csr(A)
    n = 4 * M.blc_row
    x0 = _pad(gen.uniform_vector(A.n, 1).cuda(), n)
    b = _pad(gen.uniform_vector(A.m, 2).cuda(), n)
    dh = _dinv_host(Ao)
    d = _pad(torch.from_numpy(dh).cuda(), n)
    w = 2.0 / 3.0
    plan = amgt.SweepPlan(M)
    x1, x2, r = (torch.full((n,), np.nan, dtype=torch.float64, device="cuda") for _ in range(3))
    nrm = torch.zeros(1, dtype=torch.float64, device="cuda")
    for _ in range(2):  # the second call reuses the plan (epochs, re-armed counters)
        plan.run([("jacobi", x0, x1), ("jacobi_res", x1, x2), ("residual", x2, r)], b, d, w, norm=nrm)
        # separate kernels
        e1, e2, er, rr = (torch.empty(n, dtype=torch.float64, device="cuda") for _ in range(4))
        amgt.spmv_fused(M, x0, e1, "jacobi", b=b, dinv=d, omega=w)
        amgt.spmv_jacobi_res(M, e1, e2, b, d, rr, omega=w)
        amgt.spmv_fused(M, e2, er, "residual", b=b)
        assert torch.equal(x1, e1) and torch.equal(x2, e2) and torch.equal(r, er)
        ref = float((rr.double() ** 2).sum())
        assert abs(float(nrm) - ref) <= 1e-12 * max(ref, 1e-300)
    # oracle: Alg. 2 formulas on the oracle SpMV (FP64, 1e-12 scaled per entry)
    xh = x0.cpu().numpy()[:A.m]
    bh = b.cpu().numpy()[:A.m]
    for mode, g in (("jacobi", x1),):
        Ax = oracle.spmv(Ao, xh)
        expect = xh + w * dh * (bh - Ax)
        tol = 1e-12 * (oracle.spmv_abs(Ao, np.abs(xh)) * w * np.abs(dh) + np.abs(xh) + np.abs(bh)) + 1e-300
        assert np.all(np.abs(g.cpu().numpy()[:A.m] - expect) <= tol), mode
    assert torch.all(x1[A.m:] == 0) and torch.all(r[A.m:] == 0)
    # two-stage forms used at the first and last cycle
    y1, y2 = (torch.empty(n, dtype=torch.float64, device="cuda") for _ in range(2))
    plan.run([("jacobi_res", x0, y1), ("residual", y1, y2)], b, d, w, norm=nrm)
    r0 = b - _pad(amgt.spmv(M, x0)[:n], n)
    ref = float((r0 ** 2).sum())
    assert abs(float(nrm) - ref) <= 1e-12 * max(ref, 1e-300) + 1e-300
    plan.run([("jacobi", x0, y1), ("residual_norm", y1, y2)], b, d, w, norm=nrm)
    assert torch.equal(y1, e1)
    ref = float((y2 ** 2).sum())
    assert abs(float(nrm) - ref) <= 1e-12 * max(ref, 1e-300) + 1e-300
    plan.close()


def test_sweeps_integer_data_exact():
    """Integer stencil, dyadic dinv (1/4), integer x and b, w = 1/2: every stage exact (P6)."""
    amgt = _amgt()
    A = gen.laplacian_5pt(40)
    Ao = oracle.as_csr(A)
    M = amgt.from_csr(A)
    n = 4 * M.blc_row
    x0 = gen.integer_vector(A.n, 4).numpy()
    b = gen.integer_vector(A.m, 5).numpy()
    d = np.full(A.m, 0.25)
    w = 0.5
    T = lambda v: _pad(torch.from_numpy(np.ascontiguousarray(v)).cuda(), n)
    ys = [torch.empty(n, dtype=torch.float64, device="cuda") for _ in range(4)]
    nrm = torch.zeros(1, dtype=torch.float64, device="cuda")
    plan = amgt.SweepPlan(M)
    plan.run([("jacobi", T(x0), ys[0]), ("jacobi", ys[0], ys[1]), ("jacobi_res", ys[1], ys[2]),
              ("residual", ys[2], ys[3])], T(b), T(d), w, norm=nrm)
    x = x0.copy()
    for k in range(3):
        r = b - oracle.spmv(Ao, x)
        if k == 2:
            assert float(nrm) == float(np.dot(r, r))
        x = x + w * d * r
        assert np.array_equal(ys[k].cpu().numpy()[:A.m], x), k
    assert np.array_equal(ys[3].cpu().numpy()[:A.m], b - oracle.spmv(Ao, x))


def test_sweeps_argument_errors():
    amgt = _amgt()
    A = gen.laplacian_5pt(16)
    M = amgt.from_csr(A)
    n = 4 * M.blc_row
    v = [torch.zeros(n, dtype=torch.float64, device="cuda") for _ in range(3)]
    plan = amgt.SweepPlan(M)
    with pytest.raises(amgt.AmgtError):  # y aliases x
        plan.run([("jacobi", v[0], v[0])], v[1], v[2])
    with pytest.raises(amgt.AmgtError):  # stage 1 does not read stage 0's output
        plan.run([("jacobi", v[0], v[1]), ("residual", v[0], v[2])], v[1], v[2])
    with pytest.raises(amgt.AmgtError):  # norm stage without a norm buffer
        plan.run([("residual_norm", v[0], v[1])], v[2])
    with pytest.raises(amgt.AmgtError):  # FP32 operator
        amgt.SweepPlan(amgt.from_csr(A, prec="f32"))


@pytest.mark.parametrize("kind,N,nlev,prec", [("7pt", 32, 5, ("f64",) * 8), ("27pt", 24, 4, ("f64",) * 8),
                                              ("7pt", 32, 5, ("f64", "f32", "f16", "f16", "f16")),
                                              ("5pt", 64, 5, ("f64",) * 8)])
def test_vcycle_with_sweeps_equals_unfused(kind, N, nlev, prec, monkeypatch):
    amgt = _amgt()
    mk = {"7pt": gen.laplacian_7pt, "27pt": gen.laplacian_27pt, "5pt": gen.laplacian_5pt}[kind]
    A = mk(N)
    dims = (N, N) if kind == "5pt" else (N, N, N)
    PR = gen.aggregation_hierarchy(dims, nlev)
    b = gen.uniform_vector(A.m, 3).cuda()
    out = {}
    for mode in ("1", "0"):
        monkeypatch.setenv("AMGT_SWEEP", mode)
        H = amgt.Hierarchy(amgt.from_csr(A), [amgt.from_csr(P) for P, _ in PR], level_prec=prec)
        for ncyc in (1, 7):
            x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
            res, calls = H.vcycle(b, x, ncyc)
            out[(mode, ncyc)] = (np.array(res), calls, x.clone())
        H.close()
    for ncyc in (1, 7):
        (r1, c1, x1), (r0, c0, x0) = out[("1", ncyc)], out[("0", ncyc)]
        assert c1 == c0 == 1 + ncyc * (5 * (nlev - 1) + 1)
        assert torch.equal(x1, x0)
        np.testing.assert_allclose(r1, r0, rtol=1e-12)
    if prec[1] == "f64":
        As = oracle.build_hierarchy(A, PR)
        _, res_o, _ = oracle.vcycle(As, PR, b.cpu().numpy(), ncycles=7)
        np.testing.assert_allclose(out[("1", 7)][0], res_o, rtol=1e-9)
