"""GPU parity: SpMV (a9) vs the oracle's CSR SpMV (O3).
FP64: |g - o| <= 1e-12 (|A||x|)_i per entry, exact on integer data; FP32 matrix levels:
1e-5 relative in the inf-norm; FP16 levels: 5e-3 relative in the 2-norm (north_star),
measured against the oracle's FP64 result on the unrounded inputs (R29)."""
import numpy as np
import pytest
import torch

import gen
import oracle
from gpu_helpers import check_fp64_entrywise, rel_2, rel_inf

pytestmark = pytest.mark.gpu


def _amgt():
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    return amgt


MATS = [
    ("cfg1", lambda: gen.laplacian_5pt(64)),
    ("7pt_24_spd", lambda: gen.laplacian_7pt(24, spd_seed=2)),
    ("27pt_12", lambda: gen.laplacian_27pt(12)),
    ("irregular_small", lambda: gen.irregular_block_sparse(1 << 11)),
    ("rand_ragged", lambda: gen.random_csr(333, 271, 0.03, 9, empty_rows=20)),
    ("rand_longrows", lambda: gen.random_csr(40, 2000, 0.4, 10)),
    ("aggregation_P", lambda: gen.aggregation_P((16, 16, 16))),            # 1 tile per block row
    ("sparse_rows", lambda: gen.random_csr(999, 3001, 0.0004, 14, empty_rows=50)),  # <= 2 tiles per row
]


@pytest.mark.parametrize("analyze", [False, True])
@pytest.mark.parametrize("name,mk", MATS, ids=[m[0] for m in MATS])
def test_spmv_fp64(name, mk, analyze):
    amgt = _amgt()
    A = mk()
    Ao = oracle.as_csr(A)
    M = amgt.from_csr(A)
    if analyze:
        M.analyze()
    x = gen.uniform_vector(A.n, 11).numpy()
    y = amgt.spmv(M, torch.from_numpy(x).cuda()).cpu().numpy()
    assert y.size == 4 * M.blc_row
    assert np.all(y[A.m:] == 0)
    check_fp64_entrywise(y[:A.m], oracle.spmv(Ao, x), oracle.spmv_abs(Ao, x))
    xi = gen.integer_vector(A.n, 12).numpy()
    Ai = oracle.Csr(Ao.m, Ao.n, Ao.row_ptr, Ao.col, np.round(Ao.val * 8))
    Mi = amgt.from_csr(gen.CSR(A.m, A.n, A.row_ptr, A.col, torch.from_numpy(Ai.val)))
    if analyze:
        Mi.analyze()
    yi = amgt.spmv(Mi, torch.from_numpy(xi).cuda()).cpu().numpy()
    assert np.array_equal(yi[:A.m], oracle.spmv(Ai, xi))  # integer data: exact


def test_spmv_long_rows_plan():
    amgt = _amgt()
    A = gen.random_csr(64, 4000, 0.5, 13)  # block rows with ~1000 tiles -> split into chunks
    M = amgt.from_csr(A).analyze()
    st = M.spmv_stats()
    assert st["long_rows"] == M.blc_row and st["chunks"] > M.blc_row
    x = gen.uniform_vector(A.n, 1).numpy()
    y = amgt.spmv(M, torch.from_numpy(x).cuda()).cpu().numpy()
    Ao = oracle.as_csr(A)
    check_fp64_entrywise(y[:A.m], oracle.spmv(Ao, x), oracle.spmv_abs(Ao, x))


@pytest.mark.parametrize("thr", [0, 4, 10])
def test_spmv_tensor_core_route(thr):
    """Per-tile DMMA route (popcount >= thr) gives the same result within FP64 tolerance."""
    amgt = _amgt()
    try:
        amgt.set_tc_threshold(10, thr)
        for mk in (lambda: gen.laplacian_27pt(12), lambda: gen.irregular_block_sparse(1 << 10)):
            A = mk()
            Ao = oracle.as_csr(A)
            M = amgt.from_csr(A)
            x = gen.uniform_vector(A.n, 3).numpy()
            y = amgt.spmv(M, torch.from_numpy(x).cuda()).cpu().numpy()
            check_fp64_entrywise(y[:A.m], oracle.spmv(Ao, x), oracle.spmv_abs(Ao, x))
    finally:
        amgt.set_tc_threshold(17, 17)


@pytest.mark.parametrize("prec,xdt", [("f32", torch.float32), ("f32", torch.float64), ("f16", torch.float32)])
def test_spmv_low_precision(prec, xdt):
    amgt = _amgt()
    for mk in (lambda: gen.laplacian_7pt(24, spd_seed=2), lambda: gen.irregular_block_sparse(1 << 11)):
        A = mk()
        Ao = oracle.as_csr(A)
        M = amgt.from_csr(A, prec=prec).analyze()
        x = gen.uniform_vector(A.n, 4).numpy()
        yo = oracle.spmv(Ao, x)
        for ydt in (torch.float32, torch.float64):
            y = torch.empty(4 * M.blc_row, dtype=ydt, device="cuda")
            amgt.spmv(M, torch.from_numpy(x).to(xdt).cuda(), y)
            g = y.double().cpu().numpy()[:A.m]
            if prec == "f32":
                assert rel_inf(g, yo) <= 1e-5, rel_inf(g, yo)
            else:
                assert rel_2(g, yo) <= 5e-3, rel_2(g, yo)


def test_spmv_fp64_matrix_fp32_vectors():
    amgt = _amgt()
    A = gen.aggregation_P((16, 16, 16))  # P * x_coarse (interpolation with FP32 coarse vector)
    M = amgt.from_csr(A)
    x = gen.uniform_vector(A.n, 5).numpy().astype(np.float32)
    y = amgt.spmv(M, torch.from_numpy(x).cuda()).cpu().numpy()
    assert np.array_equal(y[:A.m], oracle.spmv(oracle.as_csr(A), x.astype(np.float64)))


@pytest.mark.slow
@pytest.mark.parametrize("cfg", ["cfg2", "cfg4"])
def test_spmv_full_size(cfg):
    """Full sizes in the bench launch configuration, entrywise against the oracle."""
    amgt = _amgt()
    A = gen.configs.build_matrix(gen.configs.CONFIGS[cfg])
    Ao = oracle.as_csr(A)
    M = amgt.from_csr(A).analyze()
    x = gen.uniform_vector(A.n, 21).numpy()
    y = amgt.spmv(M, torch.from_numpy(x).cuda()).cpu().numpy()
    check_fp64_entrywise(y[:A.m], oracle.spmv(Ao, x), oracle.spmv_abs(Ao, x))


@pytest.mark.parametrize("dt", [torch.float64, torch.float32])
def test_spmv_fused_epilogues(dt):
    """amgt_spmv_fused: Jacobi / residual / accumulate epilogues vs oracle SpMV + the
    Alg. 2 vector formulas (FP64: 1e-12 scaled; FP32 vectors: 1e-5 inf-norm)."""
    amgt = _amgt()
    A = gen.laplacian_7pt(20, spd_seed=2)
    Ao = oracle.as_csr(A)
    M = amgt.from_csr(A, prec="f64" if dt == torch.float64 else "f32")
    x = gen.uniform_vector(A.n, 1).numpy()
    b = gen.uniform_vector(A.n, 2).numpy()
    y0 = gen.uniform_vector(A.n, 3).numpy()
    d = 1.0 / Ao.dense().diagonal()
    w = 2.0 / 3.0
    Ax = oracle.spmv(Ao, x)
    scale = oracle.spmv_abs(Ao, x)
    T = lambda v: torch.from_numpy(np.ascontiguousarray(v)).to(dt).cuda()
    cases = {"jacobi": x + w * d * (b - Ax), "residual": b - Ax, "accum": y0 + Ax, "y": Ax}
    for mode, expect in cases.items():
        y = T(y0) if mode == "accum" else torch.empty(A.m, dtype=dt, device="cuda")
        amgt.spmv_fused(M, T(x), y, mode, b=T(b), dinv=T(d), omega=w)
        g = y.double().cpu().numpy()
        if dt == torch.float64:
            tol = 1e-12 * (scale * (w * np.abs(d) if mode == "jacobi" else 1.0)) + 1e-15 * (np.abs(expect) + 1)
            assert np.all(np.abs(g - expect) <= tol), mode
        else:
            assert rel_inf(g, expect) <= 1e-5, (mode, rel_inf(g, expect))


@pytest.mark.parametrize("dt", [torch.float64, torch.float32])
def test_spmv_jacobi_res(dt):
    """amgt_spmv_fused_r: one pass gives the Jacobi sweep and the residual of its input,
    bit-identical to the separate EPI_JACOBI and EPI_RESIDUAL calls."""
    amgt = _amgt()
    A = gen.laplacian_7pt(20, spd_seed=2)
    Ao = oracle.as_csr(A)
    M = amgt.from_csr(A, prec="f64" if dt == torch.float64 else "f32")
    T = lambda v: torch.from_numpy(np.ascontiguousarray(v)).to(dt).cuda()
    x, b = T(gen.uniform_vector(A.n, 1).numpy()), T(gen.uniform_vector(A.n, 2).numpy())
    d = T(1.0 / Ao.dense().diagonal())
    y, r = torch.empty_like(x), torch.empty_like(x)
    amgt.spmv_jacobi_res(M, x, y, b, d, r)
    y2, r2 = torch.empty_like(x), torch.empty_like(x)
    amgt.spmv_fused(M, x, y2, "jacobi", b=b, dinv=d)
    amgt.spmv_fused(M, x, r2, "residual", b=b)
    assert torch.equal(y, y2) and torch.equal(r, r2)
