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


@pytest.mark.parametrize("thr", [0, 4, 10, 16])
@pytest.mark.parametrize("name,mk", MATS, ids=[m[0] for m in MATS])
def test_spmv_tensor_core_route(name, mk, thr):
    """Per-tile tensor-core route (R10; DMMA m8n8k4 with [A_t; A_t+1] fragments, L222-228): tiles
    with popcount >= thr through the mma, the rest on CUDA cores, long rows through the chunk
    kernel.  FP64 within 1e-12 scaled; integer data exact; every fused epilogue equals the
    CUDA-core route's within FP64 rounding."""
    amgt = _amgt()
    A = mk()
    Ao = oracle.as_csr(A)
    try:
        amgt.set_tc_threshold(17, thr)
        M = amgt.from_csr(A).analyze()
        x = gen.uniform_vector(A.n, 3).numpy()
        y = amgt.spmv(M, torch.from_numpy(x).cuda()).cpu().numpy()
        assert np.all(y[A.m:] == 0)
        check_fp64_entrywise(y[:A.m], oracle.spmv(Ao, x), oracle.spmv_abs(Ao, x))
        xi = gen.integer_vector(A.n, 12).numpy()
        Ai = oracle.Csr(Ao.m, Ao.n, Ao.row_ptr, Ao.col, np.round(Ao.val * 8))
        Mi = amgt.from_csr(gen.CSR(A.m, A.n, A.row_ptr, A.col, torch.from_numpy(Ai.val))).analyze()
        yi = amgt.spmv(Mi, torch.from_numpy(xi).cuda()).cpu().numpy()
        assert np.array_equal(yi[:A.m], oracle.spmv(Ai, xi))
        if A.m == A.n:  # fused epilogues against the plain result
            n4 = 4 * M.blc_row
            xv = torch.zeros(n4, dtype=torch.float64, device="cuda")
            xv[:A.m] = torch.from_numpy(x[:A.m])
            b = torch.from_numpy(gen.uniform_vector(n4, 5).numpy()).cuda()
            d = torch.from_numpy(gen.uniform_vector(n4, 6, 0.5, 1.0).numpy()).cuda()
            t = torch.from_numpy(y).cuda()
            for mode in ("jacobi", "residual", "accum"):
                out = torch.from_numpy(gen.uniform_vector(n4, 7).numpy()).cuda()
                ref = {"jacobi": xv + (2.0 / 3.0) * d * (b - t), "residual": b - t, "accum": out + t}[mode]
                amgt.spmv_fused(M, xv, out, mode, b=b, dinv=d)
                scale = torch.from_numpy(oracle.spmv_abs(Ao, np.abs(x)))
                err = (out - ref).abs().cpu()[:A.m]
                assert torch.all(err <= 1e-12 * (scale + ref.abs().cpu()[:A.m] + 1)), (mode, float(err.max()))
    finally:
        amgt.set_tc_threshold(17, 17)


@pytest.mark.parametrize("thr", [0, 10])
def test_spmv_fp16_tensor_core_route(thr):
    """FP16 levels on HMMA m16n8k16 (FP16 operands, x rounded to FP16, FP32 accumulation, R18): 16
    tile products per instruction from four block rows; exact on small-integer data, within the
    FP16-level tolerance (5e-3 in the 2-norm) on random data."""
    amgt = _amgt()
    try:
        amgt.set_tc_threshold(17, thr)
        for mk in (lambda: gen.laplacian_27pt(12), lambda: gen.irregular_block_sparse(1 << 11),
                   lambda: gen.random_csr(333, 333, 0.03, 9, empty_rows=20)):
            A = mk()
            Ao = oracle.as_csr(A)
            M = amgt.from_csr(A, prec="f16").analyze()
            x = gen.uniform_vector(A.n, 4).numpy()
            y = torch.empty(4 * M.blc_row, dtype=torch.float32, device="cuda")
            amgt.spmv(M, torch.from_numpy(x).float().cuda(), y)
            assert rel_2(y.double().cpu().numpy()[:A.m], oracle.spmv(Ao, x)) <= 5e-3
            Ai = oracle.Csr(Ao.m, Ao.n, Ao.row_ptr, Ao.col, np.round(Ao.val * 8))
            Mi = amgt.from_csr(gen.CSR(A.m, A.n, A.row_ptr, A.col, torch.from_numpy(Ai.val)), prec="f16").analyze()
            xi = gen.integer_vector(A.n, 12).numpy()
            amgt.spmv(Mi, torch.from_numpy(xi).float().cuda(), y)
            assert np.array_equal(y.double().cpu().numpy()[:A.m], oracle.spmv(Ai, xi))
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


@pytest.mark.parametrize("prec", [("f64",) * 4, ("f64", "f32", "f16", "f16")])
def test_vcycle_with_tensor_core_spmv(prec):
    """The V-cycle with every SpMV tile on the tensor-core routes (threshold 0): FP64 residual
    history within 1e-9 of the oracle, mixed precision within 1% per cycle, same call count."""
    amgt = _amgt()
    N, nlev = 24, 4
    A = gen.laplacian_27pt(N)
    PR = gen.aggregation_hierarchy((N, N, N), nlev)
    b = gen.uniform_vector(A.m, 3)
    try:
        amgt.set_tc_threshold(17, 0)
        H = amgt.Hierarchy(amgt.from_csr(A), [amgt.from_csr(P) for P, _ in PR], level_prec=prec)
        x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
        res, calls = H.vcycle(b.cuda(), x, 6)
        H.close()
    finally:
        amgt.set_tc_threshold(17, 17)
    _, res_o, calls_o = oracle.vcycle(oracle.build_hierarchy(A, PR), PR, b.numpy(), ncycles=6)
    assert calls == calls_o
    if prec[1] == "f64":
        np.testing.assert_allclose(res, res_o, rtol=1e-9)
    else:
        res, res_o = np.array(res), np.array(res_o)
        rho, rho_o = res[1:] / res[:-1], res_o[1:] / res_o[:-1]
        assert np.all(np.abs(rho - rho_o) <= 0.01 * rho_o), (rho, rho_o)


def _long_row_ragged(n=1536, seed=11):
    """Rows of 1..17 entries spread over the whole column range (block rows of ~4-60 tiles, mean
    >= 16): the warp-per-row kernel's loop over several 32-tile batches and its near-empty rows."""
    rng = np.random.default_rng(seed)
    rp, cols = [0], []
    for i in range(n):
        k = 0 if i % 97 == 5 else int(rng.integers(4, 17))
        c = np.unique(np.concatenate([[i], rng.integers(0, n, size=k)]))
        cols.append(c)
        rp.append(rp[-1] + len(c))
    col = np.concatenate(cols).astype(np.int32)
    val = np.round(rng.uniform(-4, 4, size=len(col))) / 4
    return gen.CSR(n, n, torch.tensor(rp, dtype=torch.int64), torch.from_numpy(col), torch.from_numpy(val))


@pytest.mark.parametrize("prec", ["f32", "f16"])
@pytest.mark.parametrize("name,mk", [("27pt_16", lambda: gen.laplacian_27pt(16)), ("long_ragged", _long_row_ragged)])
def test_spmv_warp_per_row(prec, name, mk):
    """FP32 / FP16 operators with >= 16 tiles per block row and <= 65,536 block columns take the
    warp-per-row kernel (k_spmv_wrow): dyadic data with few significant bits is exact in FP16 and
    FP32 with FP32 accumulation; every fused epilogue equals its definition on the plain product."""
    amgt = _amgt()
    A = mk()
    Ao = oracle.as_csr(A)
    M = amgt.from_csr(A, prec=prec).analyze()
    assert M.blc_num / M.blc_row >= 16
    x = (gen.integer_vector(A.n, 13).numpy() / 4).astype(np.float32)
    y = amgt.spmv(M, torch.from_numpy(x).cuda(), torch.zeros(4 * M.blc_row, dtype=torch.float32,
                                                                device="cuda")).cpu().numpy()
    assert np.array_equal(y[:A.m].astype(np.float64), oracle.spmv(Ao, x.astype(np.float64)))
    n4 = 4 * M.blc_row
    xv = torch.zeros(n4, dtype=torch.float32, device="cuda")
    xv[:A.m] = torch.from_numpy(x[:A.m])
    t = torch.from_numpy(y).cuda()
    b = torch.from_numpy((gen.integer_vector(n4, 5).numpy() / 8).astype(np.float32)).cuda()
    d = torch.full((n4,), 0.25, dtype=torch.float32, device="cuda")
    w = torch.tensor(2.0 / 3.0, dtype=torch.float32)
    for mode in ("jacobi", "residual", "accum"):
        out = torch.from_numpy((gen.integer_vector(n4, 7).numpy() / 2).astype(np.float32)).cuda()
        ref = {"jacobi": xv + w.item() * d * (b - t), "residual": b - t, "accum": out + t}[mode]
        amgt.spmv_fused(M, xv, out, mode, b=b, dinv=d)
        assert torch.allclose(out[:A.m], ref[:A.m], rtol=1e-6, atol=1e-6), mode
