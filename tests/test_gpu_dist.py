"""Distributed path through libamgt's distributed C ABI on one B200.

G = 2 / 4 / 8 virtual ranks run as host threads over the loopback transport
(amgt_dist_group: every transfer a device-to-device copy ordered by CUDA events, all-reduce a
rank-order sum) — the same code paths the NCCL transport runs across GPUs.  Inputs: z-slab
row partitions of the config-5 shape (7-point Laplacian, 2x2x2 aggregation, alpha = 1/2) at
sizes the oracle finishes in seconds, plus a 27-point case and a partition whose aggregates
straddle ranks.  Bar:
  * amgt_dist_spmv: bit-exact against the oracle on integer x;
  * amgt_dist_rap: structure bit-exact, values exact (dyadic data) against the oracle's rows;
  * amgt_dist_vcycle: FP64 residual history within 1e-9 of the global oracle, x within 1e-10,
    SpMV call counts equal, and identical to the single-GPU amgt_vcycle up to the order of the
    norm sums; mixed precision: per-cycle reduction within 1% of the oracle's.
"""
import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu


def _amgt():
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    return amgt


def _slab_rows(n_planes, plane, size):
    return gen.partition.slab_ranges(n_planes, plane, size)


def _run(size, rows, fn):
    from paper_conf_sc_luzwflcy0c024_b200.dist import run_loopback
    return run_loopback(size, lambda r: rows[r], fn)


@pytest.mark.parametrize("kind,dims,size", [("7pt", (32, 32, 32), 2), ("7pt", (32, 32, 32), 4),
                                            ("7pt", (16, 16, 64), 8), ("27pt", (16, 16, 32), 4)])
def test_dist_spmv_bit_exact(kind, dims, size):
    amgt = _amgt()
    offs, center = gen.partition.STENCILS[kind]
    plane = dims[0] * dims[1]
    rows = _slab_rows(dims[2], plane, size)
    A = oracle.as_csr(gen.stencil(dims, offs, center, -1.0))
    x = np.arange(A.n, dtype=np.float64) % 97 - 48
    y_ref = oracle.spmv(A, x)

    def fn(r, comm, st):
        Ar = gen.stencil(dims, offs, center, -1.0, device="cuda", rows=rows[r])
        M = amgt.from_csr(Ar)
        xl = torch.from_numpy(x[rows[r][0]:rows[r][1]]).cuda()
        y = torch.zeros(M.m, dtype=torch.float64, device="cuda")
        comm.spmv(M, xl, y)
        comm.spmv(M, xl, y)  # the cached plan
        return y.cpu().numpy()

    out = _run(size, rows, fn)
    for r, y in enumerate(out):
        assert np.array_equal(y, y_ref[rows[r][0]:rows[r][1]]), r


def _csr_rows(C, r0, r1):
    rp = C.row_ptr[r0:r1 + 1] - C.row_ptr[r0]
    return rp, C.col[C.row_ptr[r0]:C.row_ptr[r1]], C.val[C.row_ptr[r0]:C.row_ptr[r1]]


@pytest.mark.parametrize("kind,dims,splits", [
    ("7pt", (16, 16, 16), [0, 8, 16]),        # even plane split: aggregates rank-local
    ("27pt", (16, 16, 16), [0, 4, 8, 12, 16]),
    ("7pt", (8, 8, 16), [0, 5, 11, 16]),      # odd splits: aggregates straddle ranks (AP rows gathered)
])
def test_dist_rap_matches_oracle(kind, dims, splits):
    amgt = _amgt()
    offs, center = gen.partition.STENCILS[kind]
    plane = dims[0] * dims[1]
    size = len(splits) - 1
    rows = [(splits[r] * plane, splits[r + 1] * plane) for r in range(size)]
    A = oracle.as_csr(gen.stencil(dims, offs, center, -1.0))
    P = oracle.as_csr(gen.aggregation_P(dims))
    R = oracle.transpose(P)
    Ac = oracle.rap(R, A, P)
    cplane = (dims[0] // 2) * (dims[1] // 2)
    nc = P.n
    # coarse rows split evenly in whole coarse planes (independent of the fine split)
    cz = dims[2] // 2
    crows = [((r * cz) // size * cplane, ((r + 1) * cz) // size * cplane) for r in range(size)]
    Rt = gen.aggregation_R(dims)

    def fn(r, comm, st):
        Ar = amgt.from_csr(gen.stencil(dims, offs, center, -1.0, device="cuda", rows=rows[r]))
        Pr = amgt.from_csr(gen.aggregation_P(dims, device="cuda", rows=rows[r]))
        c0, c1 = crows[r]
        rp = Rt.row_ptr[c0:c1 + 1] - Rt.row_ptr[c0]
        Rc = gen.CSR(c1 - c0, Rt.n, rp.contiguous(), Rt.col[Rt.row_ptr[c0]:Rt.row_ptr[c1]].contiguous(),
                     Rt.val[Rt.row_ptr[c0]:Rt.row_ptr[c1]].contiguous())
        Rr = amgt.from_csr(Rc)
        C = comm.rap(Rr, Ar, Pr)
        rp, ci, v = C.to_csr()
        return C.m, C.n, rp.cpu().numpy(), ci.cpu().numpy(), v.cpu().numpy()

    out = _run(size, rows, fn)
    for r, (m, n, rp, ci, v) in enumerate(out):
        c0, c1 = crows[r]
        assert (m, n) == (c1 - c0, nc)
        erp, eci, ev = _csr_rows(Ac, c0, c1)
        assert np.array_equal(rp, erp) and np.array_equal(ci, eci) and np.array_equal(v, ev), r


def _vcycle_case(dims, nlev, size, prec, agg_rows, ncyc, kind="7pt"):
    amgt = _amgt()
    from paper_conf_sc_luzwflcy0c024_b200.dist import DistHierarchy
    offs, center = gen.partition.STENCILS[kind]
    plane = dims[0] * dims[1]
    rows = _slab_rows(dims[2], plane, size)
    n = plane * dims[2]
    bglob = gen.uniform_vector(n, 3)

    def fn(r, comm, st):
        A, rws, nn, Ps = gen.partition.slab_inputs(kind, dims, nlev, r, size, device="cuda")
        assert tuple(rws) == tuple(rows[r])
        MA = amgt.from_csr(A)
        MPs = [amgt.from_csr(P) for P in Ps]
        H = DistHierarchy(comm, MA, MPs, level_prec=prec, agg_rows=agg_rows)
        info = H.info()
        b = bglob[rws[0]:rws[1]].cuda()
        x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
        res, calls = H.vcycle(b, x, ncyc)
        x2 = torch.zeros_like(x)
        res2, calls2 = H.vcycle(b, x2, ncyc)  # repeatable (graphs, plans, buffers reused)
        H.close()
        return res, calls, x.cpu().numpy(), info, res2, calls2, x2.cpu().numpy()

    return _run(size, rows, fn), rows, bglob


def _expected_agg_level(dims, nlev, size, agg_rows):
    """First agglomerated level: the first level below level 1 with <= agg_rows rows, or the
    first whose 2x2x2 aggregates straddle the z-slabs (an odd number of planes per rank), the
    coarsest at the latest; everything with one rank."""
    if size == 1:
        return 0
    planes, rows = dims[2], dims[0] * dims[1] * dims[2]
    for k in range(nlev - 1):
        if k >= 1 and rows <= agg_rows:
            return k
        if planes < 2 * size or (planes // size) % 2:
            return k
        planes, rows = planes // 2, rows // 8
    return nlev - 1


def _oracle_vcycle(dims, nlev, ncyc, kind="7pt"):
    offs, center = gen.partition.STENCILS[kind]
    A = gen.stencil(dims, offs, center, -1.0)
    PR = gen.aggregation_hierarchy(dims, nlev)
    b = gen.uniform_vector(A.m, 3).numpy()
    return oracle.vcycle(oracle.build_hierarchy(A, PR), PR, b, ncycles=ncyc)


@pytest.mark.parametrize("dims,nlev,size,agg_rows", [((32, 32, 32), 4, 2, 32768), ((32, 32, 64), 5, 4, 32768),
                                                     ((32, 32, 64), 5, 8, 0), ((64, 64, 64), 6, 8, 32768),
                                                     ((32, 32, 32), 4, 4, 10 ** 9)])
def test_dist_vcycle_fp64_matches_oracle(dims, nlev, size, agg_rows):
    ncyc = 5
    out, rows, _ = _vcycle_case(dims, nlev, size, ("f64",) * nlev, agg_rows, ncyc)
    xo, res_o, calls_o = _oracle_vcycle(dims, nlev, ncyc)
    for r, (res, calls, x, info, res2, calls2, x2) in enumerate(out):
        np.testing.assert_allclose(res, res_o, rtol=1e-9)
        np.testing.assert_allclose(x, xo[rows[r][0]:rows[r][1]], rtol=0, atol=1e-10 * np.abs(xo).max())
        assert calls == calls_o == calls2
        assert np.array_equal(x, x2) and res == res2
        assert info["nlev"] == nlev
        assert info["agg_level"] == _expected_agg_level(dims, nlev, size, agg_rows)
        # every distributed level keeps the own rows inside its extended range
        for k in range(info["agg_level"]):
            eb, ee = info["ext"][k]
            assert eb <= info["row_begin"][k] and info["row_begin"][k] + info["rows"][k] <= ee
    # all ranks report the same global residual norms
    for o in out[1:]:
        assert o[0] == out[0][0]


def test_dist_vcycle_mixed_precision_rho():
    dims, nlev, ncyc = (32, 32, 64), 5, 8
    prec = ("f64", "f32", "f16", "f16", "f16")
    out, rows, _ = _vcycle_case(dims, nlev, 4, prec, 4096, ncyc)
    _, res_o, calls_o = _oracle_vcycle(dims, nlev, ncyc)
    res_o = np.array(res_o)
    rho_o = res_o[1:] / res_o[:-1]
    live = res_o[1:] / res_o[0] > 1e-10
    for res, calls, *_ in out:
        res = np.array(res)
        rho = res[1:] / res[:-1]
        assert np.all(np.abs(rho[live] - rho_o[live]) <= 0.01 * rho_o[live]), (rho, rho_o)
        assert calls == calls_o


def test_dist_vcycle_equals_single_gpu():
    """Per-row arithmetic is the single-GPU kernels': the iterate matches amgt_vcycle's (up to the
    association of the fused zero-guess epilogues), the norms up to the order of the cross-rank sum."""
    amgt = _amgt()
    dims, nlev, ncyc = (32, 32, 64), 5, 6
    prec = ("f64", "f32", "f16", "f16", "f16")
    out, rows, bglob = _vcycle_case(dims, nlev, 4, prec, 4096, ncyc)
    A = gen.laplacian_7pt(32, device="cuda", dims=dims)
    PR = gen.aggregation_hierarchy(dims, nlev)
    H = amgt.Hierarchy(amgt.from_csr(A), [amgt.from_csr(P) for P, _ in PR], level_prec=prec)
    x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
    res_s, calls_s = H.vcycle(bglob.cuda(), x, ncyc)
    xs = x.cpu().numpy()
    for r, (res, calls, xr, *_rest) in enumerate(out):
        assert calls == calls_s
        np.testing.assert_allclose(xr, xs[rows[r][0]:rows[r][1]], rtol=0, atol=1e-12 * np.abs(xs).max())
        np.testing.assert_allclose(res, res_s, rtol=1e-12)


def test_dist_vcycle_27pt():
    ncyc = 4
    dims, nlev = (16, 16, 32), 3
    out, rows, _ = _vcycle_case(dims, nlev, 2, ("f64",) * nlev, 32768, ncyc, kind="27pt")
    xo, res_o, calls_o = _oracle_vcycle(dims, nlev, ncyc, kind="27pt")
    for r, (res, calls, x, *_rest) in enumerate(out):
        np.testing.assert_allclose(res, res_o, rtol=1e-9)
        assert calls == calls_o


def test_dist_single_rank_nccl_equals_single_gpu():
    """amgt_dist_create (NCCL transport, one rank): the hierarchy is the single-GPU one."""
    amgt = _amgt()
    from paper_conf_sc_luzwflcy0c024_b200.dist import DistComm, DistHierarchy
    dims, nlev, prec = (32, 32, 32), 5, ("f64", "f32", "f16", "f16", "f16")
    A = gen.laplacian_7pt(32, device="cuda")
    PR = gen.aggregation_hierarchy(dims, nlev)
    comm = DistComm.nccl(0, 1, (0, A.m))
    MA = amgt.from_csr(A)
    MPs = [amgt.from_csr(P) for P, _ in PR]
    H = DistHierarchy(comm, MA, MPs, level_prec=prec)
    b = gen.uniform_vector(A.m, 3).cuda()
    x1 = torch.zeros(A.m, dtype=torch.float64, device="cuda")
    res1, calls1 = H.vcycle(b, x1, 6)
    Hs = amgt.Hierarchy(MA, MPs, level_prec=prec)
    x2 = torch.zeros_like(x1)
    res2, calls2 = Hs.vcycle(b, x2, 6)
    assert calls1 == calls2 and res1 == res2 and torch.equal(x1, x2)
    y = torch.zeros(A.m, dtype=torch.float64, device="cuda")
    comm.spmv(MA, b, y)
    assert torch.equal(y, amgt.spmv(MA, b))
    H.close()
    comm.close()
