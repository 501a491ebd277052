"""Full BASELINE-size parity for config 3 (27-point 256^3, 7 levels, FP64/FP32/FP16 levels)
in the launch configuration bench.py uses (`--config cfg3`): CSR->mBSR structure and values
bit-exact, every coarse operator's structure bit-exact and values exact (dyadic data), and
the mixed-precision V-cycle's per-cycle residual reduction within 1% of the FP64 oracle's.
"""
import numpy as np
import pytest
import torch

import gen
import oracle
from gpu_helpers import assert_structure_equal, mbsr_host

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


def test_cfg3_full():
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    cfg = gen.configs.CONFIGS["cfg3"]
    A = gen.configs.build_matrix(cfg)  # CPU, shared by both sides
    PR = gen.aggregation_hierarchy(gen.configs.grid_dims(cfg), cfg.nlev, cfg.alpha)
    Ao = oracle.as_csr(A)
    assert Ao.nnz == 449_455_096
    # a1 at full size
    M = amgt.from_csr(A)
    Mo = oracle.csr_to_mbsr(Ao)
    assert M.blc_num == Mo.blc_num == 111_483_640
    assert_structure_equal(M, Mo)
    _, _, _, val = mbsr_host(M)
    assert np.array_equal(val, Mo.blc_val)
    del Mo, val
    # hierarchy (a2-a8) and V-cycle (a9-a10)
    H = amgt.Hierarchy(M, [amgt.from_csr(P) for P, _ in PR], level_prec=cfg.level_prec[:cfg.nlev])
    As = oracle.build_hierarchy(Ao, PR)
    for k in range(1, cfg.nlev):
        Ak, _, _ = H.level(k)
        assert_structure_equal(Ak, oracle.csr_to_mbsr(As[k]))
        _, _, v = Ak.to_csr()
        v = v.cpu().numpy()
        if k == 1:  # produced by the FP64 RAP of level 1, stored FP32: dyadic values, exact
            assert np.array_equal(v, As[k].val)
        else:       # FP32 / FP16 RAP chain, FP16 storage: the FP16 tolerance of north_star
            assert np.linalg.norm(v - As[k].val) <= 5e-3 * np.linalg.norm(As[k].val)
    b = gen.uniform_vector(A.m, cfg.seed)
    x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
    ncyc = 10
    res, calls = H.vcycle(b.cuda(), x, ncyc)
    _, res_o, calls_o = oracle.vcycle(As, PR, b.numpy(), ncycles=ncyc)
    assert calls == calls_o == 1 + ncyc * 31
    res, res_o = np.array(res), np.array(res_o)
    rho, rho_o = res[1:] / res[:-1], res_o[1:] / res_o[:-1]
    live = res_o[1:] / res_o[0] > 1e-10
    assert np.all(np.abs(rho[live] - rho_o[live]) <= 0.01 * rho_o[live]), (rho, rho_o)
    H.close()


def _block_rows(M, I0, I1):
    """Block rows [I0, I1) of a device mBSR as host arrays (pointers rebased to 0)."""
    ptr = M.blc_ptr[I0:I1 + 1].cpu().numpy()
    t0, t1 = int(ptr[0]), int(ptr[-1])
    return (ptr - t0, M.blc_idx[t0:t1].cpu().numpy(), (M.blc_map[t0:t1].to(torch.int32) & 0xFFFF).cpu().numpy()
            .astype(np.uint16))


def test_cfg5_full_g1_shardwise():
    """Config 5 at full size on one GPU (7-point 512^3: 134,217,728 rows, 937,951,232 nonzeros;
    the G = 1 point of the strong-scaling runs): the CSR->mBSR conversion of A_1 and the A_1 P_1
    SpGEMM of the setup, structure bit-exact against the oracle run shard-wise (the
    full 512^3 oracle would need ~22 GB of host CSR) on the first, a middle and the last 8-plane
    z-slab, plus the exact total tile counts of SURVEY 8(a) (closed forms P3)."""
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    N, planes = 512, 8
    plane = N * N
    A = gen.laplacian_7pt(N, device="cuda")
    assert A.nnz == 937_951_232
    M = amgt.from_csr(A)
    del A
    torch.cuda.empty_cache()
    assert M.blc_num == 234_094_592 == N * N * (7 * N // 4 - 3)
    P = amgt.from_csr(gen.aggregation_P((N, N, N), 0.5, device="cuda"))
    AP = amgt.spgemm_symbolic(M, P)
    assert AP.blc_num == 133_431_296 == N * N * (N - 3)  # AP tiles = N^2 (N - 3)
    for z0 in (0, N // 2 - planes // 2, N - planes):
        r0, r1 = z0 * plane, (z0 + planes) * plane
        As = oracle.as_csr(gen.laplacian_7pt(N, rows=(r0, r1)))  # global columns
        Ms = oracle.csr_to_mbsr(As)
        bp, bi, bm = _block_rows(M, r0 // 4, r1 // 4)
        assert np.array_equal(bp, Ms.blc_ptr) and np.array_equal(bi, Ms.blc_idx) and np.array_equal(bm, Ms.blc_map)
        # A P of the slab: the P rows its columns reach (one plane either side), global coarse columns
        e0, e1 = max(0, r0 - plane), min(N ** 3, r1 + plane)
        Pe = oracle.as_csr(gen.aggregation_P((N, N, N), 0.5, rows=(e0, e1)))
        Ash = oracle.Csr(As.m, e1 - e0, As.row_ptr, (As.col.astype(np.int64) - e0).astype(np.int32), As.val)
        APs = oracle.csr_to_mbsr(oracle.spgemm(Ash, Pe))
        bp, bi, bm = _block_rows(AP, r0 // 4, r1 // 4)
        assert np.array_equal(bp, APs.blc_ptr) and np.array_equal(bi, APs.blc_idx) and np.array_equal(bm, APs.blc_map)
    AP.free()
    P.free()
    M.free()
