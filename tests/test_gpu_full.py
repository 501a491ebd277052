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
