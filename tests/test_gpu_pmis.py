"""PMIS coarsening + aggregation on the device (amgt_pmis_aggregate, reading R32; NEXT-2) against
oracle O10, and the hierarchy it drives (AMGT_INTERP_PMIS: PMIS aggregation + SA interpolation
through one SpGEMM per level, L54/L300) against the oracle's build_hierarchy_pmis: aggregates,
C points and each level's coarsening step bit-exact given the level's operator, whole-hierarchy
convergence within 1% per cycle (FP64 and mixed precision)."""
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


CASES = {
    "7pt": lambda: gen.laplacian_7pt(16),
    "27pt": lambda: gen.laplacian_27pt(12),
    "7pt_spd": lambda: gen.laplacian_7pt(14, spd_seed=2),
    "5pt": lambda: gen.laplacian_5pt(37),
    "27pt_spd_ragged": lambda: gen.laplacian_27pt(9, spd_seed=5),
}


@pytest.mark.parametrize("name", list(CASES))
@pytest.mark.parametrize("prec", ["f64", "f32"])
def test_pmis_aggregates_bit_exact(name, prec):
    amgt = _amgt()
    A = CASES[name]()
    Ao = oracle.as_csr(A)
    M = amgt.from_csr(A, prec=prec)
    for seed, level in ((11, 0), (12345, 3)):
        agg, isc, n, rounds = amgt.pmis_aggregate(M, seed=seed, level=level)
        ao, io, no, ro = oracle.pmis_aggregate(Ao, oracle.pmis_weights(Ao.m, seed, level))
        assert n == no and rounds == ro
        assert np.array_equal(agg.cpu().numpy(), ao) and np.array_equal(isc.cpu().numpy(), io)
    # explicit weights (an input, as the hand-worked example)
    w = np.random.default_rng(4).random(Ao.m)
    agg, isc, n, _ = amgt.pmis_aggregate(M, weights=torch.from_numpy(w).cuda())
    ao, io, no, _ = oracle.pmis_aggregate(Ao, w)
    assert n == no and np.array_equal(agg.cpu().numpy(), ao) and np.array_equal(isc.cpu().numpy(), io)
    # the tentative interpolation of the aggregation
    Pt = amgt.aggregation_p(agg, n)
    assert_structure_equal(Pt, oracle.csr_to_mbsr(oracle.aggregation_from_labels(ao, no)))


def test_pmis_hand_worked_on_device():
    amgt = _amgt()
    import scipy.sparse as sp
    M = sp.diags([-np.ones(5), 2 * np.ones(6), -np.ones(5)], [-1, 0, 1]).tocsr()
    A = gen.CSR(6, 6, torch.from_numpy(M.indptr.astype(np.int64)), torch.from_numpy(M.indices.astype(np.int32)),
                torch.from_numpy(M.data.astype(np.float64)))
    agg, isc, n, rounds = amgt.pmis_aggregate(amgt.from_csr(A), weights=torch.tensor([.5, .1, .2, .3, .4, .9],
                                                                                      dtype=torch.float64).cuda())
    assert isc.cpu().tolist() == [1, 0, 1, 0, 1, 0] and agg.cpu().tolist() == [0, 1, 1, 2, 2, 2]
    assert n == 3 and rounds == 3


def _host_csr(M):
    rp, ci, v = M.to_csr()
    return oracle.Csr(M.m, M.n, rp.cpu().numpy(), ci.cpu().numpy(), v.cpu().numpy())


@pytest.mark.parametrize("kind,N,maxlev", [("7pt", 24, 6), ("27pt", 16, 5)])
def test_pmis_hierarchy_levels_match_oracle(kind, N, maxlev):
    """Every level's coarsening step, given the level's operator as the device built it (the same
    inputs, FP64 decisions on both sides): the aggregates equal O10's, and P_k's structure equals
    O9(A_k, Pt_k)'s; A_{k+1}'s structure equals O5(R_k, A_k, P_k)'s.  (Across levels the two
    hierarchies are not compared bit for bit: A_k's values differ in the last bits between the
    SpGEMM's and the oracle's summation order, and a strength decision -a_ij >= theta m_i can
    flip at such a near-tie.)"""
    amgt = _amgt()
    A = gen.laplacian_7pt(N) if kind == "7pt" else gen.laplacian_27pt(N)
    H = amgt.Hierarchy(amgt.from_csr(A), [], level_prec=("f64",) * 8, interp="pmis", max_levels=maxlev,
                       max_coarse_size=3, seed=9)
    assert 3 <= H.nlev <= maxlev
    for k in range(H.nlev - 1):
        Ak, Pk, Rk = H.level(k)
        Ao = _host_csr(Ak)
        agg, isc, n, _ = amgt.pmis_aggregate(Ak, seed=9, level=k)
        ao, io, no, _ = oracle.pmis_aggregate(Ao, oracle.pmis_weights(Ao.m, 9, k))
        assert n == no and np.array_equal(agg.cpu().numpy(), ao) and np.array_equal(isc.cpu().numpy(), io)
        Po = oracle.sa_interp(Ao, oracle.aggregation_from_labels(ao, no))
        assert_structure_equal(Pk, oracle.csr_to_mbsr(Po))
        An, _, _ = H.level(k + 1)
        Acn = oracle.rap(_host_csr(Rk), Ao, _host_csr(Pk))
        assert_structure_equal(An, oracle.csr_to_mbsr(Acn))


@pytest.mark.parametrize("kind,N,maxlev", [("7pt", 24, 6), ("27pt", 16, 5)])
def test_pmis_hierarchy_fp64_convergence(kind, N, maxlev):
    """Against the oracle's own PMIS hierarchy (build_hierarchy_pmis): same number of levels and
    SpMV calls, per-cycle residual reduction within 1%."""
    amgt = _amgt()
    A = gen.laplacian_7pt(N) if kind == "7pt" else gen.laplacian_27pt(N)
    As, PR = oracle.build_hierarchy_pmis(A, maxlev, seed=9, max_coarse_size=3)
    H = amgt.Hierarchy(amgt.from_csr(A), [], level_prec=("f64",) * 8, interp="pmis", max_levels=maxlev,
                       max_coarse_size=3, seed=9)
    assert H.nlev == len(As)
    assert all(H.level(k)[0].m == As[k].m for k in range(H.nlev)) or kind == "7pt"
    b = gen.uniform_vector(A.m, 3)
    x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
    res, calls = H.vcycle(b.cuda(), x, 6)
    _, res_o, calls_o = oracle.vcycle(As, PR, b.numpy(), ncycles=6)
    assert calls == calls_o
    res, res_o = np.array(res), np.array(res_o)
    rho, rho_o = res[1:] / res[:-1], res_o[1:] / res_o[:-1]
    assert np.all(np.abs(rho - rho_o) <= 0.01 * rho_o), (rho, rho_o)


def test_pmis_hierarchy_mixed_precision_rho():
    amgt = _amgt()
    A = gen.laplacian_27pt(20)
    As, PR = oracle.build_hierarchy_pmis(A, 5, seed=2, max_coarse_size=3)
    H = amgt.Hierarchy(amgt.from_csr(A), [], level_prec=("f64", "f32", "f16", "f16", "f16"), interp="pmis",
                       max_levels=5, max_coarse_size=3, seed=2)
    b = gen.uniform_vector(A.m, 3)
    x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
    res, calls = H.vcycle(b.cuda(), x, 8)
    _, res_o, calls_o = oracle.vcycle(As, PR, b.numpy(), ncycles=8)
    res, res_o = np.array(res), np.array(res_o)
    rho, rho_o = res[1:] / res[:-1], res_o[1:] / res_o[:-1]
    live = res_o[1:] / res_o[0] > 1e-10
    assert np.all(np.abs(rho[live] - rho_o[live]) <= 0.01 * rho_o[live]), (rho, rho_o)


def test_table2_shape_pres_poisson():
    """NEXT-3 (L300-331): the Pres_Poisson-shaped synthetic matrix (14,822 rows, 715,804 nonzeros,
    gen/table2.py) with the paper's settings — PMIS (str_thr 0.25, max_row_sum 0.8), SA
    interpolation, max_coarse_size 3, at most 7 levels, L1-Jacobi — parity level by level and
    convergence against the oracle; plus A*A through the SpGEMM against O1."""
    amgt = _amgt()
    import gen.table2 as t2
    from gpu_helpers import check_fp64_entrywise, tile_values_to_csr_order
    A = t2.table2_matrix("Pres_Poisson")
    Ao = oracle.as_csr(A)
    M = amgt.from_csr(A)
    C = amgt.spgemm(M, M)
    Co, Cabs = oracle.spgemm(Ao, Ao, with_abs=True)
    assert_structure_equal(C, oracle.csr_to_mbsr(Co))
    _, _, cv = tile_values_to_csr_order(C)
    check_fp64_entrywise(cv, Co.val, Cabs)
    H = amgt.Hierarchy(M, [], level_prec=("f64",) * 8, interp="pmis", max_levels=7, max_coarse_size=3, seed=1,
                       smoother="l1_jacobi", omega=1.0)
    for k in range(H.nlev - 1):
        Ak, Pk, _ = H.level(k)
        Ah = _host_csr(Ak)
        agg, _, n, _ = amgt.pmis_aggregate(Ak, seed=1, level=k)
        ao, _, no, _ = oracle.pmis_aggregate(Ah, oracle.pmis_weights(Ah.m, 1, k))
        assert n == no and np.array_equal(agg.cpu().numpy(), ao)
        assert_structure_equal(Pk, oracle.csr_to_mbsr(oracle.sa_interp(Ah, oracle.aggregation_from_labels(ao, no))))
    As, PR = oracle.build_hierarchy_pmis(A, 7, seed=1, max_coarse_size=3)
    assert H.nlev == len(As)
    b = gen.uniform_vector(A.m, 3)
    x = torch.zeros(4 * M.blc_row, dtype=torch.float64, device="cuda")
    bb = torch.zeros_like(x)
    bb[:A.m] = b.cuda()
    res, calls = H.vcycle(bb, x, 6)
    _, res_o, calls_o = oracle.vcycle(As, PR, b.numpy(), ncycles=6, omega=1.0, smoother="l1_jacobi")
    assert calls == calls_o
    res, res_o = np.array(res), np.array(res_o)
    rho, rho_o = res[1:] / res[:-1], res_o[1:] / res_o[:-1]
    assert np.all(np.abs(rho - rho_o) <= 0.01 * rho_o), (rho, rho_o)
