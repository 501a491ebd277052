"""GPU parity: interpolation through one SpGEMM call (NEXT-2, Alg. 1 line 4, L54; reading R31)
against the oracle's O8 (strength filter) and O9 (smoothed-aggregation combine):
  * A_F structure (tile pointers, columns, bitmaps) bit-exact; FP64 values exact (same
    lumping order); s = omega / diag(A_F) exact;
  * P = sa_interp(A, Pt): structure bit-exact; values exact on the integer Laplacians (T is
    dyadic, s and the two-rounding combine are the same IEEE operations), within 1e-12 of
    the scale (|Pt| + |s| |A_F| |Pt|) on random SPD data;
  * the SA hierarchy (three SpGEMM calls per level): every coarse operator's structure
    bit-exact, values to 1e-11, V-cycle residual history to 1e-9 (FP64), per-cycle
    reduction within 1% of the oracle's (mixed precision, L266)."""
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


def _dd_random(m, seed):
    """Diagonally dominant random CSR with mixed-sign off-diagonals (weak and strong ones)."""
    rng = np.random.default_rng(seed)
    d = np.where(rng.random((m, m)) < 6.0 / m, -rng.random((m, m)) * 3, 0.0)
    d += np.where(rng.random((m, m)) < 1.0 / m, rng.random((m, m)), 0.0)
    np.fill_diagonal(d, np.abs(d).sum(1) + 1.0)
    rows, cols = np.nonzero(d)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.add.at(rp, rows + 1, 1)
    return gen.CSR(m, m, torch.from_numpy(np.cumsum(rp)), torch.from_numpy(cols.astype(np.int32)),
                   torch.from_numpy(d[rows, cols].copy()))


FILTER_CASES = [
    ("7pt_spd_0.6", lambda: gen.laplacian_7pt(20, spd_seed=2), 0.6),
    ("7pt_spd_0.25", lambda: gen.laplacian_7pt(12, spd_seed=4), 0.25),
    ("27pt_10", lambda: gen.laplacian_27pt(10), 0.25),
    ("dd_random_333", lambda: _dd_random(333, 7), 0.3),
    ("dd_random_1001", lambda: _dd_random(1001, 8), 0.5),
]


@pytest.mark.parametrize("name,mk,theta", FILTER_CASES, ids=[c[0] for c in FILTER_CASES])
def test_strength_filter(name, mk, theta):
    amgt = _amgt()
    A = mk()
    AFo = oracle.strength_filter(oracle.as_csr(A), theta)
    AF, s = amgt.strength_filter(amgt.from_csr(A), theta, omega=2.0 / 3.0)
    assert_structure_equal(AF, oracle.csr_to_mbsr(AFo))
    _, _, v = AF.to_csr()
    assert np.array_equal(v.cpu().numpy(), AFo.val)
    dF = AFo.dense().diagonal() if AFo.m <= 4000 else None
    if dF is not None:
        expect = np.where(dF != 0, (2.0 / 3.0) / np.where(dF != 0, dF, 1.0), 0.0)
        assert np.array_equal(s.cpu().numpy()[:A.m], expect)


def test_strength_filter_missing_diagonal():
    amgt = _amgt()
    # row 1 has weak entries (the +1) but no diagonal entry
    d = np.array([[4.0, -1.0, 0.0], [-2.0, 0.0, 1.0], [0.0, -1.0, 3.0]])
    rows, cols = np.nonzero(d)
    A = gen.CSR(3, 3, torch.tensor([0, 2, 4, 6], dtype=torch.int64), torch.from_numpy(cols.astype(np.int32)),
                torch.from_numpy(d[rows, cols].copy()))
    with pytest.raises(amgt.AmgtError):
        amgt.strength_filter(amgt.from_csr(A), 0.25)


SA_CASES = [
    ("7pt_16", lambda: gen.laplacian_7pt(16), (16, 16, 16), True),
    ("27pt_12", lambda: gen.laplacian_27pt(12), (12, 12, 12), True),
    ("5pt_64", lambda: gen.laplacian_5pt(64), (64, 64), True),
    ("7pt_spd_16", lambda: gen.laplacian_7pt(16, spd_seed=2), (16, 16, 16), False),
]


@pytest.mark.parametrize("name,mk,dims,exact", SA_CASES, ids=[c[0] for c in SA_CASES])
def test_sa_interp(name, mk, dims, exact):
    amgt = _amgt()
    A = mk()
    Pt = gen.aggregation_P(dims)
    theta, w = 0.25, 2.0 / 3.0
    Po = oracle.sa_interp(oracle.as_csr(A), oracle.as_csr(Pt), theta, w)
    P = amgt.sa_interp(amgt.from_csr(A), amgt.from_csr(Pt), theta, w)
    assert_structure_equal(P, oracle.csr_to_mbsr(Po))
    _, _, v = P.to_csr()
    g = v.cpu().numpy()
    if exact:
        assert np.array_equal(g, Po.val)
    else:
        AFo = oracle.strength_filter(oracle.as_csr(A), theta)
        Pto = oracle.as_csr(Pt)
        T, Tabs = oracle.spgemm(AFo, Pto, with_abs=True)
        s = np.abs(w / AFo.dense().diagonal())
        scale = np.repeat(s, np.diff(T.row_ptr)) * Tabs + 1.0
        assert np.all(np.abs(g - Po.val) <= 1e-12 * scale)


def _sa_run(kind, N, nlev, prec, ncycles, spd_seed=None):
    amgt = _amgt()
    mk = {"7pt": gen.laplacian_7pt, "27pt": gen.laplacian_27pt, "5pt": gen.laplacian_5pt}[kind]
    A = mk(N, spd_seed=spd_seed) if spd_seed is not None else mk(N)
    dims = (N, N) if kind == "5pt" else (N, N, N)
    PR = gen.aggregation_hierarchy(dims, nlev)
    b = gen.uniform_vector(A.m, 3)
    H = amgt.Hierarchy(amgt.from_csr(A), [amgt.from_csr(P) for P, _ in PR], level_prec=prec, interp="sa",
                       theta=0.25, omega_p=2.0 / 3.0)
    x = torch.zeros(A.m, dtype=torch.float64, device="cuda")
    res, calls = H.vcycle(b.cuda(), x, ncycles)
    As, PRs = oracle.build_hierarchy_sa(A, [P for P, _ in PR], theta=0.25, omega=2.0 / 3.0)
    _, res_o, calls_o = oracle.vcycle(As, PRs, b.numpy(), ncycles=ncycles)
    return H, As, PRs, np.array(res), np.array(res_o), calls, calls_o


@pytest.mark.parametrize("kind,N,nlev", [("7pt", 16, 3), ("27pt", 16, 3), ("5pt", 64, 4), ("7pt", 32, 4)])
def test_sa_hierarchy_fp64(kind, N, nlev):
    H, As, PRs, res, res_o, calls, calls_o = _sa_run(kind, N, nlev, ("f64",) * 8, 8)
    assert calls == calls_o == 1 + 8 * (5 * (nlev - 1) + 1)
    np.testing.assert_allclose(res, res_o, rtol=1e-9)
    for k in range(1, H.nlev):
        Ak, Pk, _ = H.level(k)
        assert_structure_equal(Ak, oracle.csr_to_mbsr(As[k]))
        _, _, v = Ak.to_csr()
        np.testing.assert_allclose(v.cpu().numpy(), As[k].val, rtol=0, atol=1e-11 * np.abs(As[k].val).max())
    P0 = H.level(0)[1]
    assert_structure_equal(P0, oracle.csr_to_mbsr(PRs[0][0]))
    H.close()


@pytest.mark.parametrize("kind,N,nlev", [("7pt", 32, 4), ("27pt", 24, 4)])
def test_sa_hierarchy_mixed_rho_within_1pct(kind, N, nlev):
    H, As, PRs, res, res_o, calls, calls_o = _sa_run(kind, N, nlev, ("f64", "f32", "f16", "f16"), 10)
    assert calls == calls_o
    rho, rho_o = res[1:] / res[:-1], res_o[1:] / res_o[:-1]
    live = res_o[1:] / res_o[0] > 1e-10
    assert live.sum() >= 3
    assert np.all(np.abs(rho[live] - rho_o[live]) <= 0.01 * rho_o[live]), (rho, rho_o)
    H.close()
