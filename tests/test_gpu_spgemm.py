"""GPU parity: SpGEMM (a3-a6) and RAP (a7) vs the oracle (O1, O2, O5).
Structure bit-exact against O2(O1(A, B)); FP64 values |g - o| <= 1e-12 (|A||B|)_ij and
exact on integer/dyadic data; FP32 1e-5 (inf-norm), FP16 5e-3 (2-norm) against the
oracle's FP64 product of the unrounded inputs."""
import numpy as np
import pytest
import torch

import gen
import oracle
from gpu_helpers import assert_structure_equal, check_fp64_entrywise, rel_2, rel_inf, tile_values_to_csr_order

pytestmark = pytest.mark.gpu


def _amgt():
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    return amgt


def _check_product(C, Co_csr, Cabs=None, exact=False):
    Co = oracle.csr_to_mbsr(Co_csr)
    assert_structure_equal(C, Co)
    rp, ci, v = tile_values_to_csr_order(C)
    assert np.array_equal(rp, Co_csr.row_ptr) and np.array_equal(ci, Co_csr.col)
    if exact:
        assert np.array_equal(v, Co_csr.val)
    else:
        check_fp64_entrywise(v, Co_csr.val, Cabs)
    # +0.0 wherever the bitmap bit is clear (R2)
    val = C.blc_val.cpu().numpy().reshape(-1, 16)
    bits = ((C.map_u16().cpu().numpy()[:, None] >> np.arange(16)) & 1).astype(bool)
    assert np.all(val[~bits] == 0) and not np.signbit(val[~bits]).any()


PAIRS = [
    ("rand_small", lambda: (gen.random_csr(37, 29, 0.2, 1, zero_frac=0.1, empty_rows=3), gen.random_csr(29, 43, 0.2, 2))),
    ("rand_cancel_int", lambda: (gen.random_csr(64, 64, 0.15, 3, integer=True), gen.random_csr(64, 64, 0.15, 4, integer=True))),
    ("cfg1_AA", lambda: (gen.laplacian_5pt(64), gen.laplacian_5pt(64))),
    ("27pt_AA", lambda: (gen.laplacian_27pt(8), gen.laplacian_27pt(8))),
    ("dense_tiles", lambda: (gen.random_csr(96, 96, 0.8, 5), gen.random_csr(96, 80, 0.7, 6))),
    ("wide_rows", lambda: (gen.random_csr(16, 3000, 0.3, 7), gen.random_csr(3000, 900, 0.01, 8))),
]


@pytest.mark.parametrize("thr", [10, 0, 17])
@pytest.mark.parametrize("name,mk", PAIRS, ids=[p[0] for p in PAIRS])
def test_spgemm_fp64(name, mk, thr):
    amgt = _amgt()
    A, B = mk()
    Ao, Bo = oracle.as_csr(A), oracle.as_csr(B)
    Co, Cabs = oracle.spgemm(Ao, Bo, with_abs=True)
    amgt.set_tc_threshold(thr, 17)
    try:
        C, info = amgt.spgemm(amgt.from_csr(A), amgt.from_csr(B), info=True)
    finally:
        amgt.set_tc_threshold(17, 17)
    integer = name.endswith("_int") or name.startswith("cfg1") or name.startswith("27pt")
    _check_product(C, Co, Cabs, exact=integer)
    deg = np.diff(Bo.row_ptr)
    assert info["scalar_products"] == int(deg[Ao.col].sum())  # every scalar pair has mapC != 0 here


def test_spgemm_info_bins_and_long_rows():
    """Irregular power-law matrix: exercises several bins incl. bin 7 (dense bitmap) and the
    global-accumulation numeric path; structure bit-exact, values within 1e-12."""
    amgt = _amgt()
    A = gen.irregular_block_sparse(1 << 11, seed=5)
    Ao = oracle.as_csr(A)
    Co, Cabs = oracle.spgemm(Ao, Ao, with_abs=True)
    M = amgt.from_csr(A)
    C, info = amgt.spgemm(M, M, info=True)
    _check_product(C, Co, Cabs)
    # the analysis matches a direct count of Cub per block row
    Mo = oracle.csr_to_mbsr(Ao)
    lens = np.diff(Mo.blc_ptr)
    cub = np.array([lens[Mo.blc_idx[Mo.blc_ptr[I]:Mo.blc_ptr[I + 1]]].sum() for I in range(Mo.blc_row)])
    edges = 128 * 2 ** np.arange(7)
    bins = np.searchsorted(edges, cub, side="right")
    assert info["bin_rows"] == list(np.bincount(bins, minlength=8))
    assert info["cub_total"] == int(cub.sum())
    assert sum(info["bin_rows"][2:]) > 0 and info["numeric_rows"][1] > 0


LONG = [
    # power-law rows with > 512 C tiles, about one product per C tile: pair-record path
    ("long_records", lambda: (gen.irregular_block_sparse(1 << 13, seed=9),) * 2, True),
    # long rows with ~500 products per C tile: past the record capacity, pass 1 re-derives
    ("long_fallback", lambda: (gen.random_csr(32, 8192, 0.3, 31), gen.random_csr(8192, 4096, 0.02, 32)), True),
    # only 32 < nC <= 512 rows (warp-per-row kernel, no long-row launches)
    ("mid_only", lambda: (gen.random_csr(64, 3000, 0.3, 33), gen.random_csr(3000, 900, 0.01, 34)), False),
]


@pytest.mark.parametrize("prec", ["f64", "f32", "f16"])
@pytest.mark.parametrize("name,mk,has_long", LONG, ids=[p[0] for p in LONG])
def test_spgemm_long_rows(name, mk, has_long, prec):
    """Rows with > 512 C tiles (two-pass long-row kernels) and 32 < nC <= 512 (warp kernel)."""
    amgt = _amgt()
    A, B = mk()
    Ao, Bo = oracle.as_csr(A), oracle.as_csr(B)
    Co, Cabs = oracle.spgemm(Ao, Bo, with_abs=True)
    C = amgt.spgemm(amgt.from_csr(A, prec=prec), amgt.from_csr(B, prec=prec))
    nC = np.diff(C.blc_ptr.cpu().numpy())
    assert (nC.max() > 512) == has_long and nC.max() > 32
    if prec == "f64":
        _check_product(C, Co, Cabs)
        return
    assert_structure_equal(C, oracle.csr_to_mbsr(Co))
    _, _, v = tile_values_to_csr_order(C)
    if prec == "f32":
        assert rel_inf(v, Co.val) <= 1e-5
    else:
        assert rel_2(v, Co.val) <= 5e-3


@pytest.mark.parametrize("prec", ["f32", "f16"])
def test_spgemm_low_precision(prec):
    amgt = _amgt()
    A = gen.laplacian_7pt(16, spd_seed=2)
    P = gen.aggregation_P((16, 16, 16), 0.5)
    for X, Y in ((A, P), (A, A)):
        Xo, Yo = oracle.as_csr(X), oracle.as_csr(Y)
        Co = oracle.spgemm(Xo, Yo)
        C = amgt.spgemm(amgt.from_csr(X, prec=prec), amgt.from_csr(Y, prec=prec))
        assert_structure_equal(C, oracle.csr_to_mbsr(Co))
        _, _, v = tile_values_to_csr_order(C)
        if prec == "f32":
            assert rel_inf(v, Co.val) <= 1e-5
        else:
            assert rel_2(v, Co.val) <= 5e-3


@pytest.mark.parametrize("kind,N,alpha", [("7pt", 24, 0.5), ("27pt", 16, 0.5), ("7pt", 16, 1.0)])
def test_rap_closed_form_and_oracle(kind, N, alpha):
    amgt = _amgt()
    A = {"7pt": gen.laplacian_7pt, "27pt": gen.laplacian_27pt}[kind](N)
    P = gen.aggregation_P((N, N, N), alpha)
    R = gen.aggregation_R((N, N, N), alpha)
    Co = oracle.rap(R, A, P)
    Ac = amgt.rap(amgt.from_csr(R), amgt.from_csr(A), amgt.from_csr(P))
    _check_product(Ac, Co, exact=True)  # dyadic data: exact
    if kind == "7pt":
        ref = oracle.as_csr(gen.laplacian_7pt(N // 2))
        _, _, v = tile_values_to_csr_order(Ac)
        assert np.array_equal(v, ref.val * 4 * alpha * alpha)


def test_rap_random_spd_tolerance():
    amgt = _amgt()
    N = 20
    A = gen.laplacian_7pt(N, spd_seed=2)
    P = gen.aggregation_P((N, N, N), 0.5)
    R = gen.aggregation_R((N, N, N), 0.5)
    Co, Cabs = oracle.rap(R, A, P, with_abs=True)
    Ac = amgt.rap(amgt.from_csr(R), amgt.from_csr(A), amgt.from_csr(P))
    _check_product(Ac, Co, Cabs)


@pytest.mark.slow
def test_rap_cfg2_full():
    """Config 2 at full size (7-point 128^3): A*P and R*(AP) structure bit-exact, values exact."""
    amgt = _amgt()
    N = 128
    A = gen.laplacian_7pt(N)
    P = gen.aggregation_P((N, N, N), 0.5)
    R = gen.aggregation_R((N, N, N), 0.5)
    Mo_AP = oracle.spgemm(A, P)
    MA, MP, MR = amgt.from_csr(A), amgt.from_csr(P), amgt.from_csr(R)
    AP, info = amgt.spgemm(MA, MP, info=True)
    assert AP.blc_num == 2_048_000
    _check_product(AP, Mo_AP, exact=True)
    Ac = amgt.spgemm(MR, AP)
    assert Ac.blc_num == 446_464
    _check_product(Ac, oracle.spgemm(R, Mo_AP), exact=True)


@pytest.mark.slow
def test_spgemm_cfg4_full():
    """Config 4 at full size: A*A structure bit-exact, values within 1e-12 (|A||A|)."""
    amgt = _amgt()
    A = gen.configs.build_matrix(gen.configs.CONFIGS["cfg4"])
    Ao = oracle.as_csr(A)
    Co, Cabs = oracle.spgemm(Ao, Ao, with_abs=True)
    M = amgt.from_csr(A)
    C, info = amgt.spgemm(M, M, info=True)
    _check_product(C, Co, Cabs)


@pytest.mark.parametrize("thr", [0, 10, 17])
@pytest.mark.parametrize("prec", ["f16", "f64", "f32"])
def test_spgemm_tc_routes_integer_exact(prec, thr):
    """Tensor-core routes (FP64 DMMA m8n8k4, FP16 HMMA m16n8k8 with FP32 accumulation) and the
    CUDA-core route give the exact product on small-integer data (exact in every precision)."""
    amgt = _amgt()
    A = gen.random_csr(96, 88, 0.35, 21, integer=True)
    B = gen.random_csr(88, 72, 0.35, 22, integer=True)
    Co = oracle.spgemm(A, B)
    assert np.abs(Co.val).max() < 2048
    amgt.set_tc_threshold(thr, 17)
    try:
        C, info = amgt.spgemm(amgt.from_csr(A, prec=prec), amgt.from_csr(B, prec=prec), info=True)
    finally:
        amgt.set_tc_threshold(17, 17)
    if thr == 0:
        assert info["pairs_tc"] == info["pairs_nonzero"]
    assert_structure_equal(C, oracle.csr_to_mbsr(Co))
    _, _, v = tile_values_to_csr_order(C)
    assert np.array_equal(v, Co.val)


@pytest.mark.parametrize("thr", [0, 17])
def test_spgemm_fp16_tc_tolerance(thr):
    amgt = _amgt()
    A = gen.random_csr(128, 128, 0.6, 23)
    Ao = oracle.as_csr(A)
    Co = oracle.spgemm(Ao, Ao)
    amgt.set_tc_threshold(thr, 17)
    try:
        M = amgt.from_csr(A, prec="f16")
        C = amgt.spgemm(M, M)
    finally:
        amgt.set_tc_threshold(17, 17)
    _, _, v = tile_values_to_csr_order(C)
    assert rel_2(v, Co.val) <= 5e-3


_BINS_SCRIPT = r"""
import sys, numpy as np
sys.path.insert(0, sys.argv[1])
import gen, paper_conf_sc_luzwflcy0c024_b200 as amgt
A = gen.irregular_block_sparse(1 << 11, seed=5)
M = amgt.from_csr(A)
C = amgt.spgemm(M, M)
np.savez(sys.argv[2], ptr=C.blc_ptr.cpu().numpy(), idx=C.blc_idx.cpu().numpy(), map=C.map_u16().cpu().numpy(),
         val=C.blc_val.cpu().numpy())
"""


@pytest.mark.parametrize("dense_from", ["2", "7"])
def test_spgemm_hash_and_dense_bins_agree(tmp_path, dense_from):
    """The per-bin hash kernels (bins 2-6) and the dense-bitmap kernel give the same C:
    AMGT_DENSE_FROM_BIN = 7 (hash for bins 2-6) and 2 (dense for all of them) in separate
    processes (the knob is read once), each bit-exact in structure against the oracle."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    script = tmp_path / "bins.py"
    script.write_text(_BINS_SCRIPT)
    out = tmp_path / "c.npz"
    env = dict(os.environ, AMGT_DENSE_FROM_BIN=dense_from)
    p = subprocess.run([sys.executable, str(script), root, str(out)], env=env, capture_output=True, text=True,
                       timeout=300)
    assert p.returncode == 0, p.stderr[-2000:]
    got = np.load(out)
    A = gen.irregular_block_sparse(1 << 11, seed=5)
    Ao = oracle.as_csr(A)
    Co = oracle.csr_to_mbsr(oracle.spgemm(Ao, Ao))
    assert np.array_equal(got["ptr"], Co.blc_ptr)
    assert np.array_equal(got["idx"], Co.blc_idx)
    assert np.array_equal(got["map"], Co.blc_map.astype(np.int32))


def test_spgemm_plan_reused_after_value_change():
    """The symbolic phase's numeric plan (records of the whole-GPU dense rows) depends on the
    structure only: a second numeric call on the same C, and one after A's values are scaled in
    place by 2, both match the oracle (the latter against 4x the product; power-of-two scaling is
    exact) within the FP64 bound."""
    amgt = _amgt()
    A = gen.irregular_block_sparse(1 << 12, seed=11)
    Ao = oracle.as_csr(A)
    Co, Cabs = oracle.spgemm(Ao, Ao, with_abs=True)
    M = amgt.from_csr(A)
    C, info = amgt.spgemm(M, M, info=True)
    assert sum(info["bin_rows"][2:]) > 0
    _check_product(C, Co, Cabs)
    amgt.spgemm_numeric(M, M, C)  # same inputs again
    _check_product(C, Co, Cabs)
    M.blc_val.mul_(2.0)
    amgt.spgemm_numeric(M, M, C)
    Co4 = oracle.Csr(Co.m, Co.n, Co.row_ptr, Co.col, 4.0 * Co.val)
    _check_product(C, Co4, 4.0 * Cabs)


_NOPLAN_SCRIPT = r"""
import sys, numpy as np
sys.path.insert(0, sys.argv[1])
import gen, paper_conf_sc_luzwflcy0c024_b200 as amgt
cases = {
    "power_law": lambda: (gen.irregular_block_sparse(1 << 13, seed=9),) * 2,
    "long_dense": lambda: (gen.random_csr(32, 8192, 0.3, 31), gen.random_csr(8192, 4096, 0.02, 32)),
    "mid_only": lambda: (gen.random_csr(64, 3000, 0.3, 33), gen.random_csr(3000, 900, 0.01, 34)),
}
A, B = cases[sys.argv[3]]()
C = amgt.spgemm(amgt.from_csr(A, prec=sys.argv[4]), amgt.from_csr(B, prec=sys.argv[4]))
np.savez(sys.argv[2], ptr=C.blc_ptr.cpu().numpy(), idx=C.blc_idx.cpu().numpy(), map=C.map_u16().cpu().numpy(),
         val=C.blc_val.float().double().cpu().numpy() if sys.argv[4] == "f16" else C.blc_val.double().cpu().numpy())
"""


@pytest.mark.parametrize("prec", ["f64", "f16"])
@pytest.mark.parametrize("case", ["power_law", "long_dense", "mid_only"])
def test_spgemm_searching_kernels_without_plan(tmp_path, case, prec):
    """AMGT_SPGEMM_PLAN=0 (separate process; the knob is read once): the rows past 32 C tiles take
    the searching kernels (warp rows 33-512, two-pass long rows with pair records) instead of the
    symbolic phase's records (R34) — structure bit-exact, FP64 values within 1e-12 (|A||B|),
    FP16 within 5e-3 (2-norm)."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    script = tmp_path / "noplan.py"
    script.write_text(_NOPLAN_SCRIPT)
    out = tmp_path / "c.npz"
    env = dict(os.environ, AMGT_SPGEMM_PLAN="0")
    p = subprocess.run([sys.executable, str(script), root, str(out), case, prec], env=env, capture_output=True,
                       text=True, timeout=300)
    assert p.returncode == 0, p.stderr[-2000:]
    got = np.load(out)
    A, B = {
        "power_law": lambda: (gen.irregular_block_sparse(1 << 13, seed=9),) * 2,
        "long_dense": lambda: (gen.random_csr(32, 8192, 0.3, 31), gen.random_csr(8192, 4096, 0.02, 32)),
        "mid_only": lambda: (gen.random_csr(64, 3000, 0.3, 33), gen.random_csr(3000, 900, 0.01, 34)),
    }[case]()
    Ao, Bo = oracle.as_csr(A), oracle.as_csr(B)
    Co, Cabs = oracle.spgemm(Ao, Bo, with_abs=True)
    Cm = oracle.csr_to_mbsr(Co)
    assert np.array_equal(got["ptr"], Cm.blc_ptr)
    assert np.array_equal(got["idx"], Cm.blc_idx)
    assert np.array_equal(got["map"], Cm.blc_map.astype(np.int32))
    assert np.diff(got["ptr"]).max() > 32
    # values in CSR order from the dense tiles (bits set in the bitmap, row-major within a tile row)
    om = oracle.csr_to_mbsr(Co)
    vals = got["val"].reshape(-1, 16)
    ref = np.asarray(om.blc_val).reshape(-1, 16)
    bits = ((got["map"][:, None] >> np.arange(16)) & 1).astype(bool)
    g, r = vals[bits], ref[bits]
    if prec == "f64":
        absm = oracle.csr_to_mbsr(oracle.Csr(Co.m, Co.n, Co.row_ptr, Co.col, Cabs))
        bound = 1e-12 * np.asarray(absm.blc_val).reshape(-1, 16)[bits]
        assert np.all(np.abs(g - r) <= bound + 1e-300)
    else:
        assert np.linalg.norm(g - r) <= 5e-3 * np.linalg.norm(r)


_DET_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import gen, paper_conf_sc_luzwflcy0c024_b200 as amgt
prec = sys.argv[3]
A = gen.irregular_block_sparse(1 << 13, seed=9)
M = amgt.from_csr(A, prec=prec)
C, info = amgt.spgemm(M, M, info=True)
bits = {"f16": torch.int16, "f32": torch.int32, "f64": torch.int64}[prec]
v1 = C.blc_val.clone()
same = True
for _ in range(3):
    amgt.spgemm_numeric(M, M, C)
    same = same and torch.equal(C.blc_val.view(bits), v1.view(bits))
C2 = amgt.spgemm(M, M)  # a fresh symbolic phase (new slot assignment)
same = same and torch.equal(C2.blc_val.view(bits), v1.view(bits))
np.savez(sys.argv[2], same=same, multi=info["pairs_nonzero"] > C.blc_num, ptr=C.blc_ptr.cpu().numpy(),
         idx=C.blc_idx.cpu().numpy(), map=C.map_u16().cpu().numpy(), val=C.blc_val.double().cpu().numpy())
"""


@pytest.mark.parametrize("prec", ["f64", "f32", "f16"])
def test_spgemm_multi_product_tiles_bitwise_reproducible(tmp_path, prec):
    """AMGT_SPGEMM_DET=1 (separate process): the plan rows' tiles with several products are summed in
    ascending A-tile order from their product slots (k_plan_msum), not by atomics: repeated numeric
    calls and a fresh symbolic phase give bit-identical values, and the product matches the oracle."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    script = tmp_path / "det.py"
    script.write_text(_DET_SCRIPT)
    out = tmp_path / "c.npz"
    env = dict(os.environ, AMGT_SPGEMM_DET="1")
    p = subprocess.run([sys.executable, str(script), root, str(out), prec], env=env, capture_output=True, text=True,
                       timeout=300)
    assert p.returncode == 0, p.stderr[-2000:]
    got = np.load(out)
    assert bool(got["multi"]) and bool(got["same"])
    A = gen.irregular_block_sparse(1 << 13, seed=9)
    Ao = oracle.as_csr(A)
    Co, Cabs = oracle.spgemm(Ao, Ao, with_abs=True)
    Cm = oracle.csr_to_mbsr(Co)
    assert np.array_equal(got["ptr"], Cm.blc_ptr) and np.array_equal(got["idx"], Cm.blc_idx)
    bits = ((got["map"][:, None] >> np.arange(16)) & 1).astype(bool)
    g = got["val"].reshape(-1, 16)[bits]
    r = np.asarray(Cm.blc_val).reshape(-1, 16)[bits]
    if prec == "f64":
        absm = oracle.csr_to_mbsr(oracle.Csr(Co.m, Co.n, Co.row_ptr, Co.col, Cabs))
        assert np.all(np.abs(g - r) <= 1e-12 * np.asarray(absm.blc_val).reshape(-1, 16)[bits] + 1e-300)
    elif prec == "f32":
        assert np.max(np.abs(g - r)) <= 1e-5 * np.max(np.abs(r))
    else:
        assert np.linalg.norm(g - r) <= 5e-3 * np.linalg.norm(r)
