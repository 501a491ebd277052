"""GPU parity: CSR -> mBSR (a1), mBSR -> CSR (a8), cast (a2), transpose — vs the oracle.
Bit-exact structure and round trip; cast values bit-exact (both sides round directly
from FP64 to nearest even)."""
import numpy as np
import pytest
import torch

import gen
import oracle
from gpu_helpers import assert_structure_equal, mbsr_host

pytestmark = pytest.mark.gpu


def _amgt():
    import paper_conf_sc_luzwflcy0c024_b200 as amgt
    return amgt


CASES = [
    ("rand_1x1", lambda: gen.random_csr(1, 1, 1.0, 0)),
    ("rand_7x5", lambda: gen.random_csr(7, 5, 0.6, 1, zero_frac=0.2)),
    ("rand_ragged", lambda: gen.random_csr(203, 157, 0.05, 2, zero_frac=0.1, empty_rows=9)),
    ("rand_dense", lambda: gen.random_csr(64, 64, 0.9, 3)),
    ("empty_rows_all", lambda: gen.random_csr(13, 9, 0.0, 4)),
    ("cfg1", lambda: gen.laplacian_5pt(64)),
    ("7pt_24", lambda: gen.laplacian_7pt(24)),
    ("27pt_12", lambda: gen.laplacian_27pt(12)),
    ("irregular_small", lambda: gen.irregular_block_sparse(1 << 11)),
]


@pytest.mark.parametrize("name,mk", CASES, ids=[c[0] for c in CASES])
def test_csr_to_mbsr_bitexact_and_roundtrip(name, mk):
    amgt = _amgt()
    A = mk()
    Ao = oracle.as_csr(A)
    Mo = oracle.csr_to_mbsr(Ao)
    M = amgt.from_csr(A)
    assert M.m == A.m and M.n == A.n and M.blc_row == (A.m + 3) // 4 and M.blc_col == (A.n + 3) // 4
    assert_structure_equal(M, Mo)
    _, _, _, val = mbsr_host(M)
    assert np.array_equal(val.view(np.uint64), Mo.blc_val.view(np.uint64))  # incl. +0.0 fill (R2)
    assert M.nnz() == A.nnz
    rp, ci, v = M.to_csr()
    assert np.array_equal(rp.cpu().numpy(), Ao.row_ptr)
    assert np.array_equal(ci.cpu().numpy(), Ao.col)
    assert np.array_equal(v.cpu().numpy().view(np.uint64), Ao.val.view(np.uint64))


@pytest.mark.parametrize("prec", ["f32", "f16"])
def test_convert_with_precision_and_cast(prec):
    amgt = _amgt()
    A = gen.random_csr(150, 190, 0.08, 5)
    A = A.with_values(A.val * 37.0)  # exercise rounding
    Mo = oracle.csr_to_mbsr(oracle.as_csr(A))
    expect = oracle.cast_values(Mo.blc_val, prec)
    M = amgt.from_csr(A, prec=prec)
    assert_structure_equal(M, Mo)
    got = M.blc_val.cpu().numpy()
    assert np.array_equal(got.view(np.uint32 if prec == "f32" else np.uint16),
                          expect.view(np.uint32 if prec == "f32" else np.uint16))
    M64 = amgt.from_csr(A)
    Mc = M64.cast(prec)
    assert np.array_equal(Mc.blc_val.cpu().numpy().view(np.uint32 if prec == "f32" else np.uint16),
                          expect.view(np.uint32 if prec == "f32" else np.uint16))
    assert Mc.blc_num == M64.blc_num


def test_fp16_overflow_reported():
    amgt = _amgt()
    A = gen.random_csr(8, 8, 0.5, 6).to("cpu")
    A = A.with_values(A.val * 0 + 70000.0)
    with pytest.raises(amgt.AmgtError) as e:
        amgt.from_csr(A, prec="f16")
    assert e.value.status == 6
    M = amgt.from_csr(A)
    with pytest.raises(amgt.AmgtError) as e:
        M.cast("f16")
    assert e.value.status == 6


def test_format_errors():
    amgt = _amgt()
    rp = torch.tensor([0, 2, 3], dtype=torch.int64, device="cuda")
    ci = torch.tensor([3, 1, 0], dtype=torch.int32, device="cuda")  # unsorted row 0
    v = torch.ones(3, dtype=torch.float64, device="cuda")
    with pytest.raises(amgt.AmgtError) as e:
        amgt.csr_to_mbsr(2, 4, rp, ci, v)
    assert e.value.status == 2
    ci2 = torch.tensor([0, 9, 0], dtype=torch.int32, device="cuda")  # out of range
    with pytest.raises(amgt.AmgtError):
        amgt.csr_to_mbsr(2, 4, rp, ci2, v)
    ci3 = torch.tensor([1, 1, 0], dtype=torch.int32, device="cuda")  # duplicate
    with pytest.raises(amgt.AmgtError):
        amgt.csr_to_mbsr(2, 4, rp, ci3, v)


@pytest.mark.parametrize("name,mk", [("agg", lambda: gen.aggregation_P((10, 10, 10))),
                                     ("rand", lambda: gen.random_csr(77, 45, 0.1, 7, zero_frac=0.1))])
def test_transpose(name, mk):
    amgt = _amgt()
    A = mk()
    T = amgt.from_csr(A).transpose()
    To = oracle.csr_to_mbsr(oracle.transpose(oracle.as_csr(A)))
    assert_structure_equal(T, To)
    assert np.array_equal(T.blc_val.cpu().numpy(), To.blc_val)


@pytest.mark.slow
@pytest.mark.parametrize("cfg", ["cfg2", "cfg4"])
def test_full_size_conversion(cfg):
    """Full BASELINE sizes: structure bit-exact against the oracle packing."""
    amgt = _amgt()
    c = gen.configs.CONFIGS[cfg]
    A = gen.configs.build_matrix(c)
    Mo = oracle.csr_to_mbsr(oracle.as_csr(A))
    M = amgt.from_csr(A)
    assert_structure_equal(M, Mo)
    assert np.array_equal(M.blc_val.cpu().numpy(), Mo.blc_val)
    if cfg == "cfg2":
        assert M.blc_num == 3_620_864
