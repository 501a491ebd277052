"""Helpers for the -m gpu parity tests (compare the CUDA path with the oracle)."""
import numpy as np
import torch

import oracle


def mbsr_host(M):
    """Pull a device Mbsr into numpy arrays."""
    return (M.blc_ptr.cpu().numpy(), M.blc_idx.cpu().numpy(), (M.map_u16().cpu().numpy()).astype(np.uint16),
            M.blc_val.cpu().numpy())


def assert_structure_equal(M, Mo):
    """Bit-exact structure: tile row pointers, tile columns, bitmaps."""
    bp, bi, bm, _ = mbsr_host(M)
    assert M.blc_num == Mo.blc_num, (M.blc_num, Mo.blc_num)
    assert np.array_equal(bp, Mo.blc_ptr)
    assert np.array_equal(bi, Mo.blc_idx)
    assert np.array_equal(bm, Mo.blc_map)


def tile_values_to_csr_order(M):
    """Values of the structural entries in CSR order (via the device mBSR->CSR)."""
    rp, ci, v = M.to_csr()
    return rp.cpu().numpy(), ci.cpu().numpy(), v.cpu().numpy()


def check_fp64_entrywise(g, o, scale, tol=1e-12):
    """|g - o| <= tol * (|A||B|)_ij  (reading R28)."""
    err = np.abs(g - o)
    bad = err > tol * scale + 1e-300
    assert not bad.any(), f"{bad.sum()} entries out of tolerance; max rel {np.max(err / np.maximum(scale, 1e-300))}"


def rel_inf(g, o):
    return np.max(np.abs(g - o)) / max(np.max(np.abs(o)), 1e-300)


def rel_2(g, o):
    return np.linalg.norm(g - o) / max(np.linalg.norm(o), 1e-300)


def to_dev_vec(x):
    return torch.as_tensor(np.ascontiguousarray(x)).cuda()
