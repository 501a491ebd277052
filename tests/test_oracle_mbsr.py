"""Pins for oracle O2 (CSR -> mBSR) and O7 (mBSR -> CSR) — SURVEY §8(c) P5, plus the
tile-count closed forms of P3/P4 and SURVEY §8(a) a1 popcount histogram for cfg1."""
import numpy as np
import pytest

import gen
import oracle


def _tiles_to_dense(M):
    """Expand tiles into a dense matrix + pattern via the paper's geometric meaning of a
    4x4 tile (Fig. 3 caption, L120): tile (I, J) covers rows 4I..4I+3, cols 4J..4J+3."""
    BR, BC = M.blc_row, M.blc_col
    d = np.zeros((4 * BR, 4 * BC))
    pat = np.zeros((4 * BR, 4 * BC), dtype=bool)
    for I in range(BR):
        for t in range(M.blc_ptr[I], M.blc_ptr[I + 1]):
            J = M.blc_idx[t]
            d[4 * I:4 * I + 4, 4 * J:4 * J + 4] = M.blc_val[16 * t:16 * t + 16].reshape(4, 4)
            bits = np.array([(int(M.blc_map[t]) >> b) & 1 for b in range(16)], dtype=bool).reshape(4, 4)
            pat[4 * I:4 * I + 4, 4 * J:4 * J + 4] = bits
    return d[:M.m, :M.n], pat[:M.m, :M.n], d, pat


@pytest.mark.parametrize("m,n,dens,seed", [(1, 1, 1.0, 0), (7, 5, 0.5, 1), (29, 31, 0.1, 2), (64, 64, 0.05, 3),
                                           (50, 3, 0.3, 4), (16, 16, 0.0, 5)])
def test_o2_dense_equivalence(m, n, dens, seed):
    A = oracle.as_csr(gen.random_csr(m, n, dens, seed, zero_frac=0.2, empty_rows=1))
    M = oracle.csr_to_mbsr(A)
    d, pat, dfull, patfull = _tiles_to_dense(M)
    assert np.array_equal(pat, A.pattern())            # bitmaps = structure (explicit zeros kept)
    assert np.array_equal(d, A.dense())                # values placed row-major
    assert not patfull[m:, :].any() and not patfull[:, n:].any()  # padding never set (R25)
    assert np.all(dfull[~patfull] == 0) and not np.signbit(dfull[~patfull]).any()  # +0.0 (R2)
    # P5 invariants
    assert int(sum(bin(int(x)).count("1") for x in M.blc_map)) == A.nnz
    assert np.all(M.blc_map != 0)
    for I in range(M.blc_row):
        assert np.all(np.diff(M.blc_idx[M.blc_ptr[I]:M.blc_ptr[I + 1]]) > 0)
    # O7 round trip is exact
    B = oracle.mbsr_to_csr(M)
    assert np.array_equal(B.row_ptr, A.row_ptr) and np.array_equal(B.col, A.col)
    assert np.array_equal(B.val.view(np.uint64), A.val.view(np.uint64))


def test_bit_order_single_entries():
    """Reading R1: bit = 4*row + col with LSB = (0,0)."""
    for r in range(4):
        for c in range(4):
            A = oracle.Csr(4, 4, np.array([0] * (r + 1) + [1] * (4 - r)), np.array([c], np.int32), np.array([2.5]))
            M = oracle.csr_to_mbsr(A)
            assert M.blc_num == 1 and int(M.blc_map[0]) == 1 << (4 * r + c)
            assert M.blc_val[4 * r + c] == 2.5 and np.count_nonzero(M.blc_val) == 1


def test_cfg1_tiles_and_popcounts():
    """cfg1 has 4,960 tiles with popcounts x1:1920, x4:2016, x10:1024."""
    M = oracle.csr_to_mbsr(gen.laplacian_5pt(64))
    pc = np.bincount([bin(int(x)).count("1") for x in M.blc_map], minlength=17)
    assert M.blc_num == 4960 and pc[1] == 1920 and pc[4] == 2016 and pc[10] == 1024


@pytest.mark.parametrize("N", [8, 16, 32])
def test_7pt_tile_closed_form(N):
    """P3: tiles(A_7) = N^2 (7N/4 - 3)."""
    M = oracle.csr_to_mbsr(gen.laplacian_7pt(N))
    assert M.blc_num == N * N * (7 * N // 4 - 3)


@pytest.mark.parametrize("N", [8, 16])
def test_27pt_tile_closed_form(N):
    """P4: nnz = (3N-2)^3, tiles = (3N/4 - 2)(3N-2)^2."""
    A = gen.laplacian_27pt(N)
    assert A.nnz == (3 * N - 2) ** 3
    M = oracle.csr_to_mbsr(A)
    assert M.blc_num == (3 * N // 4 - 2) * (3 * N - 2) ** 2


def test_empty_matrix():
    A = oracle.Csr(9, 6, np.zeros(10, np.int64), np.zeros(0, np.int32), np.zeros(0))
    M = oracle.csr_to_mbsr(A)
    assert M.blc_num == 0 and M.blc_ptr.size == 4 and not M.blc_ptr.any()
    B = oracle.mbsr_to_csr(M)
    assert B.nnz == 0 and not B.row_ptr.any()
