"""Pins of oracle O10 (PMIS aggregation, reading R32; L300, [71] L385) against a hand-worked
example, the published splitmix64 test vector, and the invariants PMIS guarantees."""
import numpy as np
import pytest
import scipy.sparse as sp

import gen
import oracle


def _csr(M):
    M = sp.csr_matrix(M)
    M.sort_indices()
    return oracle.Csr(M.shape[0], M.shape[1], M.indptr.astype(np.int64), M.indices.astype(np.int32),
                      M.data.astype(np.float64))


def _lap1d(n):
    return _csr(sp.diags([-np.ones(n - 1), 2 * np.ones(n), -np.ones(n - 1)], [-1, 0, 1]))


def test_hand_worked_1d():
    """1D Laplacian, 5 points, w = (.1, .9, .3, .8, .5): every point influences its 1-2
    neighbours, lambda = (1.1, 2.9, 2.3, 2.8, 1.5).  Round 1: points 1 (2.9 > 1.1, 2.3) and 3
    (2.8 > 2.3, 1.5) beat all neighbours -> C; 0, 2, 4 depend on them -> F.  Aggregates: {1} = 0,
    {3} = 1; 0 -> 0; 2 depends on 1 and 3, lambda_1 = 2.9 > 2.8 -> 0; 4 -> 1."""
    agg, isc, nagg, rounds = oracle.pmis_aggregate(_lap1d(5), [0.1, 0.9, 0.3, 0.8, 0.5])
    assert list(isc) == [0, 1, 0, 1, 0] and list(agg) == [0, 0, 0, 1, 1] and nagg == 2 and rounds == 1


def test_hand_worked_two_rounds():
    """1D, 6 points, w = (.5, .1, .2, .3, .4, .9): lambda = (1.5, 2.1, 2.2, 2.3, 2.4, 1.9).
    Round 1: only 4 (2.4 > 2.3, 1.9) -> C; 3 and 5 -> F.  Round 2 (undecided 0, 1, 2): 0 (1.5 <
    2.1) no; 1 (2.1 < 2.2) no; 2 (2.2 > 2.1; 3 is decided) -> C; 1 -> F.  Round 3: 0 alone -> C.
    Aggregates: C = {0, 2, 4} -> 0, 1, 2; 1 depends on 0 and 2 (lambda 1.5 vs 2.2) -> 1; 3 on 2
    and 4 (2.2 vs 2.4) -> 2; 5 -> 2."""
    agg, isc, nagg, rounds = oracle.pmis_aggregate(_lap1d(6), [0.5, 0.1, 0.2, 0.3, 0.4, 0.9])
    assert list(isc) == [1, 0, 1, 0, 1, 0] and rounds == 3
    assert list(agg) == [0, 1, 1, 2, 2, 2] and nagg == 3


def test_strength_threshold_and_max_row_sum():
    """Row 0 of [[4, -1, -0.2], [-1, 4, -1], [-0.2, -1, 4]]: -a_02 = 0.2 < 0.25 * 1 -> weak, so
    point 2 influences only 1, point 0 only 1.  With max_row_sum = 0.6, rows whose |row sum| >
    0.6 |a_ii| (rows 0 and 2: 2.8 > 2.4; row 1: 2 <= 2.4) have no strong dependencies: only row
    1 depends on 0 and 2, so 1 influences nobody (F) and 0, 2 (no undecided neighbour) become C;
    1 joins the smaller index on the lambda tie.  With 0.4 every row is weak: all F, singletons."""
    A = _csr(np.array([[4, -1, -0.2], [-1, 4, -1], [-0.2, -1, 4]]))
    agg, isc, nagg, _ = oracle.pmis_aggregate(A, [0.5, 0.5, 0.5])
    assert list(isc) == [0, 1, 0] and list(agg) == [0, 0, 0] and nagg == 1
    agg, isc, nagg, _ = oracle.pmis_aggregate(A, [0.5, 0.5, 0.5], max_row_sum=0.6)
    assert list(isc) == [1, 0, 1] and list(agg) == [0, 0, 1] and nagg == 2
    agg, isc, nagg, _ = oracle.pmis_aggregate(A, [0.5, 0.5, 0.5], max_row_sum=0.4)
    assert list(isc) == [0, 0, 0] and list(agg) == [0, 1, 2] and nagg == 3


def test_weights_generator_splitmix64_vector():
    """w_i = splitmix64(seed + golden (1 + i)) >> 11 * 2^-53: with seed 0 the first values are
    the published splitmix64 outputs for state 0 (0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4,
    0x06C45D188009454F)."""
    w = oracle.pmis_weights(3, 0, 0)
    ref = [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F]
    assert list(w) == [(r >> 11) * 2.0 ** -53 for r in ref]
    assert not np.array_equal(oracle.pmis_weights(3, 0, 1), w)  # levels draw different numbers


def _strong_sets(A, theta=0.25, mrs=0.8):
    S = []
    for i in range(A.m):
        cols = A.col[A.row_ptr[i]:A.row_ptr[i + 1]]
        vals = A.val[A.row_ptr[i]:A.row_ptr[i + 1]]
        off = cols != i
        mi = max([-v for v, o in zip(vals, off) if o] + [0.0])
        d = vals[~off].sum()
        if mi <= 0 or (mrs < 1 and abs(vals.sum()) > mrs * abs(d)):
            S.append(set())
        else:
            S.append({int(c) for c, v, o in zip(cols, vals, off) if o and -v >= theta * mi})
    return S


@pytest.mark.parametrize("kind", ["7pt", "27pt", "7pt_spd", "5pt"])
def test_pmis_invariants(kind):
    if kind == "5pt":
        A = oracle.as_csr(gen.laplacian_5pt(24))
    elif kind == "7pt_spd":
        A = oracle.as_csr(gen.laplacian_7pt(10, spd_seed=2))
    else:
        A = oracle.as_csr(gen.laplacian_7pt(10) if kind == "7pt" else gen.laplacian_27pt(8))
    w = oracle.pmis_weights(A.m, 7, 0)
    agg, isc, nagg, rounds = oracle.pmis_aggregate(A, w)
    S = _strong_sets(A)
    ST = [set() for _ in range(A.m)]
    for i, s in enumerate(S):
        for j in s:
            ST[j].add(i)
    C = {i for i in range(A.m) if isc[i]}
    # independence: no strong edge between two C points
    assert all(not (S[i] & C) for i in C)
    # every point that influences someone and is F depends strongly on a C point
    assert all(S[i] & C for i in range(A.m) if not isc[i] and ST[i])
    # aggregates: C points are distinct roots numbered in row order; labels cover 0..nagg-1
    assert [agg[i] for i in sorted(C)] == list(range(len(C)))
    assert set(agg.tolist()) == set(range(nagg))
    # each F point sits in the aggregate of a strong C dependency when it has one
    for i in range(A.m):
        if not isc[i] and S[i] & C:
            roots = [j for j in S[i] if isc[j]]
            assert agg[i] in {agg[j] for j in roots}
    assert 1 <= rounds <= 50
    # a real coarsening on these operators
    assert nagg < A.m / 2


def test_pmis_hierarchy_converges():
    A = gen.laplacian_7pt(16)
    As, PR = oracle.build_hierarchy_pmis(A, 5, seed=3, max_coarse_size=3)
    assert 2 <= len(As) <= 5 and all(As[k + 1].m < As[k].m for k in range(len(As) - 1))
    b = gen.uniform_vector(A.m, 3).numpy()
    _, res, calls = oracle.vcycle(As, PR, b, ncycles=8)
    rho = np.array(res[1:]) / np.array(res[:-1])
    assert rho.max() < 0.5
