"""Golden pins from the paper's Table II (fixture tests/golden/table2_levels_calls.csv).

The table prints, for 16 matrices, the number of AMG levels and the SpGEMM / SpMV calls of the
setup and of 50 solve iterations.  Its call counts follow the rules stated at L302 (one SpGEMM
in interpolation + two in RAP per non-coarsest level) and L308 (5 SpMV per non-coarsest level
per V-cycle, 1 residual per V-cycle, 1 initial residual; an iterative coarsest solve adds 1 or 3
per iteration).  The oracle's hierarchy build and V-cycle counter must reproduce them.
"""
import csv
import os

import numpy as np
import pytest

import gen
import oracle

HERE = os.path.dirname(os.path.abspath(__file__))
ITERS = 50  # L308: "we set the maximum number of iterations to 50, regardless of convergence"


def _rows():
    with open(os.path.join(HERE, "golden", "table2_levels_calls.csv")) as f:
        lines = [l for l in f if not l.startswith("#")]
    return [{k: (v if k in ("group", "matrix") else int(v)) for k, v in r.items()} for r in csv.DictReader(lines)]


ROWS = _rows()


def test_fixture_complete():
    assert len(ROWS) == 16
    assert {r["levels"] for r in ROWS} == {2, 3, 4, 5, 7}
    assert max(r["levels"] for r in ROWS) == 7  # L302: "no larger than seven"


def _hierarchy_1d(nlev):
    """1D 3-point Poisson of 2^(nlev-1) points with pairwise aggregation: exactly nlev levels."""
    n = 2 ** (nlev - 1) * 4
    A = gen.laplacian_7pt(n, dims=(n, 1, 1))
    PR = gen.aggregation_hierarchy((n, 1, 1), nlev)
    assert len(PR) == nlev - 1
    return A, PR


@pytest.mark.parametrize("nlev", [2, 3, 4, 5, 7])
def test_spgemm_calls_per_table2(nlev, monkeypatch):
    """Alg. 1 with interpolation through one SpGEMM (oracle.build_hierarchy_sa) issues exactly the
    #SpGEMM Table II prints for every matrix with that many levels (L302, L343: 'cant' 18 calls,
    six in interpolation)."""
    calls = {"n": 0}
    real = oracle.spgemm

    def counting(*a, **k):
        calls["n"] += 1
        return real(*a, **k)

    monkeypatch.setattr(oracle, "spgemm", counting)
    A, PR = _hierarchy_1d(nlev)
    As, _ = oracle.build_hierarchy_sa(A, [p for p, _ in PR])
    assert len(As) == nlev
    for r in ROWS:
        if r["levels"] == nlev:
            assert r["spgemm"] == calls["n"], r["matrix"]
    assert calls["n"] == 3 * (nlev - 1)


@pytest.mark.parametrize("nlev", [2, 3, 4, 5, 7])
def test_spmv_calls_per_table2(nlev):
    """The oracle's V-cycle (direct coarsest solve) counts 1 + 50 (5 (L-1) + 1) SpMV calls; every
    Table II row with L levels prints that number plus 0, 50 or 150 (L308: an iterative coarsest
    solve adds 1 or 3 SpMV per iteration)."""
    A, PR = _hierarchy_1d(nlev)
    As = oracle.build_hierarchy(A, PR)
    b = np.ones(A.m)
    _, res, calls = oracle.vcycle(As, PR, b, ncycles=ITERS)
    assert len(res) == ITERS + 1
    assert calls == 1 + ITERS * (5 * (nlev - 1) + 1)
    seen = [r for r in ROWS if r["levels"] == nlev]
    assert seen
    for r in seen:
        assert r["spmv"] - calls in (0, 50, 150), r["matrix"]


def test_spmv_direct_coarse_seven_levels_matches_L308():
    """L308 prints the direct-coarse count for 7 levels (1551) and the iterative ones (1601, 1701);
    Table II's 7-level rows all print 1701 (3 extra SpMV per iteration)."""
    A, PR = _hierarchy_1d(7)
    _, _, calls = oracle.vcycle(oracle.build_hierarchy(A, PR), PR, np.ones(A.m), ncycles=ITERS)
    assert calls == 1551
    assert {r["spmv"] for r in ROWS if r["levels"] == 7} == {calls + 3 * ITERS}
