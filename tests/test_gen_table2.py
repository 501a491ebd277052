"""The Table II-shaped synthetic matrices (gen/table2.py; §8(f) NEXT-3) have
exactly the printed order and number of nonzeros (TSOPF_RS_b300_c3: one fewer, the printed
nnz - order is odd), and are symmetric, strictly diagonally dominant M-matrices with sorted
unique columns."""
import csv
import os

import numpy as np
import pytest
import torch

import gen.table2 as t2

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "table2_levels_calls.csv")


def _printed():
    rows = [r for r in open(GOLDEN) if not r.startswith("#")]
    return {r["matrix"]: (int(r["orders"]), int(r["nonzeros"])) for r in csv.DictReader(rows)}


def test_orders_and_nonzeros_as_printed():
    printed = _printed()
    assert len(t2.TABLE2) == len(printed) == 16
    for _, name, n, nnz in t2.TABLE2:
        assert (n, nnz) == printed[name]
        assert t2.realised_nnz(name) == nnz - ((nnz - n) & 1)


@pytest.mark.parametrize("name", ["spmsrtls", "Pres_Poisson", "Chevron2", "venkat25", "bcsstk39", "mc2depi"])
def test_matrix_properties(name):
    A = t2.table2_matrix(name)
    _, _, n, nnz = t2.BY_NAME[name]
    assert A.m == A.n == n and A.nnz == t2.realised_nnz(name)
    rp, col, val = A.numpy()
    rows = np.repeat(np.arange(n), np.diff(rp))
    # sorted unique columns per row
    assert np.all((np.diff(col.astype(np.int64)) > 0) | (np.diff(rows) > 0))
    # symmetric pattern and values
    key = rows.astype(np.int64) * n + col
    keyT = col.astype(np.int64) * n + rows
    o = np.argsort(keyT)
    assert np.array_equal(key, keyT[o]) and np.array_equal(val, val[o])
    # strictly diagonally dominant with negative off-diagonals (an M-matrix)
    diag = val[rows == col]
    off = np.zeros(n)
    np.add.at(off, rows[rows != col], np.abs(val[rows != col]))
    assert diag.size == n and np.all(val[rows != col] < 0) and np.all(diag > off)
