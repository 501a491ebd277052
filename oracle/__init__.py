"""ORACLE — TEST INFRASTRUCTURE ONLY.

Python wrappers (ctypes) around the plain C FP64 oracle in `amgt_oracle.c`.
Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
legs may import this package.  The product path (paper_conf_sc_luzwflcy0c024_b200)
never imports it, and this package never imports the product path.

Each function below names the oracle step of SURVEY.md §8(c) and the PAPER.md lines
("Lnnn") whose definition it writes out.  Pins that tie it to the paper and to
mathematics (not to itself) live in tests/test_oracle_*.py.

Parity unpinned: none of the functions here — every one has at least one pin
(brute-force dense products, closed forms, invariants, scipy cross-checks, the
dense error-propagation operator).  See DESIGN.md "Oracle pins".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "amgt_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

_i64p = np.ctypeslib.ndpointer(dtype=np.int64, flags="C_CONTIGUOUS")
_i32p = np.ctypeslib.ndpointer(dtype=np.int32, flags="C_CONTIGUOUS")
_f64p = np.ctypeslib.ndpointer(dtype=np.float64, flags="C_CONTIGUOUS")
_u16p = np.ctypeslib.ndpointer(dtype=np.uint16, flags="C_CONTIGUOUS")
_i8p = np.ctypeslib.ndpointer(dtype=np.int8, flags="C_CONTIGUOUS")
_i64 = ctypes.c_int64


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain C99, OpenMP, no FMA contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
                               "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        L.oracle_max_threads.restype = ctypes.c_int
        L.oracle_spgemm_symbolic.restype = _i64
        L.oracle_spgemm_symbolic.argtypes = [_i64, _i64, _i64p, _i32p, _i64p, _i32p, _i64p, ctypes.c_int]
        L.oracle_spgemm_numeric.restype = None
        L.oracle_spgemm_numeric.argtypes = [_i64, _i64, _i64p, _i32p, _f64p, _i64p, _i32p, _f64p, _i64p,
                                            _i32p, _f64p, _f64p, ctypes.c_int]
        L.oracle_spmv.restype = None
        L.oracle_spmv.argtypes = [_i64, _i64p, _i32p, _f64p, _f64p, _f64p, ctypes.c_int]
        L.oracle_spmv_abs.restype = None
        L.oracle_spmv_abs.argtypes = [_i64, _i64p, _i32p, _f64p, _f64p, _f64p, ctypes.c_int]
        L.oracle_transpose.restype = None
        L.oracle_transpose.argtypes = [_i64, _i64, _i64p, _i32p, _f64p, _i64p, _i32p, _f64p]
        L.oracle_csr_to_mbsr_count.restype = _i64
        L.oracle_csr_to_mbsr_count.argtypes = [_i64, _i64p, _i32p, _i64p]
        L.oracle_csr_to_mbsr_fill.restype = None
        L.oracle_csr_to_mbsr_fill.argtypes = [_i64, _i64p, _i32p, _f64p, _i64p, _i32p, _u16p, _f64p]
        L.oracle_mbsr_to_csr_count.restype = _i64
        L.oracle_mbsr_to_csr_count.argtypes = [_i64, _i64p, _u16p, _i64p]
        L.oracle_mbsr_to_csr_fill.restype = None
        L.oracle_mbsr_to_csr_fill.argtypes = [_i64, _i64p, _i32p, _u16p, _f64p, _i64p, _i32p, _f64p]
        L.oracle_cholesky.restype = ctypes.c_int
        L.oracle_cholesky.argtypes = [_i64, _f64p]
        L.oracle_cholesky_solve.restype = None
        L.oracle_cholesky_solve.argtypes = [_i64, _f64p, _f64p, _f64p]
        L.oracle_vcycle.restype = ctypes.c_int
        L.oracle_strength_count.restype = _i64
        L.oracle_strength_count.argtypes = [_i64, _i64p, _i32p, _f64p, ctypes.c_double, _i64p]
        L.oracle_strength_fill.restype = None
        L.oracle_strength_fill.argtypes = [_i64, _i64p, _i32p, _f64p, ctypes.c_double, _i64p, _i32p, _f64p]
        L.oracle_pmis_aggregate.restype = _i64
        L.oracle_pmis_aggregate.argtypes = [_i64, _i64p, _i32p, _f64p, ctypes.c_double, ctypes.c_double, _f64p,
                                            _i8p, _i32p, ctypes.POINTER(ctypes.c_int)]
        L.oracle_pmis_weights.restype = None
        L.oracle_pmis_weights.argtypes = [_i64, ctypes.c_uint64, ctypes.c_int, _f64p]
        L.oracle_sa_combine.restype = None
        L.oracle_sa_combine.argtypes = [_i64, _i64p, _i32p, _f64p, _i64p, _i32p, _f64p, _i64p, _i32p, _f64p,
                                        ctypes.c_double]
        _lib = L
    return _lib


def max_threads() -> int:
    return int(lib().oracle_max_threads())


# ---------------------------------------------------------------- containers

@dataclass
class Csr:
    """Host CSR (numpy): row_ptr int64[m+1], col int32[nnz], val float64[nnz]."""
    m: int
    n: int
    row_ptr: np.ndarray
    col: np.ndarray
    val: np.ndarray

    @property
    def nnz(self) -> int:
        return int(self.col.size)

    def dense(self) -> np.ndarray:
        d = np.zeros((self.m, self.n))
        rows = np.repeat(np.arange(self.m), np.diff(self.row_ptr))
        np.add.at(d, (rows, self.col.astype(np.int64)), self.val)
        return d

    def pattern(self) -> np.ndarray:
        d = np.zeros((self.m, self.n), dtype=bool)
        rows = np.repeat(np.arange(self.m), np.diff(self.row_ptr))
        d[rows, self.col.astype(np.int64)] = True
        return d


@dataclass
class Mbsr:
    """Host mBSR (numpy): blc_ptr int64[BR+1], blc_idx int32[T], blc_map uint16[T],
    blc_val float64[16T] (row-major within a tile)."""
    m: int
    n: int
    blc_ptr: np.ndarray
    blc_idx: np.ndarray
    blc_map: np.ndarray
    blc_val: np.ndarray

    @property
    def blc_row(self) -> int:
        return (self.m + 3) // 4

    @property
    def blc_col(self) -> int:
        return (self.n + 3) // 4

    @property
    def blc_num(self) -> int:
        return int(self.blc_idx.size)


def as_csr(A) -> Csr:
    """Accept a gen.CSR (torch) or an oracle.Csr."""
    if isinstance(A, Csr):
        return A
    rp, ci, v = A.numpy()
    return Csr(int(A.m), int(A.n), np.ascontiguousarray(rp, dtype=np.int64),
               np.ascontiguousarray(ci, dtype=np.int32), np.ascontiguousarray(v, dtype=np.float64))


def _nt(nthreads):
    return max_threads() if nthreads is None else int(nthreads)


# ---------------------------------------------------------------- O1 / O5

def spgemm(A, B, nthreads=None, with_abs: bool = False):
    """O1: structural Gustavson C = A*B (keeps cancelled entries).  Optionally also
    returns |A||B| on C's pattern (error scale of reading R28)."""
    A, B = as_csr(A), as_csr(B)
    assert A.n == B.m, "inner dimensions"
    L = lib()
    crp = np.zeros(A.m + 1, dtype=np.int64)
    nnz = L.oracle_spgemm_symbolic(A.m, B.n, A.row_ptr, A.col, B.row_ptr, B.col, crp, _nt(nthreads))
    cci = np.zeros(max(nnz, 1), dtype=np.int32)
    cv = np.zeros(max(nnz, 1), dtype=np.float64)
    cab = np.zeros(max(nnz, 1), dtype=np.float64)
    L.oracle_spgemm_numeric(A.m, B.n, A.row_ptr, A.col, A.val, B.row_ptr, B.col, B.val, crp, cci, cv, cab,
                            _nt(nthreads))
    C = Csr(A.m, B.n, crp, cci[:nnz].copy(), cv[:nnz].copy())
    return (C, cab[:nnz].copy()) if with_abs else C


def rap(R, A, P, nthreads=None, with_abs: bool = False):
    """O5: A_c = O1(R, O1(A, P)) — the association the GPU path uses (reading R20).
    With with_abs, also returns |R|(|A||P|) on A_c's pattern (error scale, R28)."""
    R, A, P = as_csr(R), as_csr(A), as_csr(P)
    C = spgemm(R, spgemm(A, P, nthreads), nthreads)
    if not with_abs:
        return C
    Cabs = spgemm(_abs_of(R), spgemm(_abs_of(A), _abs_of(P), nthreads), nthreads)
    return C, Cabs.val


def _abs_of(A: Csr) -> Csr:
    return Csr(A.m, A.n, A.row_ptr, A.col, np.abs(A.val))


# ---------------------------------------------------------------- O3 / O4

def spmv(A, x, nthreads=None) -> np.ndarray:
    """O3: y_i = sum_k a_ik x_k in CSR order."""
    A = as_csr(A)
    x = np.ascontiguousarray(x, dtype=np.float64)
    assert x.size >= A.n
    y = np.zeros(max(A.m, 1), dtype=np.float64)
    lib().oracle_spmv(A.m, A.row_ptr, A.col, A.val, x, y, _nt(nthreads))
    return y[:A.m]


def spmv_abs(A, x, nthreads=None) -> np.ndarray:
    """|A| |x| (error scale of reading R28)."""
    A = as_csr(A)
    x = np.ascontiguousarray(x, dtype=np.float64)
    y = np.zeros(max(A.m, 1), dtype=np.float64)
    lib().oracle_spmv_abs(A.m, A.row_ptr, A.col, A.val, x, y, _nt(nthreads))
    return y[:A.m]


def transpose(A) -> Csr:
    """O4: A^T by counting sort."""
    A = as_csr(A)
    rp = np.zeros(A.n + 1, dtype=np.int64)
    ci = np.zeros(max(A.nnz, 1), dtype=np.int32)
    v = np.zeros(max(A.nnz, 1), dtype=np.float64)
    lib().oracle_transpose(A.m, A.n, A.row_ptr, A.col, A.val, rp, ci, v)
    return Csr(A.n, A.m, rp, ci[:A.nnz].copy(), v[:A.nnz].copy())


# ---------------------------------------------------------------- O2 / O7

def csr_to_mbsr(A) -> Mbsr:
    """O2: 4x4 tiles, bit = 4*(row%4) + (col%4), LSB = (0,0); values row-major,
    +0.0 where the bit is clear; tile columns ascending (L112-122; R1, R2, R6)."""
    A = as_csr(A)
    BR = (A.m + 3) // 4
    bp = np.zeros(BR + 1, dtype=np.int64)
    T = lib().oracle_csr_to_mbsr_count(A.m, A.row_ptr, A.col, bp)
    idx = np.zeros(max(T, 1), dtype=np.int32)
    mp = np.zeros(max(T, 1), dtype=np.uint16)
    val = np.zeros(max(16 * T, 16), dtype=np.float64)
    lib().oracle_csr_to_mbsr_fill(A.m, A.row_ptr, A.col, A.val, bp, idx, mp, val)
    return Mbsr(A.m, A.n, bp, idx[:T].copy(), mp[:T].copy(), val[:16 * T].copy())


def mbsr_to_csr(M: Mbsr) -> Csr:
    """O7: inverse of O2 — per scalar row, tiles in column order, set bits of the
    row's nibble in column order (L234, L262)."""
    rp = np.zeros(M.m + 1, dtype=np.int64)
    nnz = lib().oracle_mbsr_to_csr_count(M.m, M.blc_ptr, np.ascontiguousarray(M.blc_map, dtype=np.uint16), rp)
    ci = np.zeros(max(nnz, 1), dtype=np.int32)
    v = np.zeros(max(nnz, 1), dtype=np.float64)
    lib().oracle_mbsr_to_csr_fill(M.m, M.blc_ptr, np.ascontiguousarray(M.blc_idx, dtype=np.int32),
                                  np.ascontiguousarray(M.blc_map, dtype=np.uint16),
                                  np.ascontiguousarray(M.blc_val, dtype=np.float64), rp, ci, v)
    return Csr(M.m, M.n, rp, ci[:nnz].copy(), v[:nnz].copy())


def cast_values(v, prec: str) -> np.ndarray:
    """Per-level precision cast (L266): FP64 -> FP32 / FP16, round-to-nearest-even,
    directly from FP64 (reading R18).  numpy's float64->float16 conversion rounds
    directly (pinned in tests/test_oracle_cast.py)."""
    dt = {"f64": np.float64, "f32": np.float32, "f16": np.float16}[prec]
    return np.asarray(v, dtype=np.float64).astype(dt)


# ---------------------------------------------------------------- O6

def cholesky(a: np.ndarray) -> np.ndarray:
    L = np.ascontiguousarray(a, dtype=np.float64).copy()
    if lib().oracle_cholesky(L.shape[0], L) != 0:
        raise np.linalg.LinAlgError("not positive definite")
    return L


def cholesky_solve(L: np.ndarray, b: np.ndarray) -> np.ndarray:
    x = np.zeros(L.shape[0])
    lib().oracle_cholesky_solve(L.shape[0], np.ascontiguousarray(L), np.ascontiguousarray(b, dtype=np.float64), x)
    return x


def build_hierarchy(A, PR_list, nthreads=None):
    """A_1 = A; A_{k+1} = R_k A_k P_k (O5) for the given fixed (P_k, R_k)."""
    As = [as_csr(A)]
    for P, R in PR_list:
        As.append(rap(as_csr(R), As[-1], as_csr(P), nthreads))
    return As


def vcycle(As, PR_list, b, x0=None, ncycles=1, omega=2.0 / 3.0, nu1=1, nu2=1, nthreads=None, smoother="jacobi"):
    """O6: Alg. 2 (L68-82), weighted Jacobi (R21) or L1-Jacobi (D_ii = sum_j |a_ij|, L300),
    dense Cholesky coarsest (R22).  Returns (x, res_norms[ncycles+1], spmv_calls)."""
    nlev = len(As)
    assert len(PR_list) == nlev - 1
    Ps = [as_csr(p) for p, _ in PR_list]
    Rs = [as_csr(r) for _, r in PR_list]
    keep = []

    def arr(lst, attr, ctype):
        a = (ctypes.c_void_p * max(len(lst), 1))()
        for i, M in enumerate(lst):
            v = getattr(M, attr)
            keep.append(v)
            a[i] = v.ctypes.data_as(ctypes.c_void_p)
        return a

    nrows = np.array([M.m for M in As], dtype=np.int64)
    b = np.ascontiguousarray(b, dtype=np.float64)
    x = np.zeros(As[0].m) if x0 is None else np.ascontiguousarray(x0, dtype=np.float64).copy()
    res = np.zeros(ncycles + 1)
    calls = ctypes.c_int64(0)
    st = lib().oracle_vcycle(
        ctypes.c_int(nlev), nrows.ctypes.data_as(ctypes.c_void_p),
        arr(As, "row_ptr", None), arr(As, "col", None), arr(As, "val", None),
        arr(Ps, "row_ptr", None), arr(Ps, "col", None), arr(Ps, "val", None),
        arr(Rs, "row_ptr", None), arr(Rs, "col", None), arr(Rs, "val", None),
        ctypes.c_double(omega), ctypes.c_int(nu1), ctypes.c_int(nu2),
        b.ctypes.data_as(ctypes.c_void_p), x.ctypes.data_as(ctypes.c_void_p), ctypes.c_int(ncycles),
        res.ctypes.data_as(ctypes.c_void_p), ctypes.byref(calls), ctypes.c_int(_nt(nthreads)),
        ctypes.c_int({"jacobi": 0, "l1_jacobi": 1}[smoother]))
    if st != 0:
        raise RuntimeError(f"oracle_vcycle failed ({st})")
    return x, res, int(calls.value)


def vcycle_preconditioner(As, PR_list, omega=2.0 / 3.0, nu1=1, nu2=1, smoother="jacobi"):
    """M r = one O6 V-cycle on A_1 z = r from z = 0 (the PCG preconditioner, NEXT-1)."""
    def M(r):
        z, _, _ = vcycle(As, PR_list, r, x0=None, ncycles=1, omega=omega, nu1=nu1, nu2=nu2, smoother=smoother)
        return z
    return M


def pcg(A, b, M, x0=None, maxit=20):
    """PCG (NEXT-1; PCG is the solve-phase consumer named at L92), textbook recurrence in
    FP64, written out step by step:
        r0 = b - A x0, z0 = M r0, p0 = z0
        q = A p, alpha = (r,z)/(p,q), x += alpha p, r -= alpha q, z = M r,
        beta = (r,z)_new/(r,z)_old, p = z + beta p      (alpha, beta = 0 on a zero denominator)
    A: Csr (O3 SpMV), M: callable r -> z.  Returns (x, [||r_k||_2, k = 0..maxit])."""
    A = as_csr(A)
    b = np.ascontiguousarray(b, dtype=np.float64)
    x = np.zeros(A.m) if x0 is None else np.array(x0, dtype=np.float64)
    r = b - spmv(A, x)
    z = M(r)
    p = z.copy()
    rz = float(r @ z)
    res = [float(np.sqrt(r @ r))]
    for _ in range(maxit):
        q = spmv(A, p)
        pq = float(p @ q)
        alpha = rz / pq if pq != 0.0 else 0.0
        x = x + alpha * p
        r = r - alpha * q
        res.append(float(np.sqrt(r @ r)))
        z = M(r)
        rz_new = float(r @ z)
        beta = rz_new / rz if rz != 0.0 else 0.0
        p = z + beta * p
        rz = rz_new
    return x, res


# ---------------------------------------------------------------- NEXT-2: SA interpolation
def strength_filter(A, theta: float = 0.25) -> Csr:
    """O8: A_F = A without its weak off-diagonal entries, which are lumped into the diagonal
    (classical strength -a_ij >= theta max_k(-a_ik), str_thr of L300; reading R31)."""
    A = as_csr(A)
    L = lib()
    rp = np.zeros(A.m + 1, dtype=np.int64)
    nnz = L.oracle_strength_count(A.m, A.row_ptr, A.col, A.val, float(theta), rp)
    if nnz < 0:
        raise ValueError("strength filter: a row with weak entries has no diagonal entry")
    ci = np.zeros(max(nnz, 1), dtype=np.int32)
    v = np.zeros(max(nnz, 1), dtype=np.float64)
    L.oracle_strength_fill(A.m, A.row_ptr, A.col, A.val, float(theta), rp, ci, v)
    return Csr(A.m, A.n, rp, ci[:nnz], v[:nnz])


def sa_interp(A, Pt, theta: float = 0.25, omega: float = 2.0 / 3.0) -> Csr:
    """O9: P = (I - w D_F^-1 A_F) Pt through one SpGEMM (Alg. 1 line 4, L54; [35]): T = A_F Pt
    (O1, keeping cancelled entries), then P_ij = Pt_ij - (w / d_i) T_ij on T's structure."""
    AF = strength_filter(A, theta)
    Pt = as_csr(Pt)
    T = spgemm(AF, Pt)
    v = np.ascontiguousarray(T.val.copy())
    lib().oracle_sa_combine(T.m, T.row_ptr, T.col, v, Pt.row_ptr, Pt.col, Pt.val, AF.row_ptr, AF.col, AF.val,
                            float(omega))
    return Csr(T.m, T.n, T.row_ptr, T.col, v)


def build_hierarchy_sa(A, Pts, theta: float = 0.25, omega: float = 2.0 / 3.0, nthreads=None):
    """Alg. 1 with SA interpolation: per level P_k = sa_interp(A_k, Pt_k), R_k = P_k^T,
    A_{k+1} = R_k (A_k P_k) — three SpGEMM calls per level (L54, L302).  Returns (As, PR)."""
    As = [as_csr(A)]
    PR = []
    for Pt in Pts:
        P = sa_interp(As[-1], Pt, theta, omega)
        R = transpose(P)
        PR.append((P, R))
        As.append(rap(R, As[-1], P, nthreads=nthreads))
    return As, PR


# ---------------------------------------------------------------- O10 PMIS aggregation
def pmis_weights(n: int, seed: int, level: int = 0) -> np.ndarray:
    """PMIS's random weights w_i in [0, 1): the counter-based generator both sides implement
    (splitmix64 of seed + golden * (1 + i + 2^40 level); R32)."""
    w = np.zeros(max(n, 1), dtype=np.float64)
    lib().oracle_pmis_weights(int(n), int(seed) & 0xFFFFFFFFFFFFFFFF, int(level), w)
    return w[:n]


def pmis_aggregate(A, weights, theta: float = 0.25, max_row_sum: float = 0.8):
    """O10: PMIS C/F splitting on the strength graph (str_thr, max_row_sum, L300; [71] L385) and
    aggregates around the C points (reading R32).  Returns (agg int32[n], is_c int8[n],
    n_agg, rounds)."""
    A = as_csr(A)
    w = np.ascontiguousarray(weights, dtype=np.float64)
    assert w.size >= A.m
    st = np.zeros(max(A.m, 1), dtype=np.int8)
    agg = np.zeros(max(A.m, 1), dtype=np.int32)
    rounds = ctypes.c_int(0)
    nagg = lib().oracle_pmis_aggregate(A.m, A.row_ptr, A.col, A.val, float(theta), float(max_row_sum), w, st, agg,
                                       ctypes.byref(rounds))
    return agg[:A.m], st[:A.m], int(nagg), int(rounds.value)


def aggregation_from_labels(agg, nagg: int) -> Csr:
    """The tentative interpolation of an aggregation: Pt(i, agg_i) = 1."""
    agg = np.asarray(agg, dtype=np.int32)
    m = agg.size
    return Csr(m, int(nagg), np.arange(m + 1, dtype=np.int64), agg.copy(), np.ones(m, dtype=np.float64))


def build_hierarchy_pmis(A, max_levels: int, theta: float = 0.25, max_row_sum: float = 0.8, seed: int = 0,
                         max_coarse_size: int = 0, omega: float = 2.0 / 3.0, nthreads=None):
    """Alg. 1 with PMIS coarsening (O10, lines 2-3) and SA interpolation through one SpGEMM (O9,
    line 4), A_{k+1} = R_k (A_k P_k) (O5, line 5); stops at max_levels, at the first level with at
    most max_coarse_size rows (L300), or when the coarsening stalls.  Level k's PMIS weights are
    pmis_weights(n_k, seed, k).  Returns (As, PR)."""
    As = [as_csr(A)]
    PR = []
    while len(As) < max_levels:
        Ak = As[-1]
        if max_coarse_size > 0 and Ak.m <= max_coarse_size:
            break
        agg, _, nagg, _ = pmis_aggregate(Ak, pmis_weights(Ak.m, seed, len(As) - 1), theta, max_row_sum)
        if nagg == 0 or nagg >= Ak.m:
            break
        P = sa_interp(Ak, aggregation_from_labels(agg, nagg), theta, omega)
        R = transpose(P)
        PR.append((P, R))
        As.append(rap(R, Ak, P, nthreads=nthreads))
    return As, PR
