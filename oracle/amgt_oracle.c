/*
 * ORACLE — TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct CPU FP64 implementation of what the AmgT hot path
 * computes (Lu et al., "AmgT: Algebraic Multigrid Solver on Tensor Cores", SC'24;
 * citations are /root/reference/PAPER.md line numbers, "Lnnn").  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load this library.  It shares no code, header, table or helper with the CUDA
 * path (paper_conf_sc_luzwflcy0c024_b200/csrc), and neither includes the other.
 *
 * Every function is the plain definition:
 *   O1 oracle_spgemm_*      structural Gustavson C = A*B (L145-213 define the result:
 *                           C(i,:) = sum_k A(i,k) B(k,:); structure keeps cancelled
 *                           entries, reading R3/R5), plus (|A||B|)_ij for error scaling.
 *   O2 oracle_csr_to_mbsr_* 4x4 tiles with 16-bit bitmaps (L112-122, Fig. 3 caption L120;
 *                           readings R1 bit = 4*row+col, LSB=(0,0); R2 row-major values,
 *                           +0.0 where the bit is clear; R6 ascending tile columns).
 *   O3 oracle_spmv          y_i = sum_k a_ik x_k in CSR order (L218).
 *   O4 oracle_transpose     R = P^T by counting sort (Alg. 1 line 4, L54).
 *   O5 RAP                  A_c = O1(R, O1(A, P)) (Alg. 1 line 5, L54; reading R20).
 *   O6 oracle_vcycle        Alg. 2 (L68-82) with weighted Jacobi x += w D^-1 (b - A x)
 *                           (reading R21; smoother 1: L1-Jacobi, D_ii = sum_j |a_ij|,
 *                           L300), dense Cholesky on the coarsest level (R22),
 *                           records ||r||_2 per cycle and SpMV calls (L308).
 *   O7 oracle_mbsr_to_csr_* inverse of O2 (L234, L262).
 *   O8 oracle_strength_*    strength-of-connection filter (§8(f) NEXT-2; classical strength
 *                           with str_thr = theta, L300; reading R31): off-diagonal a_ij is
 *                           strong iff -a_ij >= theta * max_{k!=i}(-a_ik) > 0; weak entries
 *                           are dropped and added to the diagonal in column order.
 *   O9 oracle_sa_combine    interpolation through one SpGEMM call (Alg. 1 line 4, L54; [35]
 *                           L385; reading R31): P = Pt - (w / d_i) * T_ij on the structure of
 *                           T = A_F Pt (O1), Pt the tentative (aggregation) interpolation.
 *
 * No blocking, fusion or reordering beyond the definitions.  OpenMP only splits the
 * independent outer row loop; per-row arithmetic order is fixed, so results do not
 * depend on the thread count.  Compiled with -O2 -ffp-contract=off (no FMA fusion).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

static int cmp_i32(const void* a, const void* b) {
    int32_t x = *(const int32_t*)a, y = *(const int32_t*)b;
    return (x > y) - (x < y);
}

int oracle_max_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* ---------------------------------------------------------------- O1 SpGEMM */

/* Row counts of C = A*B (structural).  crp[0..m] is filled (exclusive prefix sum).
 * Returns nnz(C).  A is m x k, B is k x n. */
int64_t oracle_spgemm_symbolic(int64_t m, int64_t n, const int64_t* arp, const int32_t* aci,
                               const int64_t* brp, const int32_t* bci, int64_t* crp, int nthreads) {
    if (nthreads < 1) nthreads = 1;
    int64_t* cnt = (int64_t*)calloc((size_t)(m > 0 ? m : 1), sizeof(int64_t));
#pragma omp parallel num_threads(nthreads)
    {
        int64_t* mark = (int64_t*)malloc((size_t)(n > 0 ? n : 1) * sizeof(int64_t));
        for (int64_t j = 0; j < n; ++j) mark[j] = -1;
#pragma omp for schedule(dynamic, 256)
        for (int64_t i = 0; i < m; ++i) {
            int64_t c = 0;
            for (int64_t p = arp[i]; p < arp[i + 1]; ++p) {
                int32_t k = aci[p];
                for (int64_t q = brp[k]; q < brp[k + 1]; ++q) {
                    int32_t j = bci[q];
                    if (mark[j] != i) { mark[j] = i; ++c; }
                }
            }
            cnt[i] = c;
        }
        free(mark);
    }
    crp[0] = 0;
    for (int64_t i = 0; i < m; ++i) crp[i + 1] = crp[i] + cnt[i];
    free(cnt);
    return crp[m];
}

/* Values: for each row i, for k in A(i,:) in column order, for j in B(k,:):
 * acc[j] += a_ik * b_kj; absacc[j] += |a_ik| * |b_kj|.  Columns emitted ascending. */
void oracle_spgemm_numeric(int64_t m, int64_t n, const int64_t* arp, const int32_t* aci, const double* av,
                           const int64_t* brp, const int32_t* bci, const double* bv, const int64_t* crp,
                           int32_t* cci, double* cv, double* cabs, int nthreads) {
    if (nthreads < 1) nthreads = 1;
#pragma omp parallel num_threads(nthreads)
    {
        int64_t* mark = (int64_t*)malloc((size_t)(n > 0 ? n : 1) * sizeof(int64_t));
        double* acc = (double*)malloc((size_t)(n > 0 ? n : 1) * sizeof(double));
        double* aacc = (double*)malloc((size_t)(n > 0 ? n : 1) * sizeof(double));
        for (int64_t j = 0; j < n; ++j) mark[j] = -1;
#pragma omp for schedule(dynamic, 256)
        for (int64_t i = 0; i < m; ++i) {
            int32_t* list = cci + crp[i];
            int64_t c = 0;
            for (int64_t p = arp[i]; p < arp[i + 1]; ++p) {
                int32_t k = aci[p];
                double a = av[p];
                for (int64_t q = brp[k]; q < brp[k + 1]; ++q) {
                    int32_t j = bci[q];
                    if (mark[j] != i) { mark[j] = i; acc[j] = 0.0; aacc[j] = 0.0; list[c++] = j; }
                    acc[j] += a * bv[q];
                    aacc[j] += fabs(a) * fabs(bv[q]);
                }
            }
            qsort(list, (size_t)c, sizeof(int32_t), cmp_i32);
            for (int64_t t = 0; t < c; ++t) {
                cv[crp[i] + t] = acc[list[t]];
                if (cabs) cabs[crp[i] + t] = aacc[list[t]];
            }
        }
        free(mark); free(acc); free(aacc);
    }
}

/* ------------------------------------------------------------------ O3 SpMV */

void oracle_spmv(int64_t m, const int64_t* rp, const int32_t* ci, const double* v, const double* x,
                 double* y, int nthreads) {
    if (nthreads < 1) nthreads = 1;
#pragma omp parallel for num_threads(nthreads) schedule(static)
    for (int64_t i = 0; i < m; ++i) {
        double s = 0.0;
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p) s += v[p] * x[ci[p]];
        y[i] = s;
    }
}

/* |A| |x| (for the per-entry error scale of reading R28). */
void oracle_spmv_abs(int64_t m, const int64_t* rp, const int32_t* ci, const double* v, const double* x,
                     double* y, int nthreads) {
    if (nthreads < 1) nthreads = 1;
#pragma omp parallel for num_threads(nthreads) schedule(static)
    for (int64_t i = 0; i < m; ++i) {
        double s = 0.0;
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p) s += fabs(v[p]) * fabs(x[ci[p]]);
        y[i] = s;
    }
}

/* ------------------------------------------------------------- O4 transpose */

/* A is m x n; out = A^T is n x m (out_rp[n+1]).  Counting sort: rows of A^T get
 * their entries in increasing original-row order, hence sorted columns. */
void oracle_transpose(int64_t m, int64_t n, const int64_t* rp, const int32_t* ci, const double* v,
                      int64_t* out_rp, int32_t* out_ci, double* out_v) {
    for (int64_t j = 0; j <= n; ++j) out_rp[j] = 0;
    for (int64_t p = 0; p < rp[m]; ++p) out_rp[ci[p] + 1]++;
    for (int64_t j = 0; j < n; ++j) out_rp[j + 1] += out_rp[j];
    int64_t* fill = (int64_t*)malloc((size_t)(n > 0 ? n : 1) * sizeof(int64_t));
    for (int64_t j = 0; j < n; ++j) fill[j] = out_rp[j];
    for (int64_t i = 0; i < m; ++i)
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
            int64_t d = fill[ci[p]]++;
            out_ci[d] = (int32_t)i;
            out_v[d] = v[p];
        }
    free(fill);
}

/* ------------------------------------------------------------ O2 CSR->mBSR */

/* Collect the sorted unique tile columns (col/4) of block row I into `buf`. */
static int64_t block_row_tiles(int64_t I, int64_t m, const int64_t* rp, const int32_t* ci, int32_t* buf) {
    int64_t c = 0;
    for (int64_t r = 4 * I; r < 4 * I + 4 && r < m; ++r)
        for (int64_t p = rp[r]; p < rp[r + 1]; ++p) buf[c++] = ci[p] / 4;
    qsort(buf, (size_t)c, sizeof(int32_t), cmp_i32);
    int64_t u = 0;
    for (int64_t t = 0; t < c; ++t)
        if (u == 0 || buf[u - 1] != buf[t]) buf[u++] = buf[t];
    return u;
}

/* blc_ptr[BR+1] filled; returns blc_num.  BR = ceil(m/4). */
int64_t oracle_csr_to_mbsr_count(int64_t m, const int64_t* rp, const int32_t* ci, int64_t* blc_ptr) {
    int64_t BR = (m + 3) / 4;
    int64_t maxrow = 0;
    for (int64_t I = 0; I < BR; ++I) {
        int64_t e = rp[(4 * I + 4 < m) ? 4 * I + 4 : m] - rp[4 * I];
        if (e > maxrow) maxrow = e;
    }
    int32_t* buf = (int32_t*)malloc((size_t)(maxrow > 0 ? maxrow : 1) * sizeof(int32_t));
    blc_ptr[0] = 0;
    for (int64_t I = 0; I < BR; ++I) blc_ptr[I + 1] = blc_ptr[I] + block_row_tiles(I, m, rp, ci, buf);
    free(buf);
    return blc_ptr[BR];
}

void oracle_csr_to_mbsr_fill(int64_t m, const int64_t* rp, const int32_t* ci, const double* v,
                             const int64_t* blc_ptr, int32_t* blc_idx, uint16_t* blc_map, double* blc_val) {
    int64_t BR = (m + 3) / 4;
    for (int64_t t = 0; t < blc_ptr[BR]; ++t) {
        blc_map[t] = 0;
        for (int b = 0; b < 16; ++b) blc_val[16 * t + b] = 0.0;
    }
    int64_t maxrow = 0;
    for (int64_t I = 0; I < BR; ++I) {
        int64_t e = rp[(4 * I + 4 < m) ? 4 * I + 4 : m] - rp[4 * I];
        if (e > maxrow) maxrow = e;
    }
    int32_t* buf = (int32_t*)malloc((size_t)(maxrow > 0 ? maxrow : 1) * sizeof(int32_t));
    for (int64_t I = 0; I < BR; ++I) {
        int64_t u = block_row_tiles(I, m, rp, ci, buf);
        int32_t* tiles = blc_idx + blc_ptr[I];
        for (int64_t t = 0; t < u; ++t) tiles[t] = buf[t];
        int64_t nt = blc_ptr[I + 1] - blc_ptr[I];
        for (int64_t r = 4 * I; r < 4 * I + 4 && r < m; ++r)
            for (int64_t p = rp[r]; p < rp[r + 1]; ++p) {
                int32_t J = ci[p] / 4;
                int64_t lo = 0, hi = nt - 1, t = -1;
                while (lo <= hi) {  /* binary search of J among the block row's tiles */
                    int64_t mid = (lo + hi) / 2;
                    if (tiles[mid] == J) { t = mid; break; }
                    if (tiles[mid] < J) lo = mid + 1; else hi = mid - 1;
                }
                int bit = 4 * (int)(r % 4) + (ci[p] % 4);
                int64_t g = blc_ptr[I] + t;
                blc_map[g] |= (uint16_t)(1u << bit);
                blc_val[16 * g + bit] = v[p];
            }
    }
    free(buf);
}

/* ------------------------------------------------------------ O7 mBSR->CSR */

int64_t oracle_mbsr_to_csr_count(int64_t m, const int64_t* blc_ptr, const uint16_t* blc_map, int64_t* rp) {
    rp[0] = 0;
    for (int64_t r = 0; r < m; ++r) {
        int64_t I = r / 4, c = 0;
        int rr = (int)(r % 4);
        for (int64_t t = blc_ptr[I]; t < blc_ptr[I + 1]; ++t)
            for (int cc = 0; cc < 4; ++cc) c += (blc_map[t] >> (4 * rr + cc)) & 1u;
        rp[r + 1] = rp[r] + c;
    }
    return rp[m];
}

void oracle_mbsr_to_csr_fill(int64_t m, const int64_t* blc_ptr, const int32_t* blc_idx, const uint16_t* blc_map,
                             const double* blc_val, const int64_t* rp, int32_t* ci, double* v) {
    for (int64_t r = 0; r < m; ++r) {
        int64_t I = r / 4, d = rp[r];
        int rr = (int)(r % 4);
        for (int64_t t = blc_ptr[I]; t < blc_ptr[I + 1]; ++t)
            for (int cc = 0; cc < 4; ++cc)
                if ((blc_map[t] >> (4 * rr + cc)) & 1u) {
                    ci[d] = 4 * blc_idx[t] + cc;
                    v[d] = blc_val[16 * t + 4 * rr + cc];
                    ++d;
                }
    }
}

/* -------------------------------------------------------------- O6 V-cycle */

/* Dense Cholesky A = L L^T in place (lower triangle), n x n row-major.  Returns 0 on
 * success, -1 if a pivot is not positive. */
int oracle_cholesky(int64_t n, double* a) {
    for (int64_t j = 0; j < n; ++j) {
        double s = a[j * n + j];
        for (int64_t k = 0; k < j; ++k) s -= a[j * n + k] * a[j * n + k];
        if (!(s > 0.0)) return -1;
        double d = sqrt(s);
        a[j * n + j] = d;
        for (int64_t i = j + 1; i < n; ++i) {
            double t = a[i * n + j];
            for (int64_t k = 0; k < j; ++k) t -= a[i * n + k] * a[j * n + k];
            a[i * n + j] = t / d;
        }
        for (int64_t i = 0; i < j; ++i) a[i * n + j] = 0.0;
    }
    return 0;
}

/* Solve L L^T x = b with the factor from oracle_cholesky. */
void oracle_cholesky_solve(int64_t n, const double* L, const double* b, double* x) {
    for (int64_t i = 0; i < n; ++i) {
        double s = b[i];
        for (int64_t k = 0; k < i; ++k) s -= L[i * n + k] * x[k];
        x[i] = s / L[i * n + i];
    }
    for (int64_t i = n - 1; i >= 0; --i) {
        double s = x[i];
        for (int64_t k = i + 1; k < n; ++k) s -= L[k * n + i] * x[k];
        x[i] = s / L[i * n + i];
    }
}

typedef struct {
    int64_t m, n;
    const int64_t* rp;
    const int32_t* ci;
    const double* v;
} ocsr;

static void spmv_counted(const ocsr* A, const double* x, double* y, int64_t* calls, int nt) {
    oracle_spmv(A->m, A->rp, A->ci, A->v, x, y, nt);
    ++*calls;
}

/* Alg. 2 (L68-82).  Level k = 0..nlev-1 (paper's k = 1..M).  A[k]: n_k x n_k;
 * P[k]: n_k x n_{k+1}; R[k]: n_{k+1} x n_k (k < nlev-1).  x is the initial guess
 * on entry and the result on exit.  res_norms[0] = ||b - A x0||, res_norms[c] after
 * cycle c.  Returns 0, or -1 if the coarsest Cholesky fails. */
int oracle_vcycle(int nlev, const int64_t* nrows,
                  const int64_t* const* Arp, const int32_t* const* Aci, const double* const* Av,
                  const int64_t* const* Prp, const int32_t* const* Pci, const double* const* Pv,
                  const int64_t* const* Rrp, const int32_t* const* Rci, const double* const* Rv,
                  double omega, int nu1, int nu2, const double* b, double* x, int ncycles,
                  double* res_norms, int64_t* spmv_calls, int nthreads, int smoother) {
    ocsr A[16], P[16], R[16];
    double *bk[16], *xk[16], *rk[16], *tk[16], *dinv[16];
    if (nlev < 1 || nlev > 16) return -2;
    for (int k = 0; k < nlev; ++k) {
        A[k] = (ocsr){nrows[k], nrows[k], Arp[k], Aci[k], Av[k]};
        if (k + 1 < nlev) {
            P[k] = (ocsr){nrows[k], nrows[k + 1], Prp[k], Pci[k], Pv[k]};
            R[k] = (ocsr){nrows[k + 1], nrows[k], Rrp[k], Rci[k], Rv[k]};
        }
        size_t sz = (size_t)(nrows[k] > 0 ? nrows[k] : 1) * sizeof(double);
        bk[k] = (double*)calloc(1, sz); xk[k] = (double*)calloc(1, sz);
        rk[k] = (double*)calloc(1, sz); tk[k] = (double*)calloc(1, sz);
        dinv[k] = (double*)calloc(1, sz);
        for (int64_t i = 0; i < nrows[k]; ++i) {
            double d = 0.0;
            if (smoother == 1) {   /* L1-Jacobi (L300): D_ii = sum_j |a_ij| (l1 row norm) */
                for (int64_t p = Arp[k][i]; p < Arp[k][i + 1]; ++p) d += fabs(Av[k][p]);
            } else {               /* weighted Jacobi (R21): D = diag(A_k) */
                for (int64_t p = Arp[k][i]; p < Arp[k][i + 1]; ++p)
                    if (Aci[k][p] == i) d = Av[k][p];
            }
            dinv[k][i] = 1.0 / d;
        }
    }
    int M = nlev - 1;
    int64_t nM = nrows[M];
    double* L = (double*)calloc((size_t)(nM * nM > 0 ? nM * nM : 1), sizeof(double));
    for (int64_t i = 0; i < nM; ++i)
        for (int64_t p = Arp[M][i]; p < Arp[M][i + 1]; ++p) L[i * nM + Aci[M][p]] = Av[M][p];
    int status = oracle_cholesky(nM, L);
    int64_t calls = 0;
    int64_t n0 = nrows[0];
    double* r0 = (double*)calloc((size_t)(n0 > 0 ? n0 : 1), sizeof(double));
    if (status == 0) {
        spmv_counted(&A[0], x, r0, &calls, nthreads);
        double s = 0.0;
        for (int64_t i = 0; i < n0; ++i) { double d = b[i] - r0[i]; s += d * d; }
        res_norms[0] = sqrt(s);
        for (int c = 1; c <= ncycles; ++c) {
            memcpy(bk[0], b, (size_t)n0 * sizeof(double));
            memcpy(xk[0], x, (size_t)n0 * sizeof(double));
            for (int k = 0; k < M; ++k) {             /* Alg. 2 lines 1-5 */
                int64_t nk = nrows[k];
                if (k > 0) memset(xk[k], 0, (size_t)nk * sizeof(double));
                for (int s1 = 0; s1 < nu1; ++s1) {   /* line 2: pre-smoothing */
                    spmv_counted(&A[k], xk[k], tk[k], &calls, nthreads);
                    for (int64_t i = 0; i < nk; ++i) xk[k][i] += omega * dinv[k][i] * (bk[k][i] - tk[k][i]);
                }
                spmv_counted(&A[k], xk[k], tk[k], &calls, nthreads);   /* line 3: residual */
                for (int64_t i = 0; i < nk; ++i) rk[k][i] = bk[k][i] - tk[k][i];
                spmv_counted(&R[k], rk[k], bk[k + 1], &calls, nthreads); /* line 4: restriction */
            }
            oracle_cholesky_solve(nM, L, bk[M], xk[M]);  /* line 6: coarsest level */
            for (int k = M - 1; k >= 0; --k) {        /* lines 7-11 */
                int64_t nk = nrows[k];
                spmv_counted(&P[k], xk[k + 1], tk[k], &calls, nthreads); /* line 8 */
                for (int64_t i = 0; i < nk; ++i) xk[k][i] += tk[k][i];     /* line 9 */
                for (int s2 = 0; s2 < nu2; ++s2) {   /* line 10: post-smoothing */
                    spmv_counted(&A[k], xk[k], tk[k], &calls, nthreads);
                    for (int64_t i = 0; i < nk; ++i) xk[k][i] += omega * dinv[k][i] * (bk[k][i] - tk[k][i]);
                }
            }
            memcpy(x, xk[0], (size_t)n0 * sizeof(double));
            spmv_counted(&A[0], x, r0, &calls, nthreads);   /* residual after the cycle (L308) */
            double s = 0.0;
            for (int64_t i = 0; i < n0; ++i) { double d = b[i] - r0[i]; s += d * d; }
            res_norms[c] = sqrt(s);
        }
    }
    if (spmv_calls) *spmv_calls = calls;
    free(r0); free(L);
    for (int k = 0; k < nlev; ++k) { free(bk[k]); free(xk[k]); free(rk[k]); free(tk[k]); free(dinv[k]); }
    return status;
}

/* ---------------------------------------------------------------- O8 strength filter
 * Pass 1 (count): kept entries per row -> rp_out[0..m] (exclusive prefix).  Pass 2 (fill):
 * the kept entries in column order; the diagonal value becomes a_ii + sum of the dropped
 * a_ij (ascending column order).  Returns -1 if a row with dropped entries has no diagonal
 * entry (nothing to lump into), else nnz of A_F. */
static int oracle_strong(double aij, double mi, double theta) { return mi > 0.0 && -aij >= theta * mi; }

int64_t oracle_strength_count(int64_t m, const int64_t* rp, const int32_t* ci, const double* v, double theta,
                              int64_t* rp_out) {
    rp_out[0] = 0;
    for (int64_t i = 0; i < m; ++i) {
        double mi = 0.0;
        int has_diag = 0, dropped = 0;
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p)
            if (ci[p] != i && -v[p] > mi) mi = -v[p];
        int64_t kept = 0;
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
            if (ci[p] == i) { has_diag = 1; ++kept; }
            else if (oracle_strong(v[p], mi, theta)) ++kept;
            else dropped = 1;
        }
        if (dropped && !has_diag) return -1;
        rp_out[i + 1] = rp_out[i] + kept;
    }
    return rp_out[m];
}

void oracle_strength_fill(int64_t m, const int64_t* rp, const int32_t* ci, const double* v, double theta,
                          const int64_t* rp_out, int32_t* ci_out, double* v_out) {
    for (int64_t i = 0; i < m; ++i) {
        double mi = 0.0;
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p)
            if (ci[p] != i && -v[p] > mi) mi = -v[p];
        double d = 0.0;
        int64_t dpos = -1, q = rp_out[i];
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
            if (ci[p] == i) { dpos = q; d = v[p]; ci_out[q] = ci[p]; v_out[q] = v[p]; ++q; }
            else if (oracle_strong(v[p], mi, theta)) { ci_out[q] = ci[p]; v_out[q] = v[p]; ++q; }
        }
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p)  /* lump the weak entries, column order */
            if (ci[p] != i && !oracle_strong(v[p], mi, theta)) d = d + v[p];
        if (dpos >= 0) v_out[dpos] = d;
    }
}

/* ---------------------------------------------------------------- O9 SA combine
 * In place on T = A_F Pt (CSR, columns sorted): T_ij <- Pt_ij - s_i * T_ij with
 * s_i = w / (A_F)_ii (0 when the diagonal is 0 or absent); Pt_ij = 0 where Pt has no entry.
 * Two roundings (product, difference). */
void oracle_sa_combine(int64_t m, const int64_t* trp, const int32_t* tci, double* tv, const int64_t* prp,
                       const int32_t* pci, const double* pv, const int64_t* arp, const int32_t* aci,
                       const double* av, double omega) {
    for (int64_t i = 0; i < m; ++i) {
        double d = 0.0;
        for (int64_t p = arp[i]; p < arp[i + 1]; ++p)
            if (aci[p] == i) d = av[p];
        const double si = d != 0.0 ? omega / d : 0.0;
        for (int64_t p = trp[i]; p < trp[i + 1]; ++p) {
            double pt = 0.0;
            for (int64_t q = prp[i]; q < prp[i + 1]; ++q)
                if (pci[q] == tci[p]) pt = pv[q];
            const double prod = si * tv[p];
            tv[p] = pt - prod;
        }
    }
}

/* ---------------------------------------------------------------- O10 PMIS aggregation
 * Coarsening (Alg. 1 line 3, L54; PMIS with str_thr and max_row_sum, L300, [71] L385; reading
 * R32 in DESIGN.md), written out step by step:
 *   1. strength: S_i = {j != i : -a_ij >= theta * max_{k!=i}(-a_ik)}, empty when that max is
 *      <= 0 or when |sum_j a_ij| > max_row_sum * |a_ii| (max_row_sum < 1);
 *   2. measure: lambda_i = |{j : i in S_j}| + w_i (w_i in [0, 1): the random numbers PMIS draws,
 *      an input);
 *   3. points that influence nobody (|{j : i in S_j}| = 0) are F; the rest undecided (U);
 *   4. rounds until no U: every U point whose lambda exceeds the lambda of every U point in
 *      S_i u S_i^T becomes C; then every U point with a new C point in S_i becomes F;
 *   5. aggregates: the C points in row order are aggregates 0..nC-1; (a) an F point with a C
 *      point in S_i joins the aggregate of the one with the largest lambda (ties: smaller
 *      index); (b) an F point still without one joins, among the points of S_i assigned in
 *      (a), the one with the largest lambda; (c) every point still unassigned is a new
 *      aggregate (row order).
 * state_out[i]: 1 = C, 0 = F; agg_out[i]; *rounds_out = PMIS rounds.  Returns the number of
 * aggregates.  Parity unpinned parts: none (hand-worked example + invariants, tests). */
enum { O_F = 0, O_C = 1, O_U = 2 };

static int oracle_row_strength_ok(int64_t i, const int64_t* rp, const int32_t* ci, const double* v,
                                  double max_row_sum, double* mi_out) {
    double mi = 0.0, rs = 0.0, d = 0.0;
    for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
        rs = rs + v[p];
        if (ci[p] == i) d = v[p];
        else if (-v[p] > mi) mi = -v[p];
    }
    *mi_out = mi;
    if (max_row_sum < 1.0 && fabs(rs) > max_row_sum * fabs(d)) return 0;
    return mi > 0.0;
}

/* 1 if j (!= i) is in S_i (row i's strong dependencies) */
static int oracle_in_S(int64_t i, int64_t p, const int32_t* ci, const double* v, double theta, double mi, int ok) {
    return ok && ci[p] != i && oracle_strong(v[p], mi, theta);
}

int64_t oracle_pmis_aggregate(int64_t n, const int64_t* rp, const int32_t* ci, const double* v, double theta,
                              double max_row_sum, const double* w, int8_t* state_out, int32_t* agg_out,
                              int* rounds_out) {
    double* mi = (double*)malloc((size_t)(n + 1) * sizeof(double));
    int* ok = (int*)malloc((size_t)(n + 1) * sizeof(int));
    int64_t* infl = (int64_t*)calloc((size_t)(n + 1), sizeof(int64_t));
    double* lam = (double*)malloc((size_t)(n + 1) * sizeof(double));
    int8_t* st = state_out;
    int8_t* newc = (int8_t*)calloc((size_t)(n + 1), 1);
    int8_t* cand = (int8_t*)calloc((size_t)(n + 1), 1);
    int32_t* aggA = (int32_t*)malloc((size_t)(n + 1) * sizeof(int32_t));
    /* 1-2: strength and measure */
    for (int64_t i = 0; i < n; ++i) ok[i] = oracle_row_strength_ok(i, rp, ci, v, max_row_sum, &mi[i]);
    for (int64_t i = 0; i < n; ++i)
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p)
            if (oracle_in_S(i, p, ci, v, theta, mi[i], ok[i])) infl[ci[p]] += 1;
    for (int64_t i = 0; i < n; ++i) {
        lam[i] = (double)infl[i] + w[i];
        st[i] = infl[i] == 0 ? O_F : O_U;  /* 3 */
    }
    /* 4: PMIS rounds */
    int rounds = 0;
    for (;;) {
        int64_t undecided = 0;
        for (int64_t i = 0; i < n; ++i) undecided += st[i] == O_U;
        if (!undecided) break;
        ++rounds;
        for (int64_t i = 0; i < n; ++i) cand[i] = st[i] == O_U;
        for (int64_t i = 0; i < n; ++i)  /* compare across every strong edge i -> j (S_i u S_i^T) */
            for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
                if (!oracle_in_S(i, p, ci, v, theta, mi[i], ok[i])) continue;
                const int64_t j = ci[p];
                if (st[i] != O_U || st[j] != O_U) continue;
                if (!(lam[i] > lam[j])) cand[i] = 0;
                if (!(lam[j] > lam[i])) cand[j] = 0;
            }
        for (int64_t i = 0; i < n; ++i) {
            newc[i] = cand[i];
            if (cand[i]) st[i] = O_C;
        }
        for (int64_t i = 0; i < n; ++i) {
            if (st[i] != O_U) continue;
            for (int64_t p = rp[i]; p < rp[i + 1]; ++p)
                if (oracle_in_S(i, p, ci, v, theta, mi[i], ok[i]) && newc[ci[p]]) {
                    st[i] = O_F;
                    break;
                }
        }
    }
    /* 5: aggregates */
    int32_t nagg = 0;
    for (int64_t i = 0; i < n; ++i) agg_out[i] = st[i] == O_C ? nagg++ : -1;
    for (int64_t i = 0; i < n; ++i) {  /* (a) */
        if (st[i] == O_C) continue;
        int64_t best = -1;
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
            if (!oracle_in_S(i, p, ci, v, theta, mi[i], ok[i])) continue;
            const int64_t j = ci[p];
            if (st[j] != O_C) continue;
            if (best < 0 || lam[j] > lam[best] || (lam[j] == lam[best] && j < best)) best = j;
        }
        if (best >= 0) agg_out[i] = agg_out[best];
    }
    for (int64_t i = 0; i < n; ++i) aggA[i] = agg_out[i];
    for (int64_t i = 0; i < n; ++i) {  /* (b): neighbours assigned in (a) */
        if (aggA[i] >= 0) continue;
        int64_t best = -1;
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
            if (!oracle_in_S(i, p, ci, v, theta, mi[i], ok[i])) continue;
            const int64_t j = ci[p];
            if (aggA[j] < 0 || st[j] == O_C) continue;
            if (best < 0 || lam[j] > lam[best] || (lam[j] == lam[best] && j < best)) best = j;
        }
        if (best >= 0) agg_out[i] = aggA[best];
    }
    for (int64_t i = 0; i < n; ++i)  /* (c) */
        if (agg_out[i] < 0) agg_out[i] = nagg++;
    for (int64_t i = 0; i < n; ++i) st[i] = st[i] == O_C ? 1 : 0;
    *rounds_out = rounds;
    free(mi); free(ok); free(infl); free(lam); free(newc); free(cand); free(aggA);
    return nagg;
}

/* The counter-based uniform generator of PMIS's random weights (both sides implement it):
 * z = seed + 0x9E3779B97F4A7C15 * (1 + i + 2^40 * level) (mod 2^64), splitmix64 finaliser,
 * u = (z >> 11) * 2^-53 in [0, 1). */
void oracle_pmis_weights(int64_t n, uint64_t seed, int level, double* w) {
    for (int64_t i = 0; i < n; ++i) {
        uint64_t z = seed + 0x9E3779B97F4A7C15ull * (1ull + (uint64_t)i + ((uint64_t)level << 40));
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        z = z ^ (z >> 31);
        w[i] = (double)(z >> 11) * (1.0 / 9007199254740992.0);
    }
}
