/*
 * amgt.h — C ABI of libamgt.so, the B200 (sm_100a) implementation of AmgT's hot path
 * (Lu et al., "AmgT: Algebraic Multigrid Solver on Tensor Cores", SC'24).
 * Citations "Lnnn" are /root/reference/PAPER.md line numbers; "Rnn" are the readings
 * of ambiguous passages listed in DESIGN.md.
 *
 * Conventions (all entry points):
 *   - Array pointers are DEVICE pointers unless the name ends in _host.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *     Calls are stream-ordered; only functions documented as "syncs" block the host.
 *   - Inputs are never modified.  No exception crosses the ABI: every call returns an
 *     amgt_status; amgt_last_error() gives a thread-local message for the last failure.
 *     On error, outputs are left unallocated (or freed) and the status is returned.
 *   - Memory the library returns in an amgt_mbsr is obtained from the caller's
 *     amgt_allocator (NULL allocator = cudaMallocAsync/cudaFreeAsync on `stream`) and is
 *     released with amgt_mbsr_free using the same allocator.
 *   - Indices: column indices int32, pointers/counters int64 (R26).
 *   - Determinism: structure is always identical for identical inputs; values are
 *     deterministic except where a function says otherwise.
 */
#ifndef AMGT_H
#define AMGT_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#pragma GCC visibility push(default)
#endif
#ifdef __cplusplus
extern "C" {
#endif

#define AMGT_VERSION_MAJOR 0
#define AMGT_VERSION_MINOR 1

typedef enum {
    AMGT_OK = 0,
    AMGT_ERR_ARG = 1,         /* bad argument: NULL, negative size, A.n != B.m, precision mismatch */
    AMGT_ERR_FORMAT = 2,      /* CSR input with unsorted/duplicate/out-of-range columns or bad row_ptr */
    AMGT_ERR_ALLOC = 3,       /* the allocator returned NULL */
    AMGT_ERR_CUDA = 4,        /* a CUDA runtime call or kernel launch failed */
    AMGT_ERR_NCCL = 5,        /* reserved for the distributed path */
    AMGT_ERR_RANGE = 6,       /* a value does not fit the target precision (FP16 overflow, R18) */
    AMGT_ERR_UNSUPPORTED = 7  /* valid request this build does not implement */
} amgt_status;

typedef enum { AMGT_FP64 = 0, AMGT_FP32 = 1, AMGT_FP16 = 2 } amgt_prec;

/* Stream-ordered allocator supplied by the caller (e.g. the torch caching allocator). */
typedef struct {
    void* (*alloc)(size_t bytes, void* stream, void* ctx);
    void (*free)(void* p, size_t bytes, void* stream, void* ctx);
    void* ctx;
} amgt_allocator;

/*
 * mBSR matrix (§IV.B; Fig. 3 caption L120).  A two-level structure:
 *   blc_ptr[blc_row+1]   offset of the first tile of each block row (int64, non-decreasing)
 *   blc_idx[blc_num]     tile column of each tile, strictly increasing within a block row
 *                        (the paper's blcIdx / BlcCid)
 *   blc_map[blc_num]     16-bit bitmap, one unsigned short per tile (L122): bit 4*r+c set
 *                        <=> entry (4I+r, 4J+c) structurally present (R1); never 0 (R5)
 *   blc_val[16*blc_num]  dense 4x4 values, row-major within a tile (index 4r+c), exactly
 *                        +0.0 where the bit is clear (R2); element type given by `prec`
 * Tiles are 4x4 because tensor-core shapes are multiples of 4 (L116).
 * blc_row = ceil(m/4), blc_col = ceil(n/4); bits outside m x n are never set (R25).
 * `own`, `aux` and `row_max` are library-managed (zero-initialise the struct before first use).
 */
typedef struct {
    int64_t m, n;
    int64_t blc_row, blc_col, blc_num;
    int64_t* blc_ptr;
    int32_t* blc_idx;
    uint16_t* blc_map;
    void* blc_val;
    amgt_prec prec;
    uint32_t own;      /* bit0: structure arrays owned, bit1: values owned */
    void* aux;         /* library-owned analysis (SpMV plan); NULL until amgt_spmv_analyze */
    int64_t row_max;   /* library-managed: max tiles in a block row when known (set by
                          amgt_spgemm_symbolic, kept by cast), 0 = unknown; lets the numeric
                          SpGEMM skip the kernels for row classes that do not occur */
} amgt_mbsr;

const char* amgt_last_error(void);
const char* amgt_version(void);

/*
 * CSR -> mBSR conversion (CSR2MBSR, L234, L262; Fig. 6 step 4).  For each block row I
 * the tile columns are the sorted union of col/4 over CSR rows 4I..4I+3; each entry
 * sets bit 4*(r%4)+(c%4) and stores its value at 16*t + bit; explicit zeros keep their
 * bit (R3).  Values are rounded once, directly from FP64, to `prec` (R18).
 *   row_ptr[m+1] int64, col_idx[nnz] int32 (sorted, unique per row, in [0, n)),
 *   val[nnz] float64.   out: filled, structure+values allocated with `al`.
 * Errors: AMGT_ERR_FORMAT for unsorted/duplicate/out-of-range columns or a row_ptr that
 * is not non-decreasing from 0 to nnz; AMGT_ERR_RANGE if prec = FP16 and |v| > 65504.
 * Syncs once (to size the tile arrays).
 */
amgt_status amgt_csr_to_mbsr(int64_t m, int64_t n, int64_t nnz, const int64_t* row_ptr, const int32_t* col_idx,
                             const double* val, amgt_prec prec, amgt_mbsr* out, const amgt_allocator* al,
                             void* stream);

/* Number of structural nonzeros (sum of popcounts of blc_map, P5).  Syncs. */
amgt_status amgt_mbsr_nnz(const amgt_mbsr* A, int64_t* nnz_host, void* stream);

/*
 * mBSR -> CSR (MBSR2CSR, L234, L262; Fig. 6 step 5).  Per scalar row, tiles in column
 * order, set bits of the row's nibble in column order.  Caller allocates row_ptr[m+1],
 * col_idx[nnz], val[nnz] (float64) with nnz from amgt_mbsr_nnz.  Values widen exactly.
 */
amgt_status amgt_mbsr_to_csr(const amgt_mbsr* A, int64_t* row_ptr, int32_t* col_idx, double* val, void* stream);

/*
 * Per-level precision cast (L266: "data precision conversions ... completed before
 * calling the kernels").  out shares in's structure arrays (not owned) and gets new
 * values of precision `to`, rounded to nearest even directly from the source (R18).
 * Errors: AMGT_ERR_RANGE if to = FP16 and a value overflows (detected on device; the
 * call then syncs to report it), AMGT_ERR_ARG if `to` is wider than in->prec.
 */
amgt_status amgt_mbsr_cast(const amgt_mbsr* in, amgt_prec to, amgt_mbsr* out, const amgt_allocator* al,
                           void* stream);

/* Release whatever A owns (structure, values, aux) and zero the struct. */
amgt_status amgt_mbsr_free(amgt_mbsr* A, const amgt_allocator* al, void* stream);

/*
 * Tile-level transpose out = in^T (R = P^T of Alg. 1 line 4, L54): tile (I,J) becomes
 * (J,I) with its 4x4 values and bitmap transposed; block rows of out sorted by column.
 * Same precision as in.  Syncs once (to size nothing — tile count is unchanged — but to
 * read back a format flag).
 */
amgt_status amgt_mbsr_transpose(const amgt_mbsr* in, amgt_mbsr* out, const amgt_allocator* al, void* stream);

/* Build an mBSR from device arrays the caller owns (no copy; own = 0). */
amgt_status amgt_mbsr_wrap(int64_t m, int64_t n, int64_t blc_num, int64_t* blc_ptr, int32_t* blc_idx,
                           uint16_t* blc_map, void* blc_val, amgt_prec prec, amgt_mbsr* out);

/* ------------------------------------------------------------------ SpGEMM (§IV.C) */

typedef struct {
    int64_t bin_rows[8];     /* block rows of C per bin (L151; edges 128*2^b, R7)          */
    int64_t cub_total;       /* sum over rows of Cub_per_row (intermediate tile products)  */
    int64_t pairs_nonzero;   /* tile pairs with BITMAPMULTIPLY(mapA, mapB) != 0 (L165)     */
    int64_t pairs_tc;        /* of those, pairs whose A tile takes the tensor-core route   */
    int64_t scalar_products; /* sum over nonzero pairs of scalar multiply-adds (FLOP = 2x)  */
    int64_t numeric_rows[3]; /* C block rows per numeric path (warp/smem, warp/global, empty) */
} amgt_spgemm_info;

/*
 * Symbolic SpGEMM C = A*B (§IV.C.1-2; Alg. 3).  Data analysis
 * (Cub_per_row), binning into 8 bins (<128, [128,256), ..., >=8192), two-step hash
 * symbolic (step 1 counts distinct C tiles with BITMAPMULTIPLY != 0, prefix sum to
 * blc_ptrC, allocation, step 2 re-inserts, compresses and sorts -> blc_idxC) and, in
 * this build, the OR of BITMAPMULTIPLY results into blc_mapC (R15).
 * A, B: same precision, A.n == B.m.  C: output; structure allocated and filled, values
 * allocated (not computed).  info may be NULL.  Syncs once (the C tile count, L153) — twice when
 * some block row has more than 32 candidate tiles (its bin kernels count before the allocation)
 * — plus once more if info != NULL.
 * Numeric plan (R34): for the block rows of C with more than 32 tiles, step 2 also keeps
 * one 16-B record per (A tile, B tile) pair (C tile, B tile, A tile, bitmap product) and a
 * "several products" bit per C tile in library-owned device memory keyed by C's blc_idx; the
 * numeric call then streams them instead of searching C's rows.  The plan depends on the
 * structure only (values of A, B may change between numeric calls), is freed with C's structure
 * (amgt_mbsr_free) and at most 4 plans / 2 GB are cached (least recently built dropped).
 * AMGT_SPGEMM_PLAN=0 disables it.
 */
amgt_status amgt_spgemm_symbolic(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* C, amgt_spgemm_info* info,
                                 const amgt_allocator* al, void* stream);

/*
 * Numeric SpGEMM (§IV.C.3; Alg. 4).  One warp per C block row.
 * Per A tile: POPCOUNT(mapA) >= tc_threshold -> warp-level tensor-core route (FP64:
 * DMMA m8n8k4 with fragA = [A;A], fragB = [B_j | B_j'], keeping the two diagonal 4x4
 * quadrants, L157-171; FP16: HMMA m16n8k16 with FP32 accumulation, 8 tile products per
 * instruction); otherwise the thread-level CUDA-core route.  FP32 always takes the
 * CUDA-core route (no TF32, R17).  C must come from amgt_spgemm_symbolic(A, B) (same A and B
 * structure arrays; the symbolic phase's numeric plan is used when present, see above).
 * Values: deterministic for C block rows with at most 32 tiles (fixed lane order); longer rows
 * accumulate tiles that receive three or more products with FP atomics and are reproducible up
 * to rounding only (exact on integer / dyadic data) — unless AMGT_SPGEMM_DET=1:
 * then the symbolic phase gives every multi-product tile of its plan a slot range and the numeric
 * phase adds the tile's products in ascending A-tile order (bitwise reproducible; two more host
 * syncs in the symbolic phase).
 */
amgt_status amgt_spgemm_numeric(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* C, void* stream);

/* Tensor-core routing threshold on POPCOUNT(mapA) (paper: 10, L157).  17 disables the
 * tensor-core route, 0 forces it.  Applies to SpGEMM numeric and SpMV. Process-global.
 * Default 17 for both: measured on B200 the mma routes never beat the CUDA-core routes for
 * these memory-bound kernels (R9/R10); (10, 10) gives the paper's routing. */
amgt_status amgt_set_tc_threshold(int spgemm_threshold, int spmv_threshold);

/* Galerkin product Ac = R*(A*P) via two SpGEMM calls (Alg. 1 line 5, L54; R20). */
amgt_status amgt_rap(const amgt_mbsr* R, const amgt_mbsr* A, const amgt_mbsr* P, amgt_mbsr* Ac,
                     const amgt_allocator* al, void* stream);

/* -------------------------------------------------------------------- SpMV (§IV.D) */

/*
 * Optional SpMV preprocessing (L220 "data preprocessing"): computes avg_nnz_blc, the
 * variation (coefficient of variation of tiles per block row, R11) and the
 * load-balancing work list (block rows longer than 64 tiles are split into chunks of
 * WARP_CAPACITY = 64 tiles, Alg. 5, R12).  Stored in A->aux (freed by amgt_mbsr_free).
 * Without it amgt_spmv still works (no row splitting).  Syncs once — except when A->row_max
 * is known (set by conversion, SpGEMM symbolic, transpose inside amgt_hierarchy_create;
 * kept by cast) and <= 64: then nothing needs splitting, the call launches nothing and
 * returns at once, and the statistics below are computed (one sync on the legacy default
 * stream) by the first amgt_spmv_get_stats.
 */
amgt_status amgt_spmv_analyze(amgt_mbsr* A, const amgt_allocator* al, void* stream);

typedef struct {
    double avg_nnz_blc;      /* nnz / blc_num (L220)                          */
    double variation;        /* CV of tiles per block row (R11)               */
    int64_t long_rows;       /* block rows split over several warps           */
    int64_t chunks;          /* warp work items for the long rows             */
    int64_t tc_tiles;        /* tiles with popcount >= the SpMV TC threshold  */
} amgt_spmv_stats;
amgt_status amgt_spmv_get_stats(const amgt_mbsr* A, amgt_spmv_stats* st_host);

/*
 * y = A*x (§IV.D; Alg. 5).  x has 4*blc_col elements and y has
 * 4*blc_row elements (zero padding beyond n / m is read as zero / written as zero).
 * x and y precisions FP64 or FP32 independently of A's (FP64/FP32/FP16).  Arithmetic:
 * FP64 when A is FP64, else FP32 (FP16 values widened in registers).  Tiles with
 * popcount >= the SpMV TC threshold go through DMMA (FP64) two tiles per instruction,
 * y taken from the diagonal blocks of fragY (L222-228, R14); others use CUDA cores with
 * 4 lanes per tile, one tile row per lane (L230).  Values: deterministic.
 */
amgt_status amgt_spmv(const amgt_mbsr* A, const void* x, amgt_prec xprec, void* y, amgt_prec yprec,
                      void* stream);

/*
 * SpMV with a fused Alg. 2 vector epilogue (NEXT-1 of SURVEY §8(f)), element-wise on
 * t = (A x)_i, in y's precision:
 *   AMGT_EPI_Y        y = t
 *   AMGT_EPI_JACOBI   y = x + omega * dinv .* (b - t)   (weighted Jacobi sweep, Alg. 2 lines 2/10,
 *                                                       out of place: y != x, A square)
 *   AMGT_EPI_RESIDUAL y = b - t                          (Alg. 2 line 3)
 *   AMGT_EPI_ACCUM    y = y + t                          (interpolation + correction, lines 8-9)
 * b and dinv have y's precision and length 4*blc_row.
 */
#define AMGT_EPI_Y 0
#define AMGT_EPI_JACOBI 1
#define AMGT_EPI_RESIDUAL 2
#define AMGT_EPI_ACCUM 3
amgt_status amgt_spmv_fused(const amgt_mbsr* A, const void* x, amgt_prec xprec, void* y, amgt_prec yprec, int mode,
                            const void* b, const void* dinv, double omega, void* stream);

/* Weighted Jacobi sweep that also returns the residual of its input (NEXT-1 fusion):
 *   r = b - A x,   y = x + omega * dinv .* r        (one pass over A)
 * After a V-cycle, r is the Alg. 2 residual reported per cycle (L308), so the first
 * pre-smoothing sweep of the next cycle delivers it without a separate SpMV.  x, y, r, b,
 * dinv share one precision (FP64 or FP32), length 4*blc_row; x, y, r distinct; A square.
 * Mode value AMGT_EPI_JACOBI_RES is internal to this call (not accepted by amgt_spmv_fused). */
#define AMGT_EPI_JACOBI_RES 4
amgt_status amgt_spmv_fused_r(const amgt_mbsr* A, const void* x, amgt_prec xprec, void* y, amgt_prec yprec,
                              const void* b, const void* dinv, double omega, void* r, void* stream);

/* Row-range variant used by the distributed SpMV to overlap the halo exchange: only
 * block rows [blk_begin, blk_end) are computed; y indexed by local row; for Jacobi, x_i is
 * read from xs (the own segment of x when x is an extended [halo|own|halo] buffer).
 * Not available for matrices whose SpMV plan splits long rows (AMGT_ERR_UNSUPPORTED). */
amgt_status amgt_spmv_fused_range(const amgt_mbsr* A, int64_t blk_begin, int64_t blk_end, const void* x,
                                  amgt_prec xprec, void* y, amgt_prec yprec, int mode, const void* b, const void* dinv,
                                  const void* xs, double omega, void* stream);

/*
 * Consecutive Alg. 2 steps on one square FP64 operator in one pass over HBM (§8(f) NEXT-1).
 * Stage s computes t = A x_s and, element-wise in FP64:
 *   AMGT_SWEEP_J   y_s = x_s + omega * dinv .* (b - t)          (Jacobi sweep, Alg. 2 lines 2/10)
 *   AMGT_SWEEP_JR  as J; also ||b - t||^2 -> *norm_dev            (the residual of the sweep's
 *                  input: after a V-cycle the L308 residual of that cycle)
 *   AMGT_SWEEP_R   y_s = b - t                                   (Alg. 2 line 3)
 *   AMGT_SWEEP_RN  as R; also ||y_s||^2 -> *norm_dev
 * Stage s > 0 reads x_s = y_{s-1}; outputs are distinct from every vector an earlier stage
 * reads or writes; at most one norm stage; 1..AMGT_SWEEP_MAX_STAGES stages.  Vectors: FP64,
 * length 4*blc_row, b and dinv shared by all stages.  Each y_s is bit-identical to the
 * amgt_spmv_fused / amgt_spmv_fused_r result of the same step (same per-row arithmetic);
 * the norm is a deterministic sum in a different fixed order.  One kernel: stages run as a
 * wavefront over 64-block-row chunks with acquire/release flags, lagged so the tiles a later
 * stage re-reads are still in L2 (A read from HBM about once).  The plan (column-chunk
 * ranges, flags, lag) belongs to one operator; calls on one plan must be stream-ordered.
 * amgt_sweep_plan_create: no sync.  Errors: AMGT_ERR_UNSUPPORTED (not FP64), AMGT_ERR_ARG.
 */
#define AMGT_SWEEP_J 1
#define AMGT_SWEEP_JR 2
#define AMGT_SWEEP_R 3
#define AMGT_SWEEP_RN 4
#define AMGT_SWEEP_MAX_STAGES 4
typedef struct {
    int mode;
    const void* x;
    void* y;
} amgt_sweep_stage;
typedef struct amgt_sweep_plan amgt_sweep_plan;
amgt_status amgt_sweep_plan_create(const amgt_mbsr* A, const amgt_allocator* al, void* stream, amgt_sweep_plan** out);
amgt_status amgt_sweep_plan_destroy(amgt_sweep_plan* P, void* stream);
/* Diagnostics (zero unless libamgt was built with -DSW_STATS=1): summed SM cycles and counts of
 * stage-0 items, of later-stage items, cycles spent waiting, unready polls; reset on read. Syncs. */
amgt_status amgt_sweep_plan_stats(amgt_sweep_plan* P, uint64_t* out6_host, void* stream);
amgt_status amgt_spmv_sweeps(amgt_sweep_plan* P, const amgt_mbsr* A, int nstages, const amgt_sweep_stage* st,
                             const void* b, const void* dinv, double omega, double* norm_dev, void* stream);

/*
 * Interpolation through one SpGEMM call (Alg. 1 line 4, L54; [35] L385; §8(f) NEXT-2; reading
 * R31 in DESIGN.md: smoothed aggregation).
 * amgt_strength_filter: A_F = A without its weak off-diagonal entries — a_ij (i != j) is strong
 *   iff the row has a negative off-diagonal and -a_ij >= theta * max_{k != i}(-a_ik) (classical
 *   strength, str_thr = theta, L300) — each weak entry removed from the structure (tiles left
 *   empty disappear) and added to the diagonal in ascending column order (row sums kept).
 *   s_out[4*blc_row] = omega / (A_F)_ii (0 where that is 0); FP64 for FP64 operators, FP32
 *   otherwise.  A square, any precision (FP32/FP16 arithmetic in FP32).  AF allocated with al.
 *   Errors: AMGT_ERR_ARG if a row with weak entries has no diagonal entry.  Syncs once.
 * amgt_sa_interp: P = (I - omega D_F^-1 A_F) Pt: A_F as above, T = A_F Pt by the mBSR SpGEMM
 *   (amgt_spgemm_symbolic/numeric), then P_ij = Pt_ij - s_i T_ij (two roundings) on T's
 *   structure, which contains Pt's wherever A_F has its diagonal; cancelled entries stay
 *   (R3).  Pt (the tentative interpolation, e.g. fixed aggregation, R19) has A's precision.
 *   P allocated with al.  Syncs (filter + symbolic).
 */
amgt_status amgt_strength_filter(const amgt_mbsr* A, double theta, double omega, amgt_mbsr* AF, void* s_out,
                                 const amgt_allocator* al, void* stream);
amgt_status amgt_sa_interp(const amgt_mbsr* A, const amgt_mbsr* Pt, double theta, double omega, amgt_mbsr* P,
                           const amgt_allocator* al, void* stream);

/* ------------------------------------------------ distributed-path helpers (§8(e)) */

/* CSR -> mBSR with column offset: column c becomes c - col_offset, which must lie in
 * [0, n) (a rank's rows with global columns, remapped to its extended range). */
amgt_status amgt_csr_to_mbsr_ex(int64_t m, int64_t n, int64_t nnz, const int64_t* row_ptr, const int32_t* col_idx,
                                const double* val, int64_t col_offset, amgt_prec prec, amgt_mbsr* out,
                                const amgt_allocator* al, void* stream);
/* In place: blc_idx += delta_tiles; A->n = new_n (remap global -> extended-local columns). */
amgt_status amgt_mbsr_shift_cols(amgt_mbsr* A, int64_t delta_tiles, int64_t new_n, void* stream);
/* out3_host = {min column, max column, max |column - (row + row_offset)|} (syncs).  CSR: scalar
 * units; mBSR: tile units with block-row offset. */
amgt_status amgt_csr_col_range(int64_t m, const int64_t* row_ptr, const int32_t* col_idx, int64_t row_offset,
                               int64_t* out3_host, void* stream);
amgt_status amgt_mbsr_col_range(const amgt_mbsr* A, int64_t blk_row_offset, int64_t* out3_host, void* stream);
/* dinv[i] = 1 / A(i, i) with the diagonal tile of block row I at column I + diag_tile_offset. */
amgt_status amgt_dinv(const amgt_mbsr* A, int64_t diag_tile_offset, void* dinv, amgt_prec vprec, void* stream);
/* Host: inverse of an SPD n x n row-major matrix via Cholesky (coarsest level, R22). */
amgt_status amgt_dense_spd_inverse(int64_t n, const double* a_host, double* inv_host);
/* x[0:npad] = Ainv (n x n, FP64, device) * b[0:n], zero-padded to npad. */
amgt_status amgt_dense_matvec(int64_t n, int64_t npad, const double* Ainv, const void* b, void* x, amgt_prec vprec,
                              void* stream);
/* *out_dev = sum r_i^2 (deterministic two-pass reduction, FP64). */
amgt_status amgt_norm2sq(int64_t n, const double* r, double* out_dev, void* stream);

/* ------------------------------------------------------ hierarchy + V-cycle (§II) */

typedef struct {
    int max_levels;          /* <= 8 (paper: <= 7, L302) */
    int nu1, nu2;            /* pre/post smoothing sweeps (paper num_sweep = 1, L300) */
    double omega;            /* Jacobi weight (R21; default 2/3) */
    amgt_prec level_prec[8]; /* matrix precision per level (L266: FP64, FP32, FP16...) */
    int smoother;            /* AMGT_SMOOTH_JACOBI (default): D = diag(A_k), x += omega D^-1 (b - A x);
                                AMGT_SMOOTH_L1_JACOBI: D_ii = sum_j |a_ij| (the l1 row norm; the
                                paper's L1_Jacobi, L300, NEXT-3), same sweep — omega = 1 is HYPRE's */
    int interp;              /* AMGT_INTERP_GIVEN (0, default): P[k] is the interpolation itself;
                                AMGT_INTERP_SA (1): P[k] is the tentative interpolation and the level
                                builds P_k = amgt_sa_interp(A_k, P[k], theta, omega_p) in level-k
                                precision — three SpGEMM calls per level (L54, L302; NEXT-2) */
    double theta;            /* strength threshold for AMGT_INTERP_SA (paper str_thr 0.25, L300) */
    double omega_p;          /* prolongation smoothing weight for AMGT_INTERP_SA / _PMIS (default 2/3) */
    /* AMGT_INTERP_PMIS (2): no P is given; every level is coarsened on the device — PMIS C/F
       splitting of the strength graph (str_thr = theta, max_row_sum; L300) with aggregates
       around the C points (amgt_pmis_aggregate, reading R32) — and P_k is the smoothed
       aggregation amgt_sa_interp(A_k, Pt_k) (one SpGEMM, L54).  The hierarchy stops at
       nlev levels, at the first level with at most max_coarse_size rows (L300: 3), or when
       the coarsening stalls; amgt_hierarchy_nlev gives the number built. */
    int max_coarse_size;     /* 0: no size criterion */
    double max_row_sum;      /* PMIS strength: rows with |sum_j a_ij| > max_row_sum |a_ii| have no strong
                                dependencies (L300: 0.8); >= 1 or <= 0 disables */
    uint64_t seed;           /* PMIS random weights: the counter-based generator of R32 (seed, level) */
} amgt_vcycle_opts;
#define AMGT_INTERP_GIVEN 0
#define AMGT_INTERP_SA 1
#define AMGT_INTERP_PMIS 2
#define AMGT_SMOOTH_JACOBI 0
#define AMGT_SMOOTH_L1_JACOBI 1

typedef struct amgt_hierarchy amgt_hierarchy;

/*
 * Setup (Alg. 1, L52-58) with fixed interpolation: A (FP64 mBSR, level 1) and P[k]
 * (FP64 mBSR, n_k x n_{k+1}), k = 0..nlev-2.  For each level: R_k = P_k^T is built on
 * the device, A_{k+1} = R_k A_k P_k (two SpGEMM calls, run in level k's precision),
 * then cast to level k+1's precision (L266).  The coarsest level is converted back to
 * CSR (MBSR2CSR, L262) and factorised (dense Cholesky, FP64, R22).  Syncs.
 */
amgt_status amgt_hierarchy_create(const amgt_mbsr* A, const amgt_mbsr* const* P, int nlev,
                                  const amgt_vcycle_opts* o, const amgt_allocator* al, void* stream,
                                  amgt_hierarchy** H);

/* Level-k operators (borrowed pointers valid until destroy); k = 0 .. nlev-1. */
amgt_status amgt_hierarchy_level(const amgt_hierarchy* H, int k, const amgt_mbsr** A, const amgt_mbsr** P,
                                 const amgt_mbsr** R);
int amgt_hierarchy_nlev(const amgt_hierarchy* H);

/*
 * Solve phase (Alg. 2, L68-82): ncycles V-cycles on A x = b, weighted Jacobi smoothing,
 * direct coarsest solve; after each cycle the level-1 residual and its 2-norm (L308).
 * b, x: FP64 device vectors of length 4*blc_row(A_1); x = initial guess in, result out.
 * res_norms_host[ncycles+1] (||b - A x0|| first) and *spmv_calls_host (may be NULL).
 * Syncs once at the end (norms are accumulated on the device).
 */
amgt_status amgt_vcycle(amgt_hierarchy* H, const double* b, double* x, int ncycles, double* res_norms_host,
                        int64_t* spmv_calls_host, void* stream);

/*
 * Preconditioned conjugate gradient on A_1 x = b with one V-cycle (Alg. 2 from a zero
 * guess, no residual norms) as the preconditioner M — the solve-phase consumer named at
 * L92 (NEXT-1).  Textbook recurrence: r0 = b - A x0, z = M r, p = z; per iteration
 * q = A p, alpha = (r,z)/(p,q), x += alpha p, r -= alpha q, z = M r,
 * beta = (r,z)_new/(r,z)_old, p = z + beta p (alpha, beta = 0 when a denominator is 0).
 * The V-cycle is symmetric when nu1 = nu2 (Jacobi before and after), so M is SPD for SPD
 * A in exact arithmetic.  Runs maxit iterations, or stops early once ||r_k|| <= rtol ||r_0||
 * when rtol > 0 (one host round trip per iteration for the test; rtol = 0: no sync until
 * the end).  res_norms_host[maxit+1]: ||r_k||_2 for k = 0..*iters_host; *spmv_calls_host
 * counts every SpMV (1 + per iteration 1 + a V-cycle's).  b, x: FP64, 4*blc_row(A_1);
 * the level-1 vector precision must be FP64 (AMGT_ERR_UNSUPPORTED otherwise).
 */
amgt_status amgt_pcg(amgt_hierarchy* H, const double* b, double* x, int maxit, double rtol, double* res_norms_host,
                     int* iters_host, int64_t* spmv_calls_host, void* stream);

amgt_status amgt_hierarchy_destroy(amgt_hierarchy* H);

/* ------------------------------------------------------- coarsening (§8(f) NEXT-2) */
/*
 * PMIS coarsening with aggregation (Alg. 1 line 3, L54; the paper's PMIS, str_thr, max_row_sum,
 * L300; [71] L385; reading R32 in DESIGN.md).  A square, any precision (strength decisions in FP64
 * of the stored values):
 *   S_i = {j != i : -a_ij >= theta max_{k!=i}(-a_ik)}, empty when that max <= 0 or when
 *         |sum_j a_ij| > max_row_sum |a_ii| (max_row_sum < 1);
 *   lambda_i = |{j : i in S_j}| + w_i, w_i = weights[i] (device, m) or, when weights is NULL, the
 *         counter-based generator u(seed, level, i) of R32;
 *   PMIS rounds: points influencing nobody are F; every undecided point beating every undecided
 *         neighbour in S u S^T becomes C, then undecided points with a new C point in S_i become F;
 *   aggregates: C points in row order; F points join their strongest (largest lambda) C point in
 *         S_i, then the points of S_i assigned that way; the rest are singletons.
 * agg[m] (device): aggregate of each row; is_c[m] (device, nullable): 1 for C points;
 * *n_agg_host; *rounds_host (nullable): PMIS rounds.  Deterministic.  Syncs once per round.
 */
amgt_status amgt_pmis_aggregate(const amgt_mbsr* A, double theta, double max_row_sum, const double* weights,
                                uint64_t seed, int level, int32_t* agg, int8_t* is_c, int64_t* n_agg_host,
                                int* rounds_host, void* stream);
/* The tentative interpolation of an aggregation: Pt (m x n_agg, precision prec) with Pt(i, agg_i) = 1. */
amgt_status amgt_aggregation_p(int64_t m, int64_t n_agg, const int32_t* agg, amgt_prec prec, amgt_mbsr* Pt,
                               const amgt_allocator* al, void* stream);

/* ------------------------------------------------------ distributed path (§8(e)) */
/*
 * Row partition (the paper's 8-GPU runs, L363-365): rank r owns a contiguous range
 * of rows of every distributed matrix, ranks in ascending order; every range except the last
 * covers whole 4-row block rows (rows % 4 == 0).  A rank's matrices hold ITS rows with GLOBAL
 * column indices (m = own rows, n = global columns); its vectors hold its own rows, padded to
 * 4*ceil(m/4) elements.  The library derives the rest: the contiguous block-row range a rank's
 * columns touch (its halo), which pieces other ranks own, which of its own rows they need — from
 * one host all-gather of (rows, min tile column, max tile column) per rank.
 * All calls below except amgt_dist_plan_host are COLLECTIVE: every rank calls them in the same
 * order.  Transfers are stream-ordered on the call's stream (halo exchanges on an internal
 * communication stream, joined with events).
 */
typedef struct amgt_dist amgt_dist;

/* NCCL transport (one process per GPU).  amgt_nccl_unique_id on one rank, broadcast the 128
 * bytes, then amgt_dist_create on every rank with its level-1 row range [row_begin, row_end).
 * libnccl.so.2 is loaded at run time (AMGT_ERR_NCCL if absent). */
amgt_status amgt_nccl_unique_id(void* id128_host);
amgt_status amgt_dist_create(const void* id128_host, int rank, int size, int64_t row_begin, int64_t row_end,
                             amgt_dist** D);

/* Loopback transport: `size` (<= 16) virtual ranks in ONE process on ONE GPU, each driven by its
 * own host thread with its own stream.  Point-to-point messages are device-to-device copies
 * ordered by CUDA events; all-reduce sums the ranks' buffers in rank order (deterministic, the
 * same bits on every rank).  Same semantics as the NCCL transport — it runs the multi-rank code
 * paths on a single GPU.  A mismatched call sequence fails with AMGT_ERR_NCCL after 300 s. */
typedef struct amgt_dist_group amgt_dist_group;
amgt_status amgt_dist_group_create(int size, amgt_dist_group** G);
amgt_status amgt_dist_group_destroy(amgt_dist_group* G);  /* after every member's amgt_dist_destroy */
/* A member failed outside the library: every call waiting on the group returns AMGT_ERR_NCCL. */
amgt_status amgt_dist_group_abort(amgt_dist_group* G);
amgt_status amgt_dist_create_loopback(amgt_dist_group* G, int rank, int64_t row_begin, int64_t row_end,
                                      amgt_dist** D);
amgt_status amgt_dist_destroy(amgt_dist* D);

/* In-place sum over ranks of count doubles (device buffer). */
amgt_status amgt_dist_allreduce_sum(amgt_dist* D, double* buf, int64_t count, void* stream);

/*
 * y_local = (A x)_own rows (§IV.D SpMV, L218-230, over a row partition).  A_local: own rows, global
 * columns (square A; any precision).  x_local/y_local: own rows, FP64 for an FP64 matrix, else
 * FP32 (R16).  The halo of x is exchanged (one point-to-point group on the communication stream)
 * while the interior block rows (rows whose columns are all owned) run; the boundary rows follow.
 * The first call for a matrix builds its plan (syncs; a shifted column array + an extended x
 * buffer, cached in D and keyed by A's arrays — A must stay alive and unchanged while D uses it;
 * freed by amgt_dist_destroy).  Values equal amgt_spmv's on the assembled matrix bit for bit.
 */
amgt_status amgt_dist_spmv(amgt_dist* D, const amgt_mbsr* A_local, const void* x_local, void* y_local, void* stream);

/*
 * Ac_l = own rows of R (A P) (Alg. 1 line 5, L54; R20) over a row partition: R_l = own COARSE
 * rows of R (global fine columns), A_l = own fine rows of A (global columns), P_l = own fine rows
 * of P (global coarse columns); one precision.  The rows of P that A_l's columns reach are
 * gathered from their owners (row lengths, then tiles: one host sync), AP_l = A_l P_ext locally;
 * the rows of AP that R_l's columns reach likewise (none when aggregates are rank-local); then
 * Ac_l = R_l AP_ext.  Ac_l: own coarse rows, global coarse columns, allocated with al.  The
 * structure equals the corresponding rows of the single-GPU R (A P) bit for bit.
 */
amgt_status amgt_dist_rap(amgt_dist* D, const amgt_mbsr* R_l, const amgt_mbsr* A_l, const amgt_mbsr* P_l,
                          amgt_mbsr* Ac_l, const amgt_allocator* al, void* stream);

/* M_full = every rank's rows of a row-partitioned matrix, in rank order (agglomeration). */
amgt_status amgt_dist_allgather_mbsr(amgt_dist* D, const amgt_mbsr* M_local, amgt_mbsr* M_full,
                                     const amgt_allocator* al, void* stream);

/*
 * Distributed hierarchy (Alg. 1 with fixed interpolation, L52-58) and V-cycle (Alg. 2, L68-82).
 *   A_l: own rows of A_1 (FP64, global columns, rows [row_begin, row_end) of amgt_dist_create).
 *   P_l[k]: own fine rows of P_k (FP64, global coarse columns); a rank's coarse rows are the
 *   columns its P rows reach, which must form contiguous ranges in rank order (aggregates never
 *   straddle ranks — true for the z-slab partition; else AMGT_ERR_UNSUPPORTED).
 * Levels whose global row count is at most agg_rows (from level 2 on; the coarsest always) are
 * AGGLOMERATED: their operators are all-gathered at setup and the single-GPU V-cycle machinery
 * runs on them redundantly on every rank (one all-gather of the right-hand side per cycle instead
 * of a halo exchange per coarse-level SpMV).  With one rank the whole hierarchy is the
 * single-GPU one.  o: as amgt_hierarchy_create (level 1 FP64, interp = AMGT_INTERP_GIVEN).
 * A_l and P_l are borrowed (keep them alive until amgt_dist_hierarchy_destroy).  Syncs.
 */
typedef struct amgt_dist_hierarchy amgt_dist_hierarchy;
amgt_status amgt_dist_hierarchy_create(amgt_dist* D, const amgt_mbsr* A_l, const amgt_mbsr* const* P_l, int nlev,
                                       const amgt_vcycle_opts* o, int64_t agg_rows, const amgt_allocator* al,
                                       void* stream, amgt_dist_hierarchy** H);
/* ncycles V-cycles; b_local, x_local: own rows of level 1 (FP64, 4*ceil(m/4) elements).
 * res_norms_host[ncycles+1]: global ||b - A x|| (all-reduced); *spmv_calls_host: this rank's
 * SpMV operations of Alg. 2 (the same count on every rank and as amgt_vcycle).  Syncs at the end. */
amgt_status amgt_dist_vcycle(amgt_dist_hierarchy* H, const double* b_local, double* x_local, int ncycles,
                             double* res_norms_host, int64_t* spmv_calls_host, void* stream);
typedef struct {
    int nlev, agg_level;         /* levels [0, agg_level) distributed, the rest agglomerated */
    int64_t rows[8];             /* own rows (distributed levels) / global rows (agglomerated) */
    int64_t tiles[8];            /* own tiles / global tiles */
    int64_t row_begin[8];        /* first own row (distributed levels) */
    int64_t ext_begin[8], ext_end[8];  /* the row range the own rows' columns touch */
    int halo_recv[8], halo_send[8];    /* halo pieces received / sent per SpMV */
    int64_t interior[8][2];      /* interior block rows [begin, end) (computed while the halo flies) */
} amgt_dist_hier_info;
amgt_status amgt_dist_hierarchy_info(const amgt_dist_hierarchy* H, amgt_dist_hier_info* out);
amgt_status amgt_dist_hierarchy_destroy(amgt_dist_hierarchy* H);

/* Host only (no GPU, not collective): the halo plan of rank `rank` from the all-gathered metadata
 * — rows[q] own rows of the gathered operand per rank, colmin[q] / colmax[q] the min / max tile
 * column of rank q's matrix (colmin > colmax: no tiles).  ext_host = {eb, ee} (block rows);
 * recv: pieces [begin, end) of [eb, ee) owned by other ranks; send: pieces of the own block rows
 * in other ranks' ranges; at most cap each. */
typedef struct {
    int32_t peer;
    int64_t begin, end; /* global block rows */
} amgt_dist_piece;
amgt_status amgt_dist_plan_host(int rank, int size, const int64_t* rows, const int64_t* colmin, const int64_t* colmax,
                                int64_t* ext_host, amgt_dist_piece* recv, int* nrecv, amgt_dist_piece* send, int* nsend,
                                int cap);

/* ------------------------------------------------------------- instrumentation */

/* Per-kernel-class device timing with CUDA events recorded on the launching stream.
 * Classes: 0 SpMV level-1, 1 SpMV other levels, 2 SpGEMM symbolic, 3 SpGEMM numeric,
 * 4 CSR->mBSR, 5 mBSR->CSR, 6 cast, 7 vector ops. */
#define AMGT_TIMER_CLASSES 8
/* on: 0 = off, -1 = all classes, otherwise a bitmask (bit c enables class c). */
amgt_status amgt_timing_enable(int on);
/* Record events for one call in `every` (>= 1, default 1) of each enabled class: an event
 * pair between two programmatically dependent launches breaks their overlap, so sampling
 * keeps a live measurement from slowing the run it measures.  Reset by nothing. */
amgt_status amgt_timing_sample(int every);
amgt_status amgt_timing_reset(void);
/* Syncs the recorded events; fills ms_total[8], launches[8] and bytes[8] (algorithmic
 * bytes of SURVEY §8(d) per class) on the host. */
amgt_status amgt_timing_read(double* ms_total_host, int64_t* launches_host, double* bytes_host);
/* Number of kernel launches issued by the library since the last reset. */
int64_t amgt_launch_count(void);

#ifdef __cplusplus
}
#endif
#if defined(__GNUC__)
#pragma GCC visibility pop
#endif
#endif /* AMGT_H */
