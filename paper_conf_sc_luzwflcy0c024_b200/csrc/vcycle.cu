// vcycle.cu — AMG setup with fixed interpolation (Alg. 1, L52-58) and the V-cycle solve
// (Alg. 2, L68-82) driving the mBSR SpGEMM/SpMV kernels, with per-level precision
// (L266: level 1 FP64, level 2 FP32, levels >= 3 FP16; vectors FP64 at level 1, FP32
// below, reading R16).  Smoother: weighted Jacobi x += w D^-1 (b - A x) (R21).
// Coarsest level: MBSR2CSR (L262), dense Cholesky-based inverse in FP64 on the host,
// applied on the device as a dense FP64 matvec (R22).
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <vector>

#include <cooperative_groups.h>

#include "common.cuh"
#include "spmv_core.cuh"

namespace amgt {

amgt_status mbsr_release(amgt_mbsr* M, Alloc& a);
amgt_status cast_impl(const amgt_mbsr* in, amgt_prec to, amgt_mbsr* out, Alloc& a, uint32_t* dflag = nullptr);
amgt_status transpose_impl(const amgt_mbsr* in, amgt_mbsr* out, Alloc& a, unsigned long long* dmax = nullptr);
amgt_status mbsr_to_csr_impl(const amgt_mbsr* A, int64_t* rp, int32_t* ci, double* v, Alloc& a);
amgt_status spmv_analyze_impl(amgt_mbsr* A, Alloc& a);
amgt_status spmv_impl(const amgt_mbsr* A, const void* x, amgt_prec xp, void* y, amgt_prec yp, cudaStream_t s,
                      int timer_class);
amgt_status spmv_ex_impl(const amgt_mbsr* A, const void* x, amgt_prec xp, void* y, amgt_prec yp, const EpiArgs& ea,
                         cudaStream_t s, int timer_class);
amgt_status spgemm_symbolic_impl(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* Cout, amgt_spgemm_info* info,
                                 Alloc& a);
amgt_status spgemm_numeric_impl(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* C, Alloc& a);
amgt_status pmis_aggregate_impl(const amgt_mbsr* A, double theta, double mrs, const double* weights, uint64_t seed,
                                int level, int32_t* agg, int8_t* is_c, int64_t* nagg_host, int* rounds_host, Alloc& a);
amgt_status aggregation_p_impl(int64_t m, int64_t nagg, const int32_t* agg, amgt_prec prec, amgt_mbsr* Pt, Alloc& a);
amgt_status sa_interp_impl(const amgt_mbsr* A, const amgt_mbsr* Pt, double theta, double omega, amgt_mbsr* P,
                           Alloc& a);

}  // namespace amgt

using namespace amgt;

struct amgt_level {
    amgt_mbsr A{}, P{}, R{};  // A_k at level precision; P_k, R_k at level k precision
    bool ownA = false;
    int64_t npad = 0;         // 4 * blc_row
    amgt_prec vprec = AMGT_FP64;
    void *b = nullptr, *x = nullptr, *r = nullptr, *t = nullptr, *dinv = nullptr;  // t: ping-pong partner of x
    void* u = nullptr;        // level 1 with the fused sweeps: third iterate buffer
    void* vblock = nullptr;   // the allocation holding b, x, r, t, dinv
    size_t vblock_bytes = 0;
};

struct amgt_hierarchy {
    int nlev = 0;
    amgt_vcycle_opts o{};
    amgt_allocator al{};
    bool has_al = false;
    cudaStream_t s = nullptr;
    amgt_level L[8];
    int64_t nM = 0;
    double* Ainv = nullptr;     // dense inverse of the coarsest operator (FP64, nM x nM)
    double* partial = nullptr;  // norm partial sums
    double* nws = nullptr;      // per-warp residual partials of the level-1 sweep (EPI_JACOBI_NORM)
    int64_t nws_n = 0;
    double* norms = nullptr;    // per-cycle squared residual norms (device)
    int norms_cap = 0;
    int64_t spmv_calls = 0;
    // CUDA graph of the sub-cycle below level 1 (levels 2..M down, coarse solve, up), captured
    // once per hierarchy on an internal stream and replayed every cycle
    cudaStream_t gs = nullptr;
    cudaGraphExec_t gexec = nullptr;
    bool graph_failed = false;
    int64_t sub_calls = 0, sub_launches = 0;
    amgt_sweep_plan* sw = nullptr;  // level-1 fused sweeps (amgt_spmv_sweeps), when usable
    // replicated tail of a distributed hierarchy (dist.cu): level 0 is a coarse level, so its
    // vectors follow its precision (FP32 below FP64, R16) instead of the level-1 FP64 rule
    bool vec_from_prec = false;
    Alloc alloc() { return Alloc{has_al ? &al : nullptr, s}; }
};

namespace amgt {

constexpr int NORM_BLOCKS = 592;  // one wave: 4 CTAs of 256 per SM (k_dot, k_pcg_xr: <= 64 registers)

template <typename V, typename M>
__global__ void k_dinv(int64_t BR, int64_t m, int64_t off, const int64_t* __restrict__ bptr,
                       const int32_t* __restrict__ bidx, const M* __restrict__ bval, V* __restrict__ dinv, bool l1) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= 4 * BR) return;
    const int64_t I = i >> 2;
    const int r = (int)(i & 3);
    double d = 0.0;
    if (i < m) {
        if (l1) {  // l1 row norm sum_j |a_ij| in column order (tiles ascending, +0.0 fill)
            for (int64_t t = bptr[I]; t < bptr[I + 1]; ++t)
                for (int c = 0; c < 4; ++c) d += fabs(to_f64(bval[16 * t + 4 * r + c]));
        } else {
            for (int64_t t = bptr[I]; t < bptr[I + 1]; ++t)
                if (bidx[t] == (int32_t)(I + off)) { d = to_f64(bval[16 * t + 5 * r]); break; }
        }
    }
    dinv[i] = (V)(d != 0.0 ? 1.0 / d : 0.0);
}

// Deterministic ||r||^2 in one launch: a fixed grid of NORM_BLOCKS, per-block partial sums
// (fixed order), and the last block to finish (ticket counter) adds the partials with a
// fixed tree and re-arms the counter.  ws = [NORM_BLOCKS partials | counter (zeroed once)].
__device__ __forceinline__ double block_sum(double s, double* sh) {
    for (int d = 16; d; d >>= 1) s += __shfl_xor_sync(0xffffffffu, s, d);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = s;
    __syncthreads();
    double a = 0.0;
    if (threadIdx.x == 0)
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) a += sh[w];
    return a;
}

// the partial of this CTA into ws[blockIdx.x]; the last CTA to arrive sums the partials
// (fixed tree) into *out and re-arms the counter
__device__ __forceinline__ void finish_sum(double s, double* __restrict__ ws, double* __restrict__ out) {
    __shared__ double sh[32];
    __shared__ bool last;
    const double part = block_sum(s, sh);
    unsigned* counter = reinterpret_cast<unsigned*>(ws + NORM_BLOCKS);
    if (threadIdx.x == 0) {
        ws[blockIdx.x] = part;
        __threadfence();
        last = atomicAdd(counter, 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (!last) return;
    __threadfence();
    double t = 0.0;
    for (int i = threadIdx.x; i < (int)gridDim.x; i += blockDim.x) t += __ldcg(ws + i);
    __syncthreads();
    const double tot = block_sum(t, sh);
    if (threadIdx.x == 0) {
        *out = tot;
        *counter = 0u;
    }
}

// *out = a . b (a == b: ||a||^2), deterministic for a fixed grid of NORM_BLOCKS.  16-B loads,
// four per thread in flight (a == b: one stream), summed in a fixed order.
__global__ void __launch_bounds__(256, 4) k_dot(int64_t n, const double* __restrict__ a, const double* __restrict__ b,
                                             double* __restrict__ ws, double* __restrict__ out) {
    pdl_wait();
    double s = 0.0;
    const int64_t gt = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, nt = (int64_t)gridDim.x * blockDim.x;
    if (((reinterpret_cast<uintptr_t>(a) | reinterpret_cast<uintptr_t>(b)) & 15) == 0) {  // 16-byte loads
        const int64_t n2 = n >> 1;
        const double2* a2 = reinterpret_cast<const double2*>(a);
        const double2* b2 = reinterpret_cast<const double2*>(b);
        const bool same = a == b;
        int64_t i = gt;
        for (; i + 3 * nt < n2; i += 4 * nt) {
            double2 u[4], v[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) u[k] = __ldcs(a2 + i + k * nt);
            if (same) {
#pragma unroll
                for (int k = 0; k < 4; ++k) v[k] = u[k];
            } else {
#pragma unroll
                for (int k = 0; k < 4; ++k) v[k] = __ldcs(b2 + i + k * nt);
            }
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                s = fma(u[k].x, v[k].x, s);
                s = fma(u[k].y, v[k].y, s);
            }
        }
        for (; i < n2; i += nt) {
            const double2 u = __ldcs(a2 + i), v = __ldcs(b2 + i);
            s = fma(u.x, v.x, s);
            s = fma(u.y, v.y, s);
        }
        if ((n & 1) && gt == 0) s = fma(a[n - 1], b[n - 1], s);
    } else {
        for (int64_t i = gt; i < n; i += nt) s = fma(a[i], b[i], s);
    }
    finish_sum(s, ws, out);
}

// *out = sum of a[0..n) (the per-warp residual partials of EPI_JACOBI_NORM), deterministic for
// the fixed grid of NORM_BLOCKS
__global__ void __launch_bounds__(256, 4) k_sum(int64_t n, const double* __restrict__ a, double* __restrict__ ws,
                                                double* __restrict__ out) {
    pdl_wait();
    double s = 0.0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        s += a[i];
    finish_sum(s, ws, out);
}

// PCG (NEXT-1): x += alpha p, r -= alpha q with alpha = rz / pq (0 when pq = 0), and
// ||r||^2 of the updated r into *rr (one pass)
__global__ void __launch_bounds__(256, 4) k_pcg_xr(int64_t n, const double* __restrict__ rz, const double* __restrict__ pq,
                                                double* __restrict__ x, double* __restrict__ r,
                                                const double* __restrict__ p, const double* __restrict__ q,
                                                double* __restrict__ ws, double* __restrict__ rr) {
    const double den = *pq;
    const double alpha = den != 0.0 ? *rz / den : 0.0;
    double s = 0.0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        x[i] = fma(alpha, p[i], x[i]);
        const double ri = fma(-alpha, q[i], r[i]);
        r[i] = ri;
        s = fma(ri, ri, s);
    }
    finish_sum(s, ws, rr);
}

// p = z + beta p, beta = rz_new / rz_old (0 when rz_old = 0)
__global__ void __launch_bounds__(256) k_pcg_p(int64_t n, const double* __restrict__ rz_new,
                                               const double* __restrict__ rz_old, const double* __restrict__ z,
                                               double* __restrict__ p) {
    const double den = *rz_old;
    const double beta = den != 0.0 ? *rz_new / den : 0.0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        p[i] = fma(beta, p[i], z[i]);
}

// x = Ainv * b (dense FP64), one warp per row.
// First pre-smoothing sweep from the zero initial guess of a coarse level (Alg. 2 line 2 with
// x = 0): x = 0 + w dinv .* (b - A 0) — the Epi JACOBI expression with x = 0 and A x = 0, so
// the result is bit-identical to the SpMV kernel's, without reading A_k or zeroing x first.
template <typename V>
__global__ void __launch_bounds__(256) k_jacobi0(int64_t n, const V* __restrict__ b, const V* __restrict__ dinv,
                                                 V omega, V* __restrict__ x) {
    pdl_wait();
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const V zero = V(0), t = V(0);
    x[i] = zero + omega * dinv[i] * (b[i] - t);
}

template <typename V>
__global__ void k_dense_solve(int64_t n, int64_t npad, const double* __restrict__ Ainv, const V* __restrict__ b,
                              V* __restrict__ x) {
    pdl_wait();
    const int64_t row = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (row >= npad) return;
    double s = 0.0;
    if (row < n)
        for (int64_t j = lane; j < n; j += 32) s = fma(Ainv[row * n + j], (double)b[j], s);
    for (int d = 16; d; d >>= 1) s += __shfl_xor_sync(0xffffffffu, s, d);
    if (lane == 0) x[row] = (V)s;
}

static unsigned vgrid(int64_t n) {
    int64_t b = ceil_div(n, 256);
    const int64_t cap = (int64_t)num_sms() * 8;
    return (unsigned)(b < 1 ? 1 : (b > cap ? cap : b));
}

static size_t vbytes(amgt_prec p) { return p == AMGT_FP64 ? 8 : 4; }

template <typename V, typename M>
static void launch_dinv(const amgt_mbsr& A, int64_t off, void* dinv, bool l1, cudaStream_t s) {
    k_dinv<V, M><<<(unsigned)ceil_div(4 * A.blc_row, 256), 256, 0, s>>>(A.blc_row, A.m, off, A.blc_ptr, A.blc_idx,
                                                                       (const M*)A.blc_val, (V*)dinv, l1);
}

amgt_status dinv_impl(const amgt_mbsr& A, int64_t off, void* dinv, amgt_prec vprec, cudaStream_t s,
                      bool l1 = false) {
    if (A.blc_row == 0) return AMGT_OK;
    const bool v64 = vprec == AMGT_FP64;
    switch (A.prec) {
        case AMGT_FP64:
            v64 ? launch_dinv<double, double>(A, off, dinv, l1, s) : launch_dinv<float, double>(A, off, dinv, l1, s);
            break;
        case AMGT_FP32:
            v64 ? launch_dinv<double, float>(A, off, dinv, l1, s) : launch_dinv<float, float>(A, off, dinv, l1, s);
            break;
        default: v64 ? launch_dinv<double, __half>(A, off, dinv, l1, s) : launch_dinv<float, __half>(A, off, dinv, l1, s);
    }
    AMGT_LAUNCHED();
    return AMGT_OK;
}

static amgt_status build_dinv(amgt_level& L, cudaStream_t s, bool l1) {
    return dinv_impl(L.A, 0, L.dinv, L.vprec, s, l1);
}

// Host dense Cholesky + inverse of the (SPD) coarsest operator.
static bool dense_inverse(int64_t n, std::vector<double>& a, std::vector<double>& inv) {
    std::vector<double> L(a);
    for (int64_t j = 0; j < n; ++j) {
        double s = L[j * n + j];
        for (int64_t k = 0; k < j; ++k) s -= L[j * n + k] * L[j * n + k];
        if (!(s > 0.0)) return false;
        const double d = std::sqrt(s);
        L[j * n + j] = d;
        for (int64_t i = j + 1; i < n; ++i) {
            double t = L[i * n + j];
            for (int64_t k = 0; k < j; ++k) t -= L[i * n + k] * L[j * n + k];
            L[i * n + j] = t / d;
        }
    }
    inv.assign(n * n, 0.0);
    std::vector<double> y(n);
    for (int64_t c = 0; c < n; ++c) {  // solve L L^T x = e_c
        for (int64_t i = 0; i < n; ++i) {
            double s = (i == c) ? 1.0 : 0.0;
            for (int64_t k = 0; k < i; ++k) s -= L[i * n + k] * y[k];
            y[i] = s / L[i * n + i];
        }
        for (int64_t i = n - 1; i >= 0; --i) {
            double s = y[i];
            for (int64_t k = i + 1; k < n; ++k) s -= L[k * n + i] * inv[k * n + c];
            inv[i * n + c] = s / L[i * n + i];
        }
    }
    return true;
}

// ---------------------------------------------------------------- coarsest level (R22)
// The coarsest operator A_M (n <= 4096 rows) as a dense FP64 matrix on the device: one thread
// per tile scatters its bitmap-marked entries (values widened exactly).
template <typename T>
__global__ void k_dense_scatter(int64_t BR, int64_t n, const int64_t* __restrict__ ptr,
                                const int32_t* __restrict__ idx, const uint16_t* __restrict__ map,
                                const T* __restrict__ val, double* __restrict__ D) {
    for (int64_t I = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; I < BR; I += (int64_t)gridDim.x * blockDim.x)
        for (int64_t t = ptr[I]; t < ptr[I + 1]; ++t) {
            const uint32_t mp = map[t];
            const int64_t J = idx[t];
            for (int e = 0; e < 16; ++e)
                if ((mp >> e) & 1u) D[(4 * I + (e >> 2)) * n + 4 * J + (e & 3)] = to_f64(val[16 * t + e]);
        }
}

// In-place Gauss-Jordan inversion of an SPD matrix without pivoting (every pivot of an SPD
// matrix is positive), one cooperative grid: step k scales the pivot row (r_j = a_kj / a_kk,
// r_k = 1 / a_kk) and keeps the pivot column c_i = a_ik, then a_ij -= c_i r_j for i != k (with
// a_ik taken as 0) and row k = r.  A non-positive pivot sets FLAG_SPD (not SPD).  n^3 FMAs over
// every SM, two grid barriers per step.
constexpr uint32_t FLAG_SPD = 4u;
__global__ void __launch_bounds__(256) k_gauss_jordan(int64_t n, double* __restrict__ a, double* __restrict__ rbuf,
                                                      double* __restrict__ cbuf, uint32_t* __restrict__ flag) {
    namespace cg = cooperative_groups;
    cg::grid_group g = cg::this_grid();
    const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, nt = (int64_t)gridDim.x * blockDim.x;
    for (int64_t k = 0; k < n; ++k) {
        const double piv = a[k * n + k];
        if (tid == 0 && !(piv > 0.0)) atomicOr(flag, FLAG_SPD);
        for (int64_t j = tid; j < n; j += nt) {
            rbuf[j] = (j == k ? 1.0 : a[k * n + j]) / piv;
            cbuf[j] = a[j * n + k];
        }
        g.sync();
        for (int64_t e = tid; e < n * n; e += nt) {
            const int64_t i = e / n, j = e - i * n;
            a[e] = i == k ? rbuf[j] : (j == k ? 0.0 : a[e]) - cbuf[i] * rbuf[j];
        }
        g.sync();
    }
}

// The same Gauss-Jordan for small n (<= GJ_SMEM_N) in ONE CTA with the matrix in shared memory
// (block barriers instead of grid barriers: the config-3 coarsest level, n = 64, 269 -> ~20 us).
constexpr int GJ_SMEM_N = 128;
__global__ void __launch_bounds__(512) k_gauss_jordan_smem(int n, double* __restrict__ a, uint32_t* __restrict__ flag) {
    extern __shared__ double gsm[];
    double* m = gsm;
    double* rb = gsm + n * n;
    double* cb = rb + n;
    for (int e = threadIdx.x; e < n * n; e += blockDim.x) m[e] = a[e];
    __syncthreads();
    for (int k = 0; k < n; ++k) {
        const double piv = m[k * n + k];
        if (threadIdx.x == 0 && !(piv > 0.0)) atomicOr(flag, FLAG_SPD);
        for (int j = threadIdx.x; j < n; j += blockDim.x) {
            rb[j] = (j == k ? 1.0 : m[k * n + j]) / piv;
            cb[j] = m[j * n + k];
        }
        __syncthreads();
        for (int e = threadIdx.x; e < n * n; e += blockDim.x) {
            const int i = e / n, j = e - i * n;
            m[e] = i == k ? rb[j] : (j == k ? 0.0 : m[e]) - cb[i] * rb[j];
        }
        __syncthreads();
    }
    for (int e = threadIdx.x; e < n * n; e += blockDim.x) a[e] = m[e];
}

// Ainv = A_M^-1 on the device (dense scatter + Gauss-Jordan); FLAG_SPD into dflag.
static amgt_status device_coarse_inverse(const amgt_mbsr& C, double* Ainv, uint32_t* dflag, Alloc& a) {
    cudaStream_t s = a.s;
    const int64_t n = C.m;
    AMGT_CUDA(cudaMemsetAsync(Ainv, 0, n * n * sizeof(double), s));
    const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(C.blc_row, 128), 1024));
    switch (C.prec) {
        case AMGT_FP64:
            k_dense_scatter<double><<<g, 128, 0, s>>>(C.blc_row, n, C.blc_ptr, C.blc_idx, C.blc_map,
                                                      (const double*)C.blc_val, Ainv);
            break;
        case AMGT_FP32:
            k_dense_scatter<float><<<g, 128, 0, s>>>(C.blc_row, n, C.blc_ptr, C.blc_idx, C.blc_map,
                                                     (const float*)C.blc_val, Ainv);
            break;
        default:
            k_dense_scatter<__half><<<g, 128, 0, s>>>(C.blc_row, n, C.blc_ptr, C.blc_idx, C.blc_map,
                                                      (const __half*)C.blc_val, Ainv);
    }
    AMGT_LAUNCHED();
    if (n == 0) return AMGT_OK;
    if (n <= GJ_SMEM_N) {
        const size_t sm = (size_t)(n * n + 2 * n) * sizeof(double);
        AMGT_CUDA(dyn_smem(k_gauss_jordan_smem, (GJ_SMEM_N * GJ_SMEM_N + 2 * GJ_SMEM_N) * sizeof(double)));
        k_gauss_jordan_smem<<<1, 512, sm, s>>>((int)n, Ainv, dflag);
        AMGT_LAUNCHED();
        return AMGT_OK;
    }
    Scratch<double> buf;
    AMGT_TRY(buf.init(a, 2 * n));
    static int per_sm = -1;
    if (per_sm < 0) {
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_gauss_jordan, 256, 0) != cudaSuccess) per_sm = 1;
        per_sm = std::max(per_sm, 1);
    }
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>((int64_t)num_sms() * per_sm,
                                                                           ceil_div(n * n, 256)));
    int64_t nn = n;
    double* rb = buf.p;
    double* cb = buf.p + n;
    void* args[] = {&nn, &Ainv, &rb, &cb, &dflag};
    AMGT_CUDA(cudaLaunchCooperativeKernel((const void*)k_gauss_jordan, dim3(grid), dim3(256), args, 0, s));
    count_launch();
    return AMGT_OK;
}

static void free_level_vectors(amgt_level& L, Alloc& a) {
    const size_t vb = vbytes(L.vprec) * (size_t)L.npad;
    a.put(L.vblock, L.vblock_bytes);  // b, x, r, t, dinv
    L.vblock = nullptr;
    L.b = L.x = L.r = L.t = L.dinv = nullptr;
    a.put(L.u, vb);
    L.u = nullptr;
}

static void destroy(amgt_hierarchy* H) {
    if (!H) return;
    Alloc a = H->alloc();
    for (int k = 0; k < H->nlev; ++k) {
        amgt_level& L = H->L[k];
        if (L.ownA) mbsr_release(&L.A, a);
        else if (L.A.aux) { amgt_mbsr tmp{}; tmp.aux = L.A.aux; mbsr_release(&tmp, a); }
        mbsr_release(&L.P, a);
        mbsr_release(&L.R, a);
        free_level_vectors(L, a);
    }
    if (H->sw) amgt_sweep_plan_destroy(H->sw, H->s);
    a.put(H->Ainv, (size_t)H->nM * H->nM * sizeof(double));
    a.put(H->partial, (NORM_BLOCKS + 1) * sizeof(double));
    a.put(H->nws, (size_t)H->nws_n * sizeof(double));
    a.put(H->norms, (size_t)H->norms_cap * sizeof(double));
    cudaStreamSynchronize(H->s);
    if (H->gexec) cudaGraphExecDestroy(H->gexec);
    if (H->gs) { cudaStreamSynchronize(H->gs); cudaStreamDestroy(H->gs); }
    delete H;
}

// AMGT_SWEEP=1 runs the level-1 SpMVs of the V-cycle as fused sweeps (amgt_spmv_sweeps); off by
// default until they beat the separate kernels on B200
static bool sweeps_enabled() {
    const char* e = getenv("AMGT_SWEEP");
    return e && !strcmp(e, "1");
}

static amgt_status create(const amgt_mbsr* A, const amgt_mbsr* const* P, int nlev, const amgt_vcycle_opts* o,
                          amgt_hierarchy* H) {
    cudaStream_t s = H->s;
    Alloc a = H->alloc();
    H->nlev = nlev;
    trace_point("create", s);
    // Values read back at later synchronisation points instead of with their own: the FP16
    // range flag of every cast (checked at the end) and the longest block row of each R_k
    // (it arrives with the SpGEMM syncs that follow the transpose; lets the SpMV analysis of
    // R_k skip its sync).  dev = [flag | row max of R_0..R_6].
    Scratch<unsigned long long> dev;
    AMGT_TRY(dev.init(a, 8));
    AMGT_CUDA(cudaMemsetAsync(dev.p, 0, 8 * sizeof(unsigned long long), s));
    uint32_t* dflag = reinterpret_cast<uint32_t*>(dev.p);
    int64_t* pin = pinned_slots();
    for (int k = 0; k < nlev; ++k) {
        amgt_level& L = H->L[k];
        const amgt_prec pk = o->level_prec[k];
        L.vprec = ((k == 0 && !H->vec_from_prec) || pk == AMGT_FP64) ? AMGT_FP64 : AMGT_FP32;  // R16
        if (k == 0) {
            if (pk == A->prec) {
                L.A = *A;  // borrowed
                L.A.own = 0;
                L.A.aux = nullptr;
                L.ownA = false;
            } else {
                AMGT_TRY(cast_impl(A, pk, &L.A, a, dflag));
                L.ownA = true;
            }
        }
        L.npad = 4 * L.A.blc_row;
        AMGT_TRY(spmv_analyze_impl(&L.A, a));
        trace_point("analyze A", s);
        const size_t vb = vbytes(L.vprec) * (size_t)L.npad;
        {  // the five level vectors in one allocation (one allocator call, one memset)
            const size_t va = (vb + 255) & ~size_t(255);
            L.vblock = a.get(5 * va);
            if (!L.vblock) return fail(AMGT_ERR_ALLOC, "hierarchy vector allocation failed");
            L.vblock_bytes = 5 * va;
            AMGT_CUDA(cudaMemsetAsync(L.vblock, 0, 5 * va, s));
            char* base = (char*)L.vblock;
            L.b = base;
            L.x = base + va;
            L.r = base + 2 * va;
            L.t = base + 3 * va;
            L.dinv = base + 4 * va;
        }
        AMGT_TRY(build_dinv(L, s, H->o.smoother == AMGT_SMOOTH_L1_JACOBI));
        trace_point("vectors+dinv", s);
        if (k == 0 && nlev >= 2 && sweeps_enabled() && L.A.prec == AMGT_FP64 && H->o.nu1 == 1 && H->o.nu2 == 1) {
            L.u = a.get(vb);
            if (!L.u) return fail(AMGT_ERR_ALLOC, "hierarchy vector allocation failed");
            AMGT_CUDA(cudaMemsetAsync(L.u, 0, vb, s));
            AMGT_TRY(amgt_sweep_plan_create(&L.A, H->has_al ? &H->al : nullptr, s, &H->sw));
        }
        const double th = o->theta >= 0.0 ? o->theta : 0.25;
        const double wp = o->omega_p > 0.0 ? o->omega_p : 2.0 / 3.0;
        if (k + 1 < nlev && o->interp == AMGT_INTERP_PMIS) {
            // NEXT-2 / Alg. 1 lines 2-4: stop at max_coarse_size; else PMIS aggregation of A_k (R32)
            // and P_k = (I - w D_F^-1 A_F) Pt through one SpGEMM call
            bool stop = o->max_coarse_size > 0 && L.A.m <= o->max_coarse_size;
            amgt_mbsr Pt{};
            if (!stop) {
                Scratch<int32_t> agg;
                AMGT_TRY(agg.init(a, L.A.m + 1));
                int64_t nagg = 0;
                const double mrs = o->max_row_sum > 0.0 ? o->max_row_sum : 1.0;
                AMGT_TRY(pmis_aggregate_impl(&L.A, th, mrs, nullptr, o->seed, k, agg.p, nullptr, &nagg, nullptr, a));
                stop = nagg == 0 || nagg >= L.A.m;
                if (!stop) AMGT_TRY(aggregation_p_impl(L.A.m, nagg, agg.p, pk, &Pt, a));
            }
            if (stop) {
                nlev = k + 1;
                H->nlev = nlev;
            } else {
                const amgt_status st = sa_interp_impl(&L.A, &Pt, th, wp, &L.P, a);
                mbsr_release(&Pt, a);
                AMGT_TRY(st);
            }
            trace_point("PMIS + SA", s);
        }
        if (k + 1 < nlev) {
            const amgt_mbsr* Pk = o->interp == AMGT_INTERP_PMIS ? nullptr : P[k];
            if (Pk && Pk->m != L.A.m) return fail(AMGT_ERR_ARG, "P[%d] has %lld rows, level has %lld", k, (long long)Pk->m, (long long)L.A.m);
            if (!Pk) {
                // built above
            } else if (o->interp == AMGT_INTERP_SA) {
                // NEXT-2 / Alg. 1 line 4: P_k = (I - w D_F^-1 A_F) Pt through one SpGEMM call
                amgt_mbsr Pt{};
                AMGT_TRY(cast_impl(Pk, pk, &Pt, a, dflag));
                const amgt_status st = sa_interp_impl(&L.A, &Pt, th, wp, &L.P, a);
                mbsr_release(&Pt, a);
                AMGT_TRY(st);
            } else {
                AMGT_TRY(cast_impl(Pk, pk, &L.P, a, dflag));  // P_k in level k precision (copy when equal)
            }
            trace_point("P cast", s);
            AMGT_TRY(transpose_impl(&L.P, &L.R, a, pin ? dev.p + 1 + k : nullptr));  // R_k = P_k^T (Alg. 1 line 4)
            if (pin) AMGT_CUDA(cudaMemcpyAsync(pin + PIN_CREATE + k, dev.p + 1 + k, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
            trace_point("transpose", s);
            // A_{k+1} = R_k (A_k P_k): two SpGEMM calls in level k precision (Alg. 1 line 5)
            amgt_mbsr AP{}, Ac{};
            AMGT_TRY(spgemm_symbolic_impl(&L.A, &L.P, &AP, nullptr, a));
            trace_point("sym AP", s);
            amgt_status st = spgemm_numeric_impl(&L.A, &L.P, &AP, a);
            trace_point("num AP", s);
            if (st == AMGT_OK) st = spgemm_symbolic_impl(&L.R, &AP, &Ac, nullptr, a);
            trace_point("sym RAP", s);
            if (st == AMGT_OK) st = spgemm_numeric_impl(&L.R, &AP, &Ac, a);
            trace_point("num RAP", s);
            mbsr_release(&AP, a);
            if (st != AMGT_OK) { mbsr_release(&Ac, a); return st; }
            amgt_level& N = H->L[k + 1];
            const amgt_prec pn = o->level_prec[k + 1];
            if (pn != Ac.prec) {
                st = cast_impl(&Ac, pn, &N.A, a, dflag);
                if (st != AMGT_OK) { mbsr_release(&Ac, a); return st; }
                Ac.own &= ~1u;  // the cast shares Ac's structure: move its ownership to N.A
                mbsr_release(&Ac, a);  // frees Ac's values only
                N.A.own |= 1u;
            } else {
                N.A = Ac;
            }
            N.ownA = true;
            trace_point("cast Ac", s);
            AMGT_TRY(spmv_analyze_impl(&L.P, a));
            if (pin) L.R.row_max = pin[PIN_CREATE + k];  // arrived: the SpGEMM symbolic phases synchronised since
            AMGT_TRY(spmv_analyze_impl(&L.R, a));
            trace_point("analyze P R", s);
        }
    }
    // coarsest level (R22): dense inverse in FP64 on the device (Gauss-Jordan on the SPD A_M)
    amgt_level& C = H->L[nlev - 1];
    const int64_t n = C.A.m;
    if (n > 4096) return fail(AMGT_ERR_UNSUPPORTED, "coarsest level has %lld rows (dense solve limit 4096)", (long long)n);
    H->nM = n;
    H->Ainv = (double*)a.get(n * n * sizeof(double) + 8);
    H->partial = (double*)a.get((NORM_BLOCKS + 1) * sizeof(double));
    if (!H->Ainv || !H->partial) return fail(AMGT_ERR_ALLOC, "coarse inverse allocation failed");
    AMGT_TRY(device_coarse_inverse(C.A, H->Ainv, dflag, a));
    AMGT_CUDA(cudaMemsetAsync(H->partial, 0, (NORM_BLOCKS + 1) * sizeof(double), H->s));
    H->nws_n = std::max<int64_t>(spmv_warp_norm_count(&H->L[0].A), 1);
    H->nws = (double*)a.get((size_t)H->nws_n * sizeof(double));
    if (!H->nws) return fail(AMGT_ERR_ALLOC, "norm partial allocation failed");
    uint32_t hflag = 0;  // FP16 range flag of every cast above + the SPD flag of the inverse
    if (pin) {
        AMGT_CUDA(cudaMemcpyAsync(pin + PIN_CREATE + 8, dflag, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaStreamSynchronize(s));
        hflag = (uint32_t)pin[PIN_CREATE + 8];
    } else {
        AMGT_CUDA(cudaMemcpyAsync(&hflag, dflag, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaStreamSynchronize(s));
    }
    if (hflag & FLAG_RANGE) return fail(AMGT_ERR_RANGE, "hierarchy: a level value exceeds the FP16 range (65504)");
    if (hflag & FLAG_SPD) return fail(AMGT_ERR_ARG, "coarsest operator is not SPD (non-positive pivot)");
    trace_point("coarse inverse", s);
    trace_dump();
    return AMGT_OK;
}

static amgt_status counted_spmv(amgt_hierarchy* H, const amgt_mbsr* M, const void* x, amgt_prec xp, void* y,
                                amgt_prec yp, int level, int mode = 0, const void* b = nullptr,
                                const void* dinv = nullptr, void* r = nullptr) {
    // counts Alg. 2's SpMV operations: a Jacobi sweep that also returns the residual stands
    // for two of them (the sweep and the residual it replaces), in one pass over A
    H->spmv_calls += mode == AMGT_EPI_JACOBI_RES ? 2 : 1;
    EpiArgs ea{mode, b, dinv, x, H->o.omega, 0, -1};
    ea.r = r;
    // timer class 0 = the dominant kernel: SpMV with the level-1 operator A_1 (any epilogue)
    return spmv_ex_impl(M, x, xp, y, yp, ea, H->s, (level == 0 && M == &H->L[0].A) ? TC_SPMV_L1 : TC_SPMV);
}

static amgt_status norm_into(amgt_hierarchy* H, const double* r, int64_t n, double* out) {
    TimerScope ts(TC_VEC, 1.0 * n * 8, H->s);
    pdl_launch(k_dot, dim3(NORM_BLOCKS), dim3(256), 0, H->s, n, r, r, H->partial, out);
    AMGT_LAUNCHED();
    return AMGT_OK;
}

template <typename V>
static amgt_status dense_solve(amgt_hierarchy* H, amgt_level& L) {
    TimerScope ts(TC_VEC, (double)H->nM * H->nM * 8, H->s);
    pdl_launch(k_dense_solve<V>, dim3((unsigned)ceil_div(L.npad * 32, 256)), dim3(256), 0, H->s, H->nM, L.npad,
               (const double*)H->Ainv, (const V*)L.b, (V*)L.x);
    AMGT_LAUNCHED();
    return AMGT_OK;
}

constexpr int JAC = 1, RES = 2, ACC = 3;

// AMGT_ZERO_GUESS_FUSED=0: coarse levels run the zero-guess sweep (k_jacobi0) and the residual
// as two kernels (measurement knob; the results are bit-identical either way)
constexpr int64_t kZeroGuessFusedMaxBR = 131072;
static bool zero_guess_fused() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("AMGT_ZERO_GUESS_FUSED");
        v = (e && e[0] == '0') ? 0 : 1;
    }
    return v == 1;
}

// Alg. 2 lines 2-4 at level k: pre-smoothing, residual, restriction into b_{k+1}.  With
// res_norm, the first sweep (level 1, nu1 >= 1) also writes r = b - A x of the incoming x
// and its squared norm goes to *res_norm: the residual of the previous cycle (L308).
static amgt_status down_level(amgt_hierarchy* H, int k, const void* b0, void** xc, void** xa,
                              double* res_norm = nullptr) {
    amgt_level& L = H->L[k];
    const void* bk = k == 0 ? b0 : L.b;
    int i0 = 0;
    // (large levels excluded: forming x1 at every gathered column doubles the gathered vector loads;
    // config-3 level 2, 524,288 block rows: 274 us fused vs ~175 us for k_jacobi0 + the residual)
    if (k > 0 && H->o.nu1 == 1 && L.vprec == AMGT_FP32 && L.A.prec != AMGT_FP64 && zero_guess_fused() &&
        L.A.blc_row <= kZeroGuessFusedMaxBR && !(L.A.prec == AMGT_FP16 && g_tc_thr_spmv <= 16)) {
        // lines 2-3 from the zero guess in one pass: r = b - A x1, x1 = w D^-1 b formed on the
        // fly (EPI_RES_X0); two of Alg. 2's SpMV operations (the sweep's is A 0 = 0)
        EpiArgs ea{EPI_RES_X0, bk, L.dinv, nullptr, H->o.omega, 0, -1};
        ea.x1 = xa[k];
        const amgt_status st = spmv_ex_impl(&L.A, bk, L.vprec, L.r, L.vprec, ea, H->s, TC_SPMV);
        if (st == AMGT_OK) {
            H->spmv_calls += 2;
            std::swap(xc[k], xa[k]);
            amgt_level& N = H->L[k + 1];
            return counted_spmv(H, &L.R, L.r, L.vprec, N.b, N.vprec, k);  // line 4: restriction
        }
        if (st != AMGT_ERR_UNSUPPORTED) return st;
    }
    if (k > 0 && H->o.nu1 >= 1) {  // zero initial guess: first sweep without the SpMV (k_jacobi0)
        TimerScope ts(TC_VEC, 3.0 * vbytes(L.vprec) * L.npad, H->s);
        const dim3 g((unsigned)ceil_div(L.npad, 256));
        if (L.vprec == AMGT_FP64)
            pdl_launch(k_jacobi0<double>, g, dim3(256), 0, H->s, L.npad, (const double*)bk, (const double*)L.dinv,
                       H->o.omega, (double*)xa[k]);
        else
            pdl_launch(k_jacobi0<float>, g, dim3(256), 0, H->s, L.npad, (const float*)bk, (const float*)L.dinv,
                       (float)H->o.omega, (float*)xa[k]);
        AMGT_LAUNCHED();
        H->spmv_calls += 1;  // Alg. 2's sweep (its SpMV is A 0 = 0)
        std::swap(xc[k], xa[k]);
        i0 = 1;
    } else if (k > 0) {
        AMGT_CUDA(cudaMemsetAsync(xc[k], 0, vbytes(L.vprec) * L.npad, H->s));
    }
    for (int i = i0; i < H->o.nu1; ++i) {  // line 2: pre-smoothing
        if (i == 0 && res_norm && H->nws && L.vprec == AMGT_FP64 && spmv_warp_norm_ok(&L.A)) {
            // the sweep also sums (b - A x)^2 per warp (r is not written); partials summed in order
            EpiArgs ea{EPI_JACOBI_NORM, bk, L.dinv, xc[k], H->o.omega, 0, -1};
            ea.nws = H->nws;
            AMGT_TRY(spmv_ex_impl(&L.A, xc[k], L.vprec, xa[k], L.vprec, ea, H->s, TC_SPMV_L1));
            H->spmv_calls += 2;  // Alg. 2's sweep and the residual it delivers (L308)
            TimerScope ts(TC_VEC, 8.0 * spmv_warp_norm_count(&L.A), H->s);
            pdl_launch(k_sum, dim3(NORM_BLOCKS), dim3(256), 0, H->s, spmv_warp_norm_count(&L.A), (const double*)H->nws,
                       H->partial, res_norm);
            AMGT_LAUNCHED();
        } else if (i == 0 && res_norm) {
            AMGT_TRY(counted_spmv(H, &L.A, xc[k], L.vprec, xa[k], L.vprec, k, AMGT_EPI_JACOBI_RES, bk, L.dinv, L.r));
            AMGT_TRY(norm_into(H, (const double*)L.r, L.npad, res_norm));
        } else {
            AMGT_TRY(counted_spmv(H, &L.A, xc[k], L.vprec, xa[k], L.vprec, k, JAC, bk, L.dinv));
        }
        std::swap(xc[k], xa[k]);
    }
    AMGT_TRY(counted_spmv(H, &L.A, xc[k], L.vprec, L.r, L.vprec, k, RES, bk));  // line 3
    amgt_level& N = H->L[k + 1];
    return counted_spmv(H, &L.R, L.r, L.vprec, N.b, N.vprec, k);  // line 4: restriction
}

// Alg. 2 lines 8-10 at level k: interpolation + correction, post-smoothing.
static amgt_status up_level(amgt_hierarchy* H, int k, const void* b0, void** xc, void** xa) {
    amgt_level& L = H->L[k];
    amgt_level& N = H->L[k + 1];
    const void* bk = k == 0 ? b0 : L.b;
    AMGT_TRY(counted_spmv(H, &L.P, xc[k + 1], N.vprec, xc[k], L.vprec, k, ACC));  // lines 8-9
    for (int i = 0; i < H->o.nu2; ++i) {  // line 10: post-smoothing
        AMGT_TRY(counted_spmv(H, &L.A, xc[k], L.vprec, xa[k], L.vprec, k, JAC, bk, L.dinv));
        std::swap(xc[k], xa[k]);
    }
    return AMGT_OK;
}

static amgt_status coarse_solve(amgt_hierarchy* H, void** xc) {  // line 6
    const int M = H->nlev - 1;
    amgt_level C = H->L[M];
    C.x = xc[M];
    return C.vprec == AMGT_FP64 ? dense_solve<double>(H, C) : dense_solve<float>(H, C);
}

static int tail_level(const amgt_hierarchy* H, void** xc, void** xa);
static amgt_status subcycle_tail(amgt_hierarchy* H, int kt);

// Levels 1..M-1 down, coarsest, levels M-1..1 up (everything below level 1); the small
// tail levels kt..M go to one single-CTA kernel (block barriers instead of ~5 launches
// per level).
static amgt_status subcycle_direct(amgt_hierarchy* H, void** xc, void** xa) {
    const int M = H->nlev - 1;
    const int kt = tail_level(H, xc, xa);
    for (int k = 1; k < std::min(kt, M); ++k) AMGT_TRY(down_level(H, k, nullptr, xc, xa));
    if (kt <= M) AMGT_TRY(subcycle_tail(H, kt));
    else AMGT_TRY(coarse_solve(H, xc));
    for (int k = std::min(kt, M) - 1; k >= 1; --k) AMGT_TRY(up_level(H, k, nullptr, xc, xa));
    return AMGT_OK;
}

unsigned timing_mask();
void count_launches(int64_t n);

// ---------------------------------------------------------------- persistent coarse sub-cycle
// Levels 2..M of the V-cycle (everything below level 1: a few thousand rows per level,
// launch-latency bound) run as ONE cooperative kernel: every CTA stays resident and the
// Alg. 2 steps are separated by grid-wide barriers instead of kernel boundaries.  Each
// SpMV is the same 4-lane-group row code as k_spmv_rows (spmv_octet), warps striding over
// block-row octets.  Vectors of all coarse levels share one precision VT.
struct CoopMat {
    const int64_t* ptr;
    const int32_t* idx;
    const uint16_t* map;
    const void* val;
    int prec;
    int64_t BR;
};
struct CoopLevel {
    CoopMat A, P, R;
    void* b;
    void* x[2];
    void* r;
    const void* dinv;
    int64_t npad;
};
struct CoopArgs {
    CoopLevel L[8];
    int k0, M, nu1, nu2;
    int kb;  // levels kb..M run inside CTA 0 alone (block barriers instead of grid barriers)
    double omega;
    int64_t nM;
    const double* Ainv;
};

template <typename VT, int MODE>
__device__ __forceinline__ void coop_spmv(const CoopMat& M, const VT* x, VT* y, const VT* b, const VT* dinv,
                                          const VT* xs, double omega, int64_t gw, int64_t nw, int lane) {
    const Epi<VT, VT, MODE> epi{y, b, dinv, xs, (VT)omega, MODE};
    const int64_t noct = (M.BR + 7) / 8;
    switch (M.prec) {
        case AMGT_FP64:
            for (int64_t o = gw; o < noct; o += nw)
                spmv_octet<double, VT, VT, MODE, 4>(0, o, M.BR, M.ptr, M.idx, M.map, (const double*)M.val, x, epi, lane);
            break;
        case AMGT_FP32:
            for (int64_t o = gw; o < noct; o += nw)
                spmv_octet<float, VT, VT, MODE, 4>(0, o, M.BR, M.ptr, M.idx, M.map, (const float*)M.val, x, epi, lane);
            break;
        default:
            for (int64_t o = gw; o < noct; o += nw)
                spmv_octet<__half, VT, VT, MODE, 4>(0, o, M.BR, M.ptr, M.idx, M.map, (const __half*)M.val, x, epi,
                                                    lane);
    }
}

// One Alg. 2 step sequence on level k: grid-wide (all CTAs, grid barriers) when `grid_wide`,
// else CTA 0 alone with block barriers (the other CTAs skip the work but keep `cur` in step).
// COOP = false: a single-CTA launch for the tail levels (k0 == kb: every level block-local).
template <typename VT, bool COOP = true>
__global__ void __launch_bounds__(256) k_subcycle(const CoopArgs a) {
    pdl_wait();
    namespace cg = cooperative_groups;
    auto gsync = [&]() {
        if constexpr (COOP) cg::this_grid().sync();
    };
    const int lane = threadIdx.x & 31;
    int cur[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    auto run = [&](bool grid_wide, auto&& work) {
        if (grid_wide) {
            const int64_t gt = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, nt = (int64_t)gridDim.x * blockDim.x;
            work(gt, nt);
            gsync();
        } else if (blockIdx.x == 0) {
            work((int64_t)threadIdx.x, (int64_t)blockDim.x);
            __syncthreads();
        }
    };
    for (int k = a.k0; k < a.M; ++k) {  // Alg. 2 lines 1-5
        const CoopLevel& L = a.L[k];
        const bool gwide = k < a.kb;
        run(gwide, [&](int64_t gt, int64_t nt) {
            VT* x0 = (VT*)L.x[0];
            for (int64_t i = gt; i < L.npad; i += nt) x0[i] = VT(0);
        });
        cur[k] = 0;
        for (int s = 0; s < a.nu1; ++s) {
            const int c = cur[k];
            run(gwide, [&](int64_t gt, int64_t nt) {
                coop_spmv<VT, AMGT_EPI_JACOBI>(L.A, (const VT*)L.x[c], (VT*)L.x[1 - c], (const VT*)L.b,
                                               (const VT*)L.dinv, (const VT*)L.x[c], a.omega, gt >> 5, nt >> 5, lane);
            });
            cur[k] ^= 1;
        }
        const int c = cur[k];
        run(gwide, [&](int64_t gt, int64_t nt) {
            coop_spmv<VT, AMGT_EPI_RESIDUAL>(L.A, (const VT*)L.x[c], (VT*)L.r, (const VT*)L.b, nullptr, nullptr,
                                             a.omega, gt >> 5, nt >> 5, lane);
        });
        run(gwide, [&](int64_t gt, int64_t nt) {
            coop_spmv<VT, AMGT_EPI_Y>(L.R, (const VT*)L.r, (VT*)a.L[k + 1].b, nullptr, nullptr, nullptr, a.omega,
                                      gt >> 5, nt >> 5, lane);
        });
    }
    run(a.M < a.kb, [&](int64_t gt, int64_t nt) {  // line 6: x_M = A_M^{-1} b_M (dense FP64)
        const CoopLevel& C = a.L[a.M];
        const VT* bM = (const VT*)C.b;
        VT* xM = (VT*)C.x[0];
        for (int64_t row = gt >> 5; row < C.npad; row += nt >> 5) {
            double acc = 0.0;
            if (row < a.nM)
                for (int64_t j = lane; j < a.nM; j += 32) acc = fma(a.Ainv[row * a.nM + j], (double)bM[j], acc);
            for (int d = 16; d; d >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, d);
            if (lane == 0) xM[row] = (VT)acc;
        }
    });
    cur[a.M] = 0;
    for (int k = a.M - 1; k >= a.k0; --k) {  // lines 7-11
        const CoopLevel& L = a.L[k];
        const bool gwide = k < a.kb;
        if (k + 1 == a.kb) gsync();  // leaving the block-local levels: everyone sees CTA 0's result
        const int cn = cur[k + 1], c0 = cur[k];
        run(gwide, [&](int64_t gt, int64_t nt) {
            coop_spmv<VT, AMGT_EPI_ACCUM>(L.P, (const VT*)a.L[k + 1].x[cn], (VT*)L.x[c0], nullptr, nullptr, nullptr,
                                          a.omega, gt >> 5, nt >> 5, lane);
        });
        for (int s = 0; s < a.nu2; ++s) {
            const int c = cur[k];
            run(gwide, [&](int64_t gt, int64_t nt) {
                coop_spmv<VT, AMGT_EPI_JACOBI>(L.A, (const VT*)L.x[c], (VT*)L.x[1 - c], (const VT*)L.b,
                                               (const VT*)L.dinv, (const VT*)L.x[c], a.omega, gt >> 5, nt >> 5, lane);
            });
            cur[k] ^= 1;
        }
    }
    if (a.kb <= a.k0) gsync();  // every level was block-local
}

static CoopMat coop_mat(const amgt_mbsr& M) {
    return CoopMat{M.blc_ptr, M.blc_idx, M.blc_map, M.blc_val, (int)M.prec, M.blc_row};
}

static void fill_coop_args(const amgt_hierarchy* H, int k0, CoopArgs& a) {
    const int M = H->nlev - 1;
    for (int k = k0; k <= M; ++k) {
        const amgt_level& L = H->L[k];
        CoopLevel& c = a.L[k];
        c.A = coop_mat(L.A);
        if (k < M) {
            c.P = coop_mat(L.P);
            c.R = coop_mat(L.R);
        }
        c.b = L.b;
        c.x[0] = L.x;
        c.x[1] = L.t;
        c.r = L.r;
        c.dinv = L.dinv;
        c.npad = L.npad;
    }
    a.k0 = k0;
    a.M = M;
    a.nu1 = H->o.nu1;
    a.nu2 = H->o.nu2;
    a.omega = H->o.omega;
    a.nM = H->nM;
    a.Ainv = H->Ainv;
}

// First level of the tail run by one CTA (k_subcycle<VT, false>): block rows <= TAIL_BR
// (AMGT_TAIL_BLOCKROWS, default 128; 0 disables), every tail level with one vector
// precision and its ping-pong buffers in place; M + 1 = no tail.
static int tail_level(const amgt_hierarchy* H, void** xc, void** xa) {
    static int64_t tail_br = -1;
    if (tail_br < 0) {
        const char* e = getenv("AMGT_TAIL_BLOCKROWS");
        tail_br = e ? atoll(e) : 128;
    }
    const int M = H->nlev - 1;
    if (tail_br == 0 || (H->o.nu1 + H->o.nu2) % 2 != 0 || (timing_mask() & ~1u) != 0) return M + 1;
    int kt = M + 1;
    for (int k = 1; k <= M; ++k)
        if (H->L[k].A.blc_row <= tail_br) { kt = k; break; }
    if (kt > M - 1) return M + 1;  // at least one level above the coarsest
    for (int k = kt; k <= M; ++k)
        if (H->L[k].vprec != H->L[kt].vprec || xc[k] != H->L[k].x || xa[k] != H->L[k].t) return M + 1;
    return kt;
}

// ---------------------------------------------------------------- shared-memory tail
// The tail levels kt..M (a few hundred rows and below) are latency-bound: every Alg. 2 step
// is a handful of dependent L2 round trips whatever the work.  k_tail_smem stages the tail's
// operators (A_k, P_k, R_k in mBSR, D^-1_k, the dense coarsest inverse) and b_kt into the
// shared memory of ONE CTA with independent 16-B loads, runs every step of levels kt..M
// (Alg. 2 lines 1-11) from shared memory with block barriers, and writes x_kt back.  The
// SpMV is one thread per scalar row, walking the block row's tiles in column order with
// the bitmap predicate (Alg. 5 GETBIT) — for FP32/FP16 operators the accumulation order and
// arithmetic of k_spmv_rows, so those levels are bit-identical to the global-memory path.
struct SmMat {
    int64_t ptr, idx, map, val;  // shared-memory byte offsets
    int64_t BR;
    int prec;
};
struct SmLevel {
    SmMat A, P, R;
    int64_t b, x, t, r, dinv;  // byte offsets of the level vectors
    int64_t npad;
};
struct SmSeg {
    const void* src;
    int64_t off, bytes;
};
constexpr int SM_MAXSEG = 48;
struct SmTailArgs {
    SmLevel L[8];
    SmSeg seg[SM_MAXSEG];
    int64_t pre[SM_MAXSEG + 1];  // prefix of the 16-B chunk counts of the segments
    int nseg, kt, M, nu1, nu2;
    double omega;
    int64_t nM, ainv;
    void* xout;  // x_kt in global memory
};

// y_i = epi(i, (A x)_i) for the 4*BR rows of an mBSR operator held in shared memory.  Tiles
// in groups of four: the group's bitmaps, columns and row values are read before its x
// entries (independent shared-memory loads), then accumulated in tile / column order.
template <typename VT, typename F>
__device__ __forceinline__ void sm_spmv(const unsigned char* sm, const SmMat& M, const VT* x, F&& epi) {
    const int64_t* ptr = reinterpret_cast<const int64_t*>(sm + M.ptr);
    const int32_t* idx = reinterpret_cast<const int32_t*>(sm + M.idx);
    const uint16_t* map = reinterpret_cast<const uint16_t*>(sm + M.map);
    constexpr int U = 4, U2 = 2;  // tiles per group (FP32/FP16, FP64)
    for (int64_t i = threadIdx.x; i < 4 * M.BR; i += blockDim.x) {
        const int64_t I = i >> 2;
        const int r = (int)(i & 3);
        const int t0 = (int)ptr[I], t1 = (int)ptr[I + 1];
        if (M.prec == AMGT_FP64) {
            const double* val = reinterpret_cast<const double*>(sm + M.val);
            double acc = 0.0;
            for (int t = t0; t < t1; t += U2) {
                uint32_t nib[U2];
                int J[U2];
                double a[U2][4];
#pragma unroll
                for (int u = 0; u < U2; ++u) {
                    const bool v = t + u < t1;
                    nib[u] = v ? (map[t + u] >> (4 * r)) & 0xFu : 0u;
                    J[u] = v ? idx[t + u] : 0;
                    if (v) {
                        const double2 p0 = reinterpret_cast<const double2*>(val + 16 * (t + u) + 4 * r)[0];
                        const double2 p1 = reinterpret_cast<const double2*>(val + 16 * (t + u) + 4 * r)[1];
                        a[u][0] = p0.x; a[u][1] = p0.y; a[u][2] = p1.x; a[u][3] = p1.y;
                    }
                }
#pragma unroll
                for (int u = 0; u < U2; ++u)
#pragma unroll
                    for (int c = 0; c < 4; ++c)
                        if ((nib[u] >> c) & 1u) acc = fma(a[u][c], (double)x[4 * J[u] + c], acc);
            }
            epi(i, acc);
        } else {
            float acc = 0.f;
            for (int t = t0; t < t1; t += U) {
                uint32_t nib[U];
                int J[U];
                float a[U][4];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const bool v = t + u < t1;
                    nib[u] = v ? (map[t + u] >> (4 * r)) & 0xFu : 0u;
                    J[u] = v ? idx[t + u] : 0;
                    if (v) {
                        if (M.prec == AMGT_FP32) {
                            const float4 w = *reinterpret_cast<const float4*>(sm + M.val + 4 * (16 * (int64_t)(t + u) + 4 * r));
                            a[u][0] = w.x; a[u][1] = w.y; a[u][2] = w.z; a[u][3] = w.w;
                        } else {
                            const uint2 w = *reinterpret_cast<const uint2*>(sm + M.val + 2 * (16 * (int64_t)(t + u) + 4 * r));
                            const float2 lo = __half22float2(*reinterpret_cast<const __half2*>(&w.x));
                            const float2 hi = __half22float2(*reinterpret_cast<const __half2*>(&w.y));
                            a[u][0] = lo.x; a[u][1] = lo.y; a[u][2] = hi.x; a[u][3] = hi.y;
                        }
                    }
                }
#pragma unroll
                for (int u = 0; u < U; ++u)
#pragma unroll
                    for (int c = 0; c < 4; ++c)
                        if ((nib[u] >> c) & 1u) acc = fmaf(a[u][c], (float)x[4 * J[u] + c], acc);
            }
            epi(i, acc);
        }
    }
}

template <typename VT>
__global__ void __launch_bounds__(512) k_tail_smem(const SmTailArgs a) {
    pdl_wait();
    extern __shared__ __align__(16) unsigned char sm[];
    {  // stage: all segments as one flat list of 16-B chunks, four loads in flight per thread
        __shared__ int64_t s_pre[SM_MAXSEG + 1], s_off[SM_MAXSEG];
        __shared__ const void* s_src[SM_MAXSEG];
        for (int k = threadIdx.x; k <= a.nseg; k += blockDim.x) {
            s_pre[k] = a.pre[k];
            if (k < a.nseg) { s_off[k] = a.seg[k].off; s_src[k] = a.seg[k].src; }
        }
        __syncthreads();
        const int64_t n = s_pre[a.nseg];
        for (int64_t c0 = threadIdx.x; c0 < n; c0 += 4 * (int64_t)blockDim.x) {
            uint4 v[4];
            int64_t dst[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const int64_t c = c0 + (int64_t)u * blockDim.x;
                dst[u] = -1;
                if (c < n) {
                    int lo = 0, hi = a.nseg - 1;  // segment: largest s with pre[s] <= c
                    while (lo < hi) {
                        const int mid = (lo + hi + 1) >> 1;
                        if (s_pre[mid] <= c) lo = mid; else hi = mid - 1;
                    }
                    const int64_t k = c - s_pre[lo];
                    v[u] = __ldcg(reinterpret_cast<const uint4*>(s_src[lo]) + k);
                    dst[u] = s_off[lo] + 16 * k;
                }
            }
#pragma unroll
            for (int u = 0; u < 4; ++u)
                if (dst[u] >= 0) *reinterpret_cast<uint4*>(sm + dst[u]) = v[u];
        }
        // remainders (< 16 B, whole 4-B words) of the segments
        for (int s = threadIdx.x; s < a.nseg; s += blockDim.x) {
            const SmSeg g = a.seg[s];
            for (int64_t w = (g.bytes >> 4) << 2; w < (g.bytes >> 2); ++w)
                reinterpret_cast<uint32_t*>(sm + g.off)[w] = __ldcg(reinterpret_cast<const uint32_t*>(g.src) + w);
        }
    }
    __syncthreads();
    const VT om = (VT)a.omega;
    auto V = [&](int64_t off) { return reinterpret_cast<VT*>(sm + off); };
    int64_t xo[8], to[8];  // current / partner buffer of each level
    for (int k = a.kt; k < a.M; ++k) {  // Alg. 2 lines 1-5
        const SmLevel& L = a.L[k];
        xo[k] = L.x;
        to[k] = L.t;
        const VT* b = V(L.b);
        const VT* dv = V(L.dinv);
        if (a.nu1 >= 1) {  // first sweep from x = 0 (the k_jacobi0 expression)
            VT* x = V(xo[k]);
            for (int64_t i = threadIdx.x; i < L.npad; i += blockDim.x) {
                const VT zero = VT(0), t = VT(0);
                x[i] = zero + om * dv[i] * (b[i] - t);
            }
        } else {
            for (int64_t i = threadIdx.x; i < L.npad; i += blockDim.x) V(xo[k])[i] = VT(0);
        }
        __syncthreads();
        for (int s = 1; s < a.nu1; ++s) {
            const VT* x = V(xo[k]);
            VT* y = V(to[k]);
            sm_spmv<VT>(sm, L.A, x, [&](int64_t i, auto v) { y[i] = x[i] + om * dv[i] * (b[i] - (VT)v); });
            __syncthreads();
            const int64_t tmp = xo[k]; xo[k] = to[k]; to[k] = tmp;
        }
        {  // line 3: r = b - A x
            VT* r = V(L.r);
            sm_spmv<VT>(sm, L.A, V(xo[k]), [&](int64_t i, auto v) { r[i] = b[i] - (VT)v; });
        }
        __syncthreads();
        {  // line 4: b_{k+1} = R r
            VT* bn = V(a.L[k + 1].b);
            sm_spmv<VT>(sm, L.R, V(L.r), [&](int64_t i, auto v) { bn[i] = (VT)v; });
        }
        __syncthreads();
    }
    {  // line 6: x_M = A_M^-1 b_M (dense FP64)
        const SmLevel& C = a.L[a.M];
        const VT* bM = V(C.b);
        VT* xM = V(C.x);
        const double* Ai = reinterpret_cast<const double*>(sm + a.ainv);
        xo[a.M] = C.x;
        for (int64_t row = threadIdx.x; row < C.npad; row += blockDim.x) {
            double acc = 0.0;
            if (row < a.nM)
                for (int64_t j = 0; j < a.nM; ++j) acc = fma(Ai[row * a.nM + j], (double)bM[j], acc);
            xM[row] = (VT)acc;
        }
    }
    __syncthreads();
    for (int k = a.M - 1; k >= a.kt; --k) {  // lines 7-11
        const SmLevel& L = a.L[k];
        {  // lines 8-9: x += P x_{k+1}
            VT* x = V(xo[k]);
            sm_spmv<VT>(sm, L.P, V(xo[k + 1]), [&](int64_t i, auto v) { x[i] = x[i] + (VT)v; });
        }
        __syncthreads();
        const VT* b = V(L.b);
        const VT* dv = V(L.dinv);
        for (int s = 0; s < a.nu2; ++s) {  // line 10
            const VT* x = V(xo[k]);
            VT* y = V(to[k]);
            sm_spmv<VT>(sm, L.A, x, [&](int64_t i, auto v) { y[i] = x[i] + om * dv[i] * (b[i] - (VT)v); });
            __syncthreads();
            const int64_t tmp = xo[k]; xo[k] = to[k]; to[k] = tmp;
        }
    }
    VT* out = reinterpret_cast<VT*>(a.xout);
    const VT* xk = V(xo[a.kt]);
    for (int64_t i = threadIdx.x; i < a.L[a.kt].npad; i += blockDim.x) out[i] = xk[i];
}

// Plans the shared-memory tail of levels kt..M; false when it does not fit (or too many
// segments): the caller then uses the global-memory tail kernel.
static bool plan_tail_smem(const amgt_hierarchy* H, int kt, void* xout, SmTailArgs& a, size_t& bytes) {
    static int budget = -1;
    if (budget < 0) {
        int dev = 0, optin = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
        const char* e = getenv("AMGT_TAIL_SMEM");
        budget = e ? atoi(e) : std::min(optin, 200 * 1024);
    }
    if (budget <= 0) return false;
    const int M = H->nlev - 1;
    a = SmTailArgs{};
    int64_t cur = 0;
    auto place = [&](int64_t nb) {
        const int64_t off = (cur + 15) & ~int64_t(15);
        cur = off + nb;
        return off;
    };
    auto stage = [&](const void* src, int64_t nb) -> int64_t {
        const int64_t off = place(nb);
        if (a.nseg < SM_MAXSEG && nb > 0) {
            a.seg[a.nseg] = SmSeg{src, off, nb};
            a.pre[a.nseg + 1] = a.pre[a.nseg] + (nb >> 4);
            ++a.nseg;
        } else if (nb > 0) {
            a.nseg = SM_MAXSEG + 1;  // overflow marker
        }
        return off;
    };
    auto mat = [&](const amgt_mbsr& X) {
        SmMat m{};
        m.BR = X.blc_row;
        m.prec = (int)X.prec;
        m.ptr = stage(X.blc_ptr, (X.blc_row + 1) * 8);
        m.idx = stage(X.blc_idx, X.blc_num * 4);
        m.map = stage(X.blc_map, ((X.blc_num + 1) & ~int64_t(1)) * 2);
        m.val = stage(X.blc_val, 16 * X.blc_num * (int64_t)prec_bytes(X.prec));
        return m;
    };
    const size_t vs = vbytes(H->L[kt].vprec);
    for (int k = kt; k <= M; ++k) {
        const amgt_level& L = H->L[k];
        if (L.vprec != H->L[kt].vprec) return false;
        SmLevel& s = a.L[k];
        s.npad = L.npad;
        const int64_t vb = (int64_t)vs * L.npad;
        s.b = k == kt ? stage(L.b, vb) : place(vb);
        s.x = place(vb);
        s.t = place(vb);
        if (k < M) {
            s.r = place(vb);
            s.dinv = stage(L.dinv, vb);
            s.A = mat(L.A);
            s.P = mat(L.P);
            s.R = mat(L.R);
        }
    }
    a.ainv = stage(H->Ainv, H->nM * H->nM * 8);
    if (a.nseg > SM_MAXSEG || cur > budget) return false;
    a.kt = kt;
    a.M = M;
    a.nu1 = H->o.nu1;
    a.nu2 = H->o.nu2;
    a.omega = H->o.omega;
    a.nM = H->nM;
    a.xout = xout;
    bytes = (size_t)cur;
    return true;
}

static amgt_status subcycle_tail(amgt_hierarchy* H, int kt) {
    {
        SmTailArgs* sa = new SmTailArgs();
        size_t bytes = 0;
        const bool ok = plan_tail_smem(H, kt, H->L[kt].x, *sa, bytes);
        if (ok) {
            const bool f64 = H->L[kt].vprec == AMGT_FP64;
            auto kern = f64 ? k_tail_smem<double> : k_tail_smem<float>;
            AMGT_CUDA(dyn_smem(kern, bytes));
            pdl_launch(kern, dim3(1), dim3(512), bytes, H->s, *sa);
            delete sa;
            AMGT_LAUNCHED();
            H->spmv_calls += (int64_t)(H->nlev - 1 - kt) * (H->o.nu1 + H->o.nu2 + 3);
            return AMGT_OK;
        }
        delete sa;
    }
    CoopArgs a{};
    fill_coop_args(H, kt, a);
    a.kb = kt;
    if (H->L[kt].vprec == AMGT_FP64) pdl_launch(k_subcycle<double, false>, dim3(1), dim3(256), 0, H->s, a);
    else pdl_launch(k_subcycle<float, false>, dim3(1), dim3(256), 0, H->s, a);
    AMGT_LAUNCHED();
    H->spmv_calls += (int64_t)(a.M - kt) * (H->o.nu1 + H->o.nu2 + 3);
    return AMGT_OK;
}

// Returns AMGT_ERR_UNSUPPORTED (caller falls back) when the levels' vector precisions differ
// or a cooperative launch is not possible.
static amgt_status subcycle_coop(amgt_hierarchy* H, void** xc, void** xa) {
    const int M = H->nlev - 1, k0 = 1;
    const amgt_prec vp = H->L[k0].vprec;
    for (int k = k0; k <= M; ++k)
        if (H->L[k].vprec != vp || xc[k] != H->L[k].x || xa[k] != H->L[k].t) return AMGT_ERR_UNSUPPORTED;
    CoopArgs a{};
    fill_coop_args(H, k0, a);
    // first level small enough for one CTA (AMGT_COOP_BLOCKROWS, default 128 block rows)
    static int64_t small_br = -1;
    if (small_br < 0) {
        const char* e = getenv("AMGT_COOP_BLOCKROWS");
        small_br = e ? atoll(e) : 128;
    }
    a.kb = M + 1;
    for (int k = k0; k <= M; ++k)
        if (H->L[k].A.blc_row <= small_br) { a.kb = k; break; }
    static int grid64 = 0, grid32 = 0;
    int& grid = vp == AMGT_FP64 ? grid64 : grid32;
    const void* kern = vp == AMGT_FP64 ? (const void*)k_subcycle<double, true> : (const void*)k_subcycle<float, true>;
    if (grid == 0) {
        int dev = 0, coop = 0, per_sm = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, dev);
        if (!coop || cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 256, 0) != cudaSuccess || per_sm < 1) {
            cudaGetLastError();
            grid = -1;
        } else {
            const char* e = getenv("AMGT_COOP_PER_SM");
            const int want = e ? atoi(e) : 1;
            grid = num_sms() * (per_sm < want ? per_sm : want);
        }
    }
    if (grid < 0) return AMGT_ERR_UNSUPPORTED;
    void* args[] = {&a};
    AMGT_CUDA(cudaLaunchCooperativeKernel(kern, dim3(grid), dim3(256), args, 0, H->s));
    count_launch();
    H->spmv_calls += (int64_t)(M - k0) * (H->o.nu1 + H->o.nu2 + 3);
    return AMGT_OK;
}

// The sub-cycle touches only hierarchy-owned buffers, and with nu1 + nu2 even every level's
// ping-pong pair is back in place after a cycle, so one captured graph serves every cycle of
// every amgt_vcycle call.  Graphs are skipped while per-class timing of the coarse classes is
// enabled (the instrumented profile needs one event pair per launch).
// AMGT_COARSE = graph (default: CUDA graph replay) | coop (persistent cooperative kernel,
// measured equal on config 2) | direct (plain launches).
static int coarse_mode() {
    static int m = -1;
    if (m < 0) {
        const char* e = getenv("AMGT_COARSE");
        m = (e && !strcmp(e, "coop")) ? 0 : (e && !strcmp(e, "direct")) ? 2 : 1;
    }
    return m;
}

static amgt_status subcycle(amgt_hierarchy* H, void** xc, void** xa) {
    const bool usable = !H->graph_failed && ((H->o.nu1 + H->o.nu2) % 2 == 0) && (timing_mask() & ~1u) == 0;
    if (!usable || coarse_mode() == 2) return subcycle_direct(H, xc, xa);
    if (coarse_mode() == 0) {
        const amgt_status st = subcycle_coop(H, xc, xa);
        if (st != AMGT_ERR_UNSUPPORTED) return st;
    }
    cudaStream_t user = H->s;
    if (!H->gexec) {
        if (!H->gs) AMGT_CUDA(cudaStreamCreateWithFlags(&H->gs, cudaStreamNonBlocking));
        void* xc0[8];
        void* xa0[8];
        std::copy(xc, xc + 8, xc0);
        std::copy(xa, xa + 8, xa0);
        const int64_t calls0 = H->spmv_calls, launches0 = amgt_launch_count();
        AMGT_CUDA(cudaStreamSynchronize(user));
        H->s = H->gs;
        cudaGraph_t g = nullptr;
        amgt_status st = AMGT_OK;
        if (cudaStreamBeginCapture(H->gs, cudaStreamCaptureModeThreadLocal) != cudaSuccess) {
            st = AMGT_ERR_CUDA;
        } else {
            st = subcycle_direct(H, xc, xa);
            if (cudaStreamEndCapture(H->gs, &g) != cudaSuccess) st = AMGT_ERR_CUDA;
        }
        H->s = user;
        bool same = std::equal(xc, xc + 8, xc0) && std::equal(xa, xa + 8, xa0);
        if (st == AMGT_OK && same && g && cudaGraphInstantiate(&H->gexec, g, 0) == cudaSuccess) {
            H->sub_calls = H->spmv_calls - calls0;
            H->sub_launches = amgt_launch_count() - launches0;
        } else {
            H->gexec = nullptr;
            H->graph_failed = true;
        }
        if (g) cudaGraphDestroy(g);
        cudaGetLastError();
        H->spmv_calls = calls0;  // the capture executed nothing
        std::copy(xc0, xc0 + 8, xc);
        std::copy(xa0, xa0 + 8, xa);
        if (!H->gexec) return subcycle_direct(H, xc, xa);
    }
    AMGT_CUDA(cudaGraphLaunch(H->gexec, user));  // replayed on the caller's stream (captured on gs)
    H->spmv_calls += H->sub_calls;
    count_launches(H->sub_launches);
    return AMGT_OK;
}

// Level-1 steps of Alg. 2 through amgt_spmv_sweeps (one HBM pass over A_1 for consecutive
// SpMVs): stage s reads bufs[s] and writes bufs[s+1]; SpMV operations counted as in Alg. 2.
static amgt_status sweeps(amgt_hierarchy* H, int n, const int* modes, void* const* bufs, const double* b,
                          double* norm) {
    amgt_level& L0 = H->L[0];
    amgt_sweep_stage st[AMGT_SWEEP_MAX_STAGES];
    for (int i = 0; i < n; ++i) {
        st[i] = amgt_sweep_stage{modes[i], bufs[i], bufs[i + 1]};
        H->spmv_calls += modes[i] == AMGT_SWEEP_JR ? 2 : 1;
    }
    return amgt_spmv_sweeps(H->sw, &L0.A, n, st, b, L0.dinv, H->o.omega, norm, H->s);
}

// V-cycles with nu1 = nu2 = 1 whose level-1 SpMVs run as fused sweeps.  Per cycle c, level 1:
// restriction of r (line 4), levels 2..M (graph replay), interpolation + correction (lines
// 8-9), then ONE pass: post-smoothing of cycle c (line 10) -> pre-smoothing of cycle c+1
// (line 2) with the residual norm of cycle c (L308) -> residual of cycle c+1 (line 3).  The
// first cycle starts with {pre-smoothing + initial residual norm, residual}; the last ends
// with {post-smoothing, residual + norm}.  Three iterate buffers rotate (x, t, u).
static amgt_status vcycle_sweeps(amgt_hierarchy* H, const double* b, double* x, int ncycles, void** xc, void** xa) {
    const int M = H->nlev - 1;
    amgt_level& L0 = H->L[0];
    amgt_level& L1 = H->L[1];
    void* X[3] = {x, L0.t, L0.u};
    int cur = 0;
    auto nx = [&](int k) { return X[(cur + k) % 3]; };
    {
        const int modes[2] = {AMGT_SWEEP_JR, AMGT_SWEEP_R};
        void* bufs[3] = {nx(0), nx(1), L0.r};
        AMGT_TRY(sweeps(H, 2, modes, bufs, b, H->norms));
        cur = (cur + 1) % 3;
    }
    for (int c = 1; c <= ncycles; ++c) {
        AMGT_TRY(counted_spmv(H, &L0.R, L0.r, L0.vprec, L1.b, L1.vprec, 0));  // line 4
        xc[0] = nx(0);
        if (M >= 2) AMGT_TRY(subcycle(H, xc, xa));
        else AMGT_TRY(coarse_solve(H, xc));
        AMGT_TRY(counted_spmv(H, &L0.P, xc[1], L1.vprec, nx(0), L0.vprec, 0, ACC));  // lines 8-9
        if (c < ncycles) {
            const int modes[3] = {AMGT_SWEEP_J, AMGT_SWEEP_JR, AMGT_SWEEP_R};
            void* bufs[4] = {nx(0), nx(1), nx(2), L0.r};
            AMGT_TRY(sweeps(H, 3, modes, bufs, b, H->norms + c));
            cur = (cur + 2) % 3;
        } else {
            const int modes[2] = {AMGT_SWEEP_J, AMGT_SWEEP_RN};
            void* bufs[3] = {nx(0), nx(1), L0.r};
            AMGT_TRY(sweeps(H, 2, modes, bufs, b, H->norms + c));
            cur = (cur + 1) % 3;
        }
    }
    xc[0] = nx(0);
    xa[0] = nx(1);
    return AMGT_OK;
}

// Alg. 2 with the vector steps fused into the SpMV epilogues: each smoothing sweep is one
// kernel (out of place, ping-pong between x and t), the residual one kernel, the
// interpolation + correction one kernel.  SpMV calls are counted exactly as in Alg. 2.
static amgt_status vcycle(amgt_hierarchy* H, const double* b, double* x, int ncycles, double* res_host,
                          int64_t* calls_host) {
    PdlScope pdl;  // solve kernels: programmatic dependent launch
    cudaStream_t s = H->s;
    Alloc a = H->alloc();
    if (ncycles + 1 > H->norms_cap) {
        a.put(H->norms, (size_t)H->norms_cap * sizeof(double));
        H->norms_cap = ncycles + 1;
        H->norms = (double*)a.get((size_t)H->norms_cap * sizeof(double));
        if (!H->norms) return fail(AMGT_ERR_ALLOC, "norm buffer allocation failed");
    }
    const int M = H->nlev - 1;
    amgt_level& L0 = H->L[0];
    H->spmv_calls = 0;
    void* xc[8];   // buffer currently holding x_k
    void* xa[8];   // its ping-pong partner
    xc[0] = x;
    xa[0] = L0.t;
    for (int k = 1; k <= M; ++k) { xc[k] = H->L[k].x; xa[k] = H->L[k].t; }
    // residual norms: ||b - A x_c|| after cycle c is delivered by cycle c+1's first
    // pre-smoothing sweep (same x, same arithmetic); only the last one needs its own SpMV
    const bool fused = M > 0 && H->o.nu1 >= 1 && L0.vprec == AMGT_FP64;
    int ncycles_done = 0;
    if ((!fused || ncycles == 0) && !(H->sw && M > 0 && ncycles > 0)) {
        AMGT_TRY(counted_spmv(H, &L0.A, xc[0], AMGT_FP64, L0.r, AMGT_FP64, 0, RES, b));
        AMGT_TRY(norm_into(H, (const double*)L0.r, L0.npad, H->norms));
    }
    if (M == 0) {
        for (int c = 1; c <= ncycles; ++c) {
            amgt_level tmp = L0;
            tmp.b = (void*)b;
            tmp.x = xc[0];
            AMGT_TRY(dense_solve<double>(H, tmp));
            AMGT_TRY(counted_spmv(H, &L0.A, xc[0], AMGT_FP64, L0.r, AMGT_FP64, 0, RES, b));
            AMGT_TRY(norm_into(H, (const double*)L0.r, L0.npad, H->norms + c));
        }
    }
    if (H->sw && M > 0 && ncycles > 0) {
        AMGT_TRY(vcycle_sweeps(H, b, x, ncycles, xc, xa));
        ncycles_done = ncycles;
    }
    for (int c = ncycles_done + 1; c <= ncycles && M > 0; ++c) {
        AMGT_TRY(down_level(H, 0, b, xc, xa, fused ? H->norms + (c - 1) : nullptr));  // lines 1-5, level 1
        if (M >= 2) AMGT_TRY(subcycle(H, xc, xa));          // levels 2..M (graph replay)
        else AMGT_TRY(coarse_solve(H, xc));
        AMGT_TRY(up_level(H, 0, b, xc, xa));                // lines 7-11 at level 1
        if (!fused || c == ncycles) {                       // residual (L308)
            AMGT_TRY(counted_spmv(H, &L0.A, xc[0], AMGT_FP64, L0.r, AMGT_FP64, 0, RES, b));
            AMGT_TRY(norm_into(H, (const double*)L0.r, L0.npad, H->norms + c));
        }
    }
    if (xc[0] != (void*)x)
        AMGT_CUDA(cudaMemcpyAsync(x, xc[0], L0.npad * sizeof(double), cudaMemcpyDeviceToDevice, s));
    std::vector<double> hn(ncycles + 1);
    int64_t* pin = pinned_slots();
    if (pin && ncycles + 1 <= PIN_COARSE - PIN_NORMS) {  // pinned read-back
        AMGT_CUDA(cudaMemcpyAsync(pin + PIN_NORMS, H->norms, (ncycles + 1) * sizeof(double), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaStreamSynchronize(s));
        memcpy(hn.data(), pin + PIN_NORMS, (ncycles + 1) * sizeof(double));
    } else {
        AMGT_CUDA(cudaMemcpyAsync(hn.data(), H->norms, (ncycles + 1) * sizeof(double), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaStreamSynchronize(s));
    }
    if (res_host)
        for (int c = 0; c <= ncycles; ++c) res_host[c] = std::sqrt(hn[c]);
    if (calls_host) *calls_host = H->spmv_calls;
    return AMGT_OK;
}

// z = M r: one V-cycle (Alg. 2) on A_1 z = r from z = 0, no residual norms.
static amgt_status precond(amgt_hierarchy* H, const double* r, double* z) {
    const int M = H->nlev - 1;
    amgt_level& L0 = H->L[0];
    void* xc[8];
    void* xa[8];
    xc[0] = z;
    xa[0] = L0.t;
    for (int k = 1; k <= M; ++k) { xc[k] = H->L[k].x; xa[k] = H->L[k].t; }
    AMGT_CUDA(cudaMemsetAsync(z, 0, L0.npad * sizeof(double), H->s));
    if (M == 0) {
        amgt_level tmp = L0;
        tmp.b = (void*)r;
        tmp.x = z;
        return dense_solve<double>(H, tmp);
    }
    AMGT_TRY(down_level(H, 0, r, xc, xa));
    if (M >= 2) AMGT_TRY(subcycle(H, xc, xa));
    else AMGT_TRY(coarse_solve(H, xc));
    AMGT_TRY(up_level(H, 0, r, xc, xa));
    if (xc[0] != (void*)z)
        AMGT_CUDA(cudaMemcpyAsync(z, xc[0], L0.npad * sizeof(double), cudaMemcpyDeviceToDevice, H->s));
    return AMGT_OK;
}

// PCG on A_1 preconditioned by one V-cycle per iteration (NEXT-1; PCG is the solve-phase
// consumer named at L92).  Textbook recurrence (r0 = b - A x0, z = M r, p = z, then
// q = A p, alpha = (r,z)/(p,q), x += alpha p, r -= alpha q, z = M r, beta = (r,z)'/(r,z),
// p = z + beta p); every scalar stays on the device (no host round trip per iteration
// unless rtol > 0 asks for an early stop).  res_host[k] = ||r_k||_2, k = 0..iters.
static amgt_status pcg(amgt_hierarchy* H, const double* b, double* x, int maxit, double rtol, double* res_host,
                       int* iters_host, int64_t* calls_host) {
    PdlScope pdl;
    cudaStream_t s = H->s;
    Alloc a = H->alloc();
    amgt_level& L0 = H->L[0];
    if (L0.vprec != AMGT_FP64) return fail(AMGT_ERR_UNSUPPORTED, "amgt_pcg: level-1 vectors must be FP64");
    const int64_t n = L0.npad;
    if (maxit + 1 > H->norms_cap) {
        a.put(H->norms, (size_t)H->norms_cap * sizeof(double));
        H->norms_cap = maxit + 1;
        H->norms = (double*)a.get((size_t)H->norms_cap * sizeof(double));
        if (!H->norms) return fail(AMGT_ERR_ALLOC, "norm buffer allocation failed");
    }
    Scratch<double> r, z, p, q, sc;
    AMGT_TRY(r.init(a, n));
    AMGT_TRY(z.init(a, n));
    AMGT_TRY(p.init(a, n));
    AMGT_TRY(q.init(a, n));
    AMGT_TRY(sc.init(a, 4));  // rz[0], rz[1] (by iteration parity), pq
    H->spmv_calls = 0;
    const unsigned G = (unsigned)num_sms() * 4;
    AMGT_TRY(counted_spmv(H, &L0.A, x, AMGT_FP64, r.p, AMGT_FP64, 0, RES, b));  // r0 = b - A x0
    AMGT_TRY(norm_into(H, r.p, n, H->norms));
    AMGT_TRY(precond(H, r.p, z.p));
    AMGT_CUDA(cudaMemcpyAsync(p.p, z.p, n * sizeof(double), cudaMemcpyDeviceToDevice, s));
    k_dot<<<NORM_BLOCKS, 256, 0, s>>>(n, r.p, z.p, H->partial, sc.p);
    AMGT_LAUNCHED();
    double r0 = 0.0;
    if (rtol > 0.0) {
        AMGT_CUDA(cudaMemcpyAsync(&r0, H->norms, sizeof(double), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaStreamSynchronize(s));
    }
    int it = 0;
    for (int k = 0; k < maxit; ++k) {
        if (rtol > 0.0) {
            double rk = 0.0;
            AMGT_CUDA(cudaMemcpyAsync(&rk, H->norms + k, sizeof(double), cudaMemcpyDeviceToHost, s));
            AMGT_CUDA(cudaStreamSynchronize(s));
            if (std::sqrt(rk) <= rtol * std::sqrt(r0)) break;
        }
        double* rz_old = sc.p + (k & 1);
        double* rz_new = sc.p + ((k + 1) & 1);
        AMGT_TRY(counted_spmv(H, &L0.A, p.p, AMGT_FP64, q.p, AMGT_FP64, 0));  // q = A p
        k_dot<<<NORM_BLOCKS, 256, 0, s>>>(n, p.p, q.p, H->partial, sc.p + 2);
        AMGT_LAUNCHED();
        k_pcg_xr<<<NORM_BLOCKS, 256, 0, s>>>(n, rz_old, sc.p + 2, x, r.p, p.p, q.p, H->partial, H->norms + k + 1);
        AMGT_LAUNCHED();
        AMGT_TRY(precond(H, r.p, z.p));
        k_dot<<<NORM_BLOCKS, 256, 0, s>>>(n, r.p, z.p, H->partial, rz_new);
        AMGT_LAUNCHED();
        k_pcg_p<<<G, 256, 0, s>>>(n, rz_new, rz_old, z.p, p.p);
        AMGT_LAUNCHED();
        it = k + 1;
    }
    std::vector<double> hn(it + 1);
    AMGT_CUDA(cudaMemcpyAsync(hn.data(), H->norms, (it + 1) * sizeof(double), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaStreamSynchronize(s));
    if (res_host)
        for (int k = 0; k <= it; ++k) res_host[k] = std::sqrt(hn[k]);
    if (iters_host) *iters_host = it;
    if (calls_host) *calls_host = H->spmv_calls;
    return AMGT_OK;
}

// ---------------------------------------------------------------- internal: distributed tail
// (dist.cu) The levels a distributed hierarchy agglomerates onto every rank form an ordinary
// hierarchy whose level 0 is a coarse level: created from an operator in its level precision,
// applied as one V-cycle from a zero guess per distributed cycle (Alg. 2 lines 2-10 below the
// agglomeration level).
amgt_status hierarchy_create_tail(const amgt_mbsr* A, const amgt_mbsr* const* P, int nlev, const amgt_vcycle_opts* o,
                                  const amgt_allocator* al, cudaStream_t s, amgt_hierarchy** Hout) {
    amgt_hierarchy* H = new amgt_hierarchy();
    H->o = *o;
    H->s = s;
    H->vec_from_prec = true;
    if (al) { H->al = *al; H->has_al = true; }
    amgt_status st = create(A, P, nlev, o, H);
    if (st != AMGT_OK) {
        destroy(H);
        return st;
    }
    *Hout = H;
    return AMGT_OK;
}

void hierarchy_free(amgt_hierarchy* H) { destroy(H); }

amgt_prec hierarchy_vprec0(const amgt_hierarchy* H) { return H->L[0].vprec; }
int64_t hierarchy_npad0(const amgt_hierarchy* H) { return H->L[0].npad; }

// x = one V-cycle on A_0 x = b from x = 0 (level-0 vector precision); adds its SpMV count.
amgt_status hierarchy_apply(amgt_hierarchy* H, const void* b, void* x, cudaStream_t s, int64_t* calls) {
    H->s = s;
    H->spmv_calls = 0;
    const int M = H->nlev - 1;
    amgt_level& L0 = H->L[0];
    void* xc[8];
    void* xa[8];
    xc[0] = x;
    xa[0] = L0.t;
    for (int k = 1; k <= M; ++k) { xc[k] = H->L[k].x; xa[k] = H->L[k].t; }
    if (M == 0) {
        amgt_level tmp = L0;
        tmp.b = (void*)b;
        tmp.x = x;
        AMGT_TRY(L0.vprec == AMGT_FP64 ? dense_solve<double>(H, tmp) : dense_solve<float>(H, tmp));
        H->spmv_calls = 0;
    } else {
        AMGT_CUDA(cudaMemsetAsync(x, 0, vbytes(L0.vprec) * L0.npad, s));
        AMGT_TRY(down_level(H, 0, b, xc, xa));
        if (M >= 2) AMGT_TRY(subcycle(H, xc, xa));
        else AMGT_TRY(coarse_solve(H, xc));
        AMGT_TRY(up_level(H, 0, b, xc, xa));
        if (xc[0] != x) AMGT_CUDA(cudaMemcpyAsync(x, xc[0], vbytes(L0.vprec) * L0.npad, cudaMemcpyDeviceToDevice, s));
    }
    if (calls) *calls += H->spmv_calls;
    return AMGT_OK;
}

}  // namespace amgt

extern "C" {

amgt_status amgt_hierarchy_create(const amgt_mbsr* A, const amgt_mbsr* const* P, int nlev, const amgt_vcycle_opts* o,
                                  const amgt_allocator* al, void* stream, amgt_hierarchy** Hout) {
    const bool pmis = o && o->interp == AMGT_INTERP_PMIS;
    if (!A || !o || !Hout || nlev < 1 || nlev > 8 || (nlev > 1 && !P && !pmis))
        return fail(AMGT_ERR_ARG, "amgt_hierarchy_create: bad argument");
    if (A->prec != AMGT_FP64) return fail(AMGT_ERR_ARG, "amgt_hierarchy_create: A must be FP64");
    if (A->m != A->n) return fail(AMGT_ERR_ARG, "amgt_hierarchy_create: A must be square");
    for (int k = 0; k < nlev; ++k)
        if (!prec_valid(o->level_prec[k])) return fail(AMGT_ERR_ARG, "bad level precision %d", k);
    for (int k = 0; k + 1 < nlev && !pmis; ++k)
        if (!P[k] || P[k]->prec != AMGT_FP64) return fail(AMGT_ERR_ARG, "P[%d] missing or not FP64", k);
    if (o->nu1 < 0 || o->nu2 < 0) return fail(AMGT_ERR_ARG, "negative sweep count");
    if (o->smoother != AMGT_SMOOTH_JACOBI && o->smoother != AMGT_SMOOTH_L1_JACOBI)
        return fail(AMGT_ERR_ARG, "unknown smoother %d", o->smoother);
    amgt_hierarchy* H = new amgt_hierarchy();
    H->o = *o;
    H->s = (cudaStream_t)stream;
    if (al) { H->al = *al; H->has_al = true; }
    amgt_status st = create(A, P, nlev, o, H);
    if (st != AMGT_OK) {
        destroy(H);
        return st;
    }
    *Hout = H;
    return AMGT_OK;
}

int amgt_hierarchy_nlev(const amgt_hierarchy* H) { return H ? H->nlev : 0; }

amgt_status amgt_hierarchy_level(const amgt_hierarchy* H, int k, const amgt_mbsr** A, const amgt_mbsr** P,
                                 const amgt_mbsr** R) {
    if (!H || k < 0 || k >= H->nlev) return fail(AMGT_ERR_ARG, "amgt_hierarchy_level: bad level");
    if (A) *A = &H->L[k].A;
    if (P) *P = k + 1 < H->nlev ? &H->L[k].P : nullptr;
    if (R) *R = k + 1 < H->nlev ? &H->L[k].R : nullptr;
    return AMGT_OK;
}

amgt_status amgt_vcycle(amgt_hierarchy* H, const double* b, double* x, int ncycles, double* res_norms_host,
                        int64_t* spmv_calls_host, void* stream) {
    if (!H || !b || !x || ncycles < 0) return fail(AMGT_ERR_ARG, "amgt_vcycle: bad argument");
    H->s = (cudaStream_t)stream;
    return vcycle(H, b, x, ncycles, res_norms_host, spmv_calls_host);
}

amgt_status amgt_pcg(amgt_hierarchy* H, const double* b, double* x, int maxit, double rtol, double* res_norms_host,
                     int* iters_host, int64_t* spmv_calls_host, void* stream) {
    if (!H || !b || !x || maxit < 0 || !(rtol >= 0.0)) return fail(AMGT_ERR_ARG, "amgt_pcg: bad argument");
    H->s = (cudaStream_t)stream;
    return pcg(H, b, x, maxit, rtol, res_norms_host, iters_host, spmv_calls_host);
}

amgt_status amgt_dinv(const amgt_mbsr* A, int64_t diag_tile_offset, void* dinv, amgt_prec vprec, void* stream) {
    if (!A || !dinv || (vprec != AMGT_FP64 && vprec != AMGT_FP32)) return fail(AMGT_ERR_ARG, "amgt_dinv: bad argument");
    return dinv_impl(*A, diag_tile_offset, dinv, vprec, (cudaStream_t)stream);
}

amgt_status amgt_dense_spd_inverse(int64_t n, const double* a_host, double* inv_host) {
    if (n < 0 || (n > 0 && (!a_host || !inv_host))) return fail(AMGT_ERR_ARG, "amgt_dense_spd_inverse: bad argument");
    std::vector<double> a(a_host, a_host + n * n), inv;
    if (!dense_inverse(n, a, inv)) return fail(AMGT_ERR_ARG, "matrix is not SPD (Cholesky failed)");
    std::copy(inv.begin(), inv.end(), inv_host);
    return AMGT_OK;
}

amgt_status amgt_dense_matvec(int64_t n, int64_t npad, const double* Ainv, const void* b, void* x, amgt_prec vprec,
                              void* stream) {
    if (n < 0 || npad < n || (vprec != AMGT_FP64 && vprec != AMGT_FP32)) return fail(AMGT_ERR_ARG, "amgt_dense_matvec: bad argument");
    cudaStream_t s = (cudaStream_t)stream;
    if (npad == 0) return AMGT_OK;
    if (vprec == AMGT_FP64)
        k_dense_solve<double><<<(unsigned)ceil_div(npad * 32, 256), 256, 0, s>>>(n, npad, Ainv, (const double*)b, (double*)x);
    else
        k_dense_solve<float><<<(unsigned)ceil_div(npad * 32, 256), 256, 0, s>>>(n, npad, Ainv, (const float*)b, (float*)x);
    AMGT_LAUNCHED();
    return AMGT_OK;
}

amgt_status amgt_norm2sq(int64_t n, const double* r, double* out_dev, void* stream) {
    if (n < 0 || !out_dev || (n > 0 && !r)) return fail(AMGT_ERR_ARG, "amgt_norm2sq: bad argument");
    cudaStream_t s = (cudaStream_t)stream;
    Alloc a{nullptr, s};
    Scratch<double> part;
    AMGT_TRY(part.init(a, NORM_BLOCKS + 1));
    AMGT_CUDA(cudaMemsetAsync(part.p + NORM_BLOCKS, 0, sizeof(double), s));
    k_dot<<<NORM_BLOCKS, 256, 0, s>>>(n, r, r, part.p, out_dev);
    AMGT_LAUNCHED();
    return AMGT_OK;
}

amgt_status amgt_hierarchy_destroy(amgt_hierarchy* H) {
    destroy(H);
    return AMGT_OK;
}

}  // extern "C"
