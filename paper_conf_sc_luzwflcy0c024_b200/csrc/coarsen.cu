// coarsen.cu — PMIS coarsening and aggregation on the mBSR operator (Alg. 1 line 3, L54; the
// paper's HYPRE settings PMIS, str_thr = 0.25, max_row_sum = 0.8, L300; PMIS [71], L385;
// §8(f) NEXT-2; reading R32 in DESIGN.md).
//
//   strength   S_i = {j != i : -a_ij >= theta max_k(-a_ik)} (empty if that max <= 0 or the row
//              sum exceeds max_row_sum |a_ii|): one 4-lane group per block row, lane r = row
//              4I+r, the strong entries of each tile as a 16-bit mask (the tile's bitmap subset)
//   measure    lambda_i = |S^T_i| + w_i (integer atomics over the strong entries, then the
//              PMIS random weight: an input, or the counter-based generator both sides share)
//   PMIS       rounds of: candidates = undecided points beating every undecided strong
//              neighbour (S u S^T, one pass over the strong entries clearing the loser of each
//              edge); candidates -> C; undecided points with a new C point in S_i -> F
//   aggregates C points numbered in row order (scan); F points join their strongest C neighbour
//              (largest lambda), then the neighbours assigned that way; the rest are singletons
// Every decision is integer or a comparison of identically computed FP64 values, so the result
// equals the oracle's (O10) bit for bit.
#include <algorithm>
#include <vector>

#include "common.cuh"

namespace amgt {
amgt_status csr_to_mbsr_impl(int64_t m, int64_t n, int64_t nnz, const int64_t* rp, const int32_t* ci,
                             const double* v, amgt_prec prec, amgt_mbsr* out, Alloc& a, int64_t coff);
}
using namespace amgt;

namespace {

enum : int8_t { ST_F = 0, ST_C = 1, ST_U = 2 };

template <typename T>
__device__ __forceinline__ double val64(const void* v, int64_t e) {
    return to_f64(reinterpret_cast<const T*>(v)[e]);
}

// strong-entry masks: smap[t] = the bits of tile t that are strong dependencies of their row
template <typename T>
__global__ void k_pmis_strength(int64_t BR, int64_t m, const int64_t* __restrict__ ptr, const int32_t* __restrict__ idx,
                                const uint16_t* __restrict__ map, const T* __restrict__ val, double theta, double mrs,
                                uint16_t* __restrict__ smap) {
    const int64_t gt = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t I = gt >> 2;
    const int r = (int)(gt & 3);
    const unsigned gm = 0xFu << (threadIdx.x & 28);
    if (I >= BR) return;  // whole groups exit together (4 | blockDim)
    const int64_t i = 4 * I + r;
    const int64_t t0 = ptr[I], t1 = ptr[I + 1];
    double mi = 0.0, rs = 0.0, d = 0.0;
    for (int64_t t = t0; t < t1; ++t) {
        const uint32_t nib = (map[t] >> (4 * r)) & 0xFu;
        const int64_t J = idx[t];
        for (int c = 0; c < 4; ++c) {
            if (!((nib >> c) & 1u)) continue;
            const double a = to_f64(val[16 * t + 4 * r + c]);
            rs = rs + a;  // column order, as the oracle
            if (4 * J + c == i) d = a;
            else if (-a > mi) mi = -a;
        }
    }
    const bool ok = i < m && mi > 0.0 && !(mrs < 1.0 && fabs(rs) > mrs * fabs(d));
    for (int64_t t = t0; t < t1; ++t) {
        const uint32_t nib = (map[t] >> (4 * r)) & 0xFu;
        const int64_t J = idx[t];
        uint32_t s = 0;
        if (ok)
            for (int c = 0; c < 4; ++c)
                if (((nib >> c) & 1u) && 4 * J + c != i && -to_f64(val[16 * t + 4 * r + c]) >= theta * mi) s |= 1u << c;
        uint32_t w = s << (4 * r);
        w |= __shfl_xor_sync(gm, w, 1);
        w |= __shfl_xor_sync(gm, w, 2);
        if (r == 0) smap[t] = (uint16_t)w;
    }
}

// iterate the strong entries (i, j) of row i = 4I + r
#define FOR_STRONG(BODY)                                                              \
    for (int64_t t = ptr[I]; t < ptr[I + 1]; ++t) {                                   \
        const uint32_t nib = (smap[t] >> (4 * r)) & 0xFu;                             \
        if (!nib) continue;                                                           \
        const int64_t J4 = 4 * (int64_t)idx[t];                                       \
        for (int c = 0; c < 4; ++c)                                                   \
            if ((nib >> c) & 1u) {                                                    \
                const int64_t j = J4 + c;                                             \
                BODY                                                                  \
            }                                                                         \
    }

__global__ void k_pmis_measure(int64_t BR, const int64_t* __restrict__ ptr, const int32_t* __restrict__ idx,
                               const uint16_t* __restrict__ smap, int32_t* __restrict__ infl) {
    const int64_t gt = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t I = gt >> 2;
    const int r = (int)(gt & 3);
    if (I >= BR) return;
    FOR_STRONG(atomicAdd(infl + j, 1);)
}

// lambda_i = |S^T_i| + w_i; state: F if it influences nobody, else undecided
__global__ void k_pmis_init(int64_t m, const int32_t* __restrict__ infl, const double* __restrict__ wts,
                            unsigned long long seed, int level, double* __restrict__ lam, int8_t* __restrict__ st,
                            unsigned long long* __restrict__ nu) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= m) return;
    double w;
    if (wts) {
        w = wts[i];
    } else {  // the counter-based generator of R32 (the oracle implements the same formula)
        unsigned long long z = seed + 0x9E3779B97F4A7C15ull * (1ull + (unsigned long long)i + ((unsigned long long)level << 40));
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        z = z ^ (z >> 31);
        w = (double)(z >> 11) * (1.0 / 9007199254740992.0);
    }
    lam[i] = (double)infl[i] + w;
    st[i] = infl[i] == 0 ? ST_F : ST_U;
    if (infl[i] != 0) atomicAdd(nu, 1ull);
}

__global__ void k_pmis_cand_init(int64_t m, const int8_t* __restrict__ st, int8_t* __restrict__ cand) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < m) cand[i] = st[i] == ST_U;
}

// across every strong edge between two undecided points the smaller lambda (both on a tie) loses
__global__ void k_pmis_cand_edges(int64_t BR, int64_t m, const int64_t* __restrict__ ptr,
                                  const int32_t* __restrict__ idx, const uint16_t* __restrict__ smap,
                                  const double* __restrict__ lam, const int8_t* __restrict__ st,
                                  int8_t* __restrict__ cand) {
    const int64_t gt = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t I = gt >> 2;
    const int r = (int)(gt & 3);
    const int64_t i = 4 * I + r;
    if (I >= BR || i >= m || st[i] != ST_U) return;
    const double li = lam[i];
    FOR_STRONG({
        if (st[j] == ST_U) {
            const double lj = lam[j];
            if (!(li > lj)) cand[i] = 0;
            if (!(lj > li)) cand[j] = 0;
        }
    })
}

__global__ void k_pmis_newc(int64_t m, const int8_t* __restrict__ cand, int8_t* __restrict__ st,
                            int8_t* __restrict__ newc) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= m) return;
    newc[i] = cand[i];
    if (cand[i]) st[i] = ST_C;
}

// undecided points with a new C point among their strong dependencies -> F; count the rest
__global__ void k_pmis_newf(int64_t BR, int64_t m, const int64_t* __restrict__ ptr, const int32_t* __restrict__ idx,
                            const uint16_t* __restrict__ smap, const int8_t* __restrict__ newc,
                            int8_t* __restrict__ st, unsigned long long* __restrict__ nu) {
    const int64_t gt = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t I = gt >> 2;
    const int r = (int)(gt & 3);
    const int64_t i = 4 * I + r;
    if (I >= BR || i >= m || st[i] != ST_U) return;
    bool f = false;
    FOR_STRONG({
        if (newc[j]) f = true;
    })
    if (f) st[i] = ST_F;
    else atomicAdd(nu, 1ull);
}

__global__ void k_flag(int64_t m, const int8_t* __restrict__ st, int8_t want, const int32_t* __restrict__ agg,
                       int64_t* __restrict__ fl) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= m) return;
    fl[i] = agg ? (agg[i] < 0 ? 1 : 0) : (st[i] == want ? 1 : 0);
}

__global__ void k_agg_roots(int64_t m, const int8_t* __restrict__ st, const int64_t* __restrict__ pos,
                            int32_t* __restrict__ agg) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= m) return;
    agg[i] = st[i] == ST_C ? (int32_t)pos[i] : -1;
}

// F point i joins the aggregate of its best strong dependency j among `eligible` points (largest
// lambda, then smaller j).  pass 0: eligible = C points (agg from `src`); pass 1: F points assigned in
// pass 0 (src = the pass-0 snapshot)
__global__ void k_agg_join(int64_t BR, int64_t m, int pass, const int64_t* __restrict__ ptr,
                           const int32_t* __restrict__ idx, const uint16_t* __restrict__ smap,
                           const double* __restrict__ lam, const int8_t* __restrict__ st,
                           const int32_t* __restrict__ src, int32_t* __restrict__ agg) {
    const int64_t gt = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t I = gt >> 2;
    const int r = (int)(gt & 3);
    const int64_t i = 4 * I + r;
    if (I >= BR || i >= m || st[i] == ST_C || src[i] >= 0) return;
    int64_t best = -1;
    double lb = 0.0;
    FOR_STRONG({
        const bool el = pass == 0 ? st[j] == ST_C : (st[j] != ST_C && src[j] >= 0);
        if (el) {
            const double lj = lam[j];
            if (best < 0 || lj > lb || (lj == lb && j < best)) {
                best = j;
                lb = lj;
            }
        }
    })
    if (best >= 0) agg[i] = src[best];
}

__global__ void k_agg_singletons(int64_t m, int64_t base, const int64_t* __restrict__ pos, int32_t* __restrict__ agg) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= m) return;
    if (agg[i] < 0) agg[i] = (int32_t)(base + pos[i]);
}

__global__ void k_is_c(int64_t m, const int8_t* __restrict__ st, int8_t* __restrict__ out) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < m) out[i] = st[i] == ST_C ? 1 : 0;
}

__global__ void k_pt_csr(int64_t m, const int32_t* __restrict__ agg, int64_t* __restrict__ rp,
                         double* __restrict__ v) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i <= m) rp[i] = i;
    if (i < m) v[i] = 1.0;
    (void)agg;
}

unsigned g256(int64_t n) { return (unsigned)std::max<int64_t>(1, ceil_div(n, 256)); }

int64_t read_i64(const int64_t* d, cudaStream_t s, amgt_status& st) {
    int64_t h = 0;
    int64_t* pin = pinned_slots();
    cudaError_t e;
    if (pin) {
        e = cudaMemcpyAsync(pin + PIN_CREATE + 12, d, 8, cudaMemcpyDeviceToHost, s);
        if (e == cudaSuccess) e = cudaStreamSynchronize(s);
        h = pin[PIN_CREATE + 12];
    } else {
        e = cudaMemcpyAsync(&h, d, 8, cudaMemcpyDeviceToHost, s);
        if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    }
    st = e == cudaSuccess ? AMGT_OK : fail(AMGT_ERR_CUDA, "PMIS read-back: %s", cudaGetErrorString(e));
    return h;
}

}  // namespace

namespace amgt {

amgt_status pmis_aggregate_impl(const amgt_mbsr* A, double theta, double mrs, const double* weights, uint64_t seed,
                                int level, int32_t* agg, int8_t* is_c, int64_t* nagg_host, int* rounds_host, Alloc& a) {
    cudaStream_t s = a.s;
    const int64_t m = A->m, BR = A->blc_row, T = A->blc_num;
    if (A->m != A->n) return fail(AMGT_ERR_ARG, "PMIS: A must be square");
    Scratch<uint16_t> smap;
    Scratch<int32_t> infl, aggA;
    Scratch<double> lam;
    Scratch<int8_t> st, cand, newc;
    Scratch<int64_t> fl, pos;
    Scratch<unsigned long long> nu;
    AMGT_TRY(smap.init(a, T + 1));
    AMGT_TRY(infl.init(a, m + 1));
    AMGT_TRY(aggA.init(a, m + 1));
    AMGT_TRY(lam.init(a, m + 1));
    AMGT_TRY(st.init(a, m + 1));
    AMGT_TRY(cand.init(a, m + 1));
    AMGT_TRY(newc.init(a, m + 1));
    AMGT_TRY(fl.init(a, m + 1));
    AMGT_TRY(pos.init(a, m + 1));
    AMGT_TRY(nu.init(a, 1));
    AMGT_CUDA(cudaMemsetAsync(infl.p, 0, (m + 1) * sizeof(int32_t), s));
    AMGT_CUDA(cudaMemsetAsync(nu.p, 0, sizeof(unsigned long long), s));
    const unsigned gG = g256(4 * BR);
    if (BR > 0) {
        switch (A->prec) {
            case AMGT_FP64:
                k_pmis_strength<double><<<gG, 256, 0, s>>>(BR, m, A->blc_ptr, A->blc_idx, A->blc_map,
                                                           (const double*)A->blc_val, theta, mrs, smap.p);
                break;
            case AMGT_FP32:
                k_pmis_strength<float><<<gG, 256, 0, s>>>(BR, m, A->blc_ptr, A->blc_idx, A->blc_map,
                                                          (const float*)A->blc_val, theta, mrs, smap.p);
                break;
            default:
                k_pmis_strength<__half><<<gG, 256, 0, s>>>(BR, m, A->blc_ptr, A->blc_idx, A->blc_map,
                                                           (const __half*)A->blc_val, theta, mrs, smap.p);
        }
        AMGT_LAUNCHED();
        k_pmis_measure<<<gG, 256, 0, s>>>(BR, A->blc_ptr, A->blc_idx, smap.p, infl.p);
        AMGT_LAUNCHED();
    }
    if (m > 0) {
        k_pmis_init<<<g256(m), 256, 0, s>>>(m, infl.p, weights, (unsigned long long)seed, level, lam.p, st.p, nu.p);
        AMGT_LAUNCHED();
    }
    amgt_status rs = AMGT_OK;
    int64_t undecided = read_i64((const int64_t*)nu.p, s, rs);
    AMGT_TRY(rs);
    int rounds = 0;
    while (undecided > 0) {
        ++rounds;
        if (rounds > 100000) return fail(AMGT_ERR_ARG, "PMIS did not converge");
        k_pmis_cand_init<<<g256(m), 256, 0, s>>>(m, st.p, cand.p);
        AMGT_LAUNCHED();
        k_pmis_cand_edges<<<gG, 256, 0, s>>>(BR, m, A->blc_ptr, A->blc_idx, smap.p, lam.p, st.p, cand.p);
        AMGT_LAUNCHED();
        k_pmis_newc<<<g256(m), 256, 0, s>>>(m, cand.p, st.p, newc.p);
        AMGT_LAUNCHED();
        AMGT_CUDA(cudaMemsetAsync(nu.p, 0, sizeof(unsigned long long), s));
        k_pmis_newf<<<gG, 256, 0, s>>>(BR, m, A->blc_ptr, A->blc_idx, smap.p, newc.p, st.p, nu.p);
        AMGT_LAUNCHED();
        undecided = read_i64((const int64_t*)nu.p, s, rs);
        AMGT_TRY(rs);
    }
    // aggregates: C points in row order, joins (two passes), singletons
    if (m > 0) {
        k_flag<<<g256(m), 256, 0, s>>>(m, st.p, ST_C, nullptr, fl.p);
        AMGT_LAUNCHED();
    }
    AMGT_TRY(scan_exclusive(fl.p, pos.p, m, a, s));
    const int64_t nC = read_i64(pos.p + m, s, rs);
    AMGT_TRY(rs);
    if (m > 0) {
        k_agg_roots<<<g256(m), 256, 0, s>>>(m, st.p, pos.p, agg);
        AMGT_LAUNCHED();
        k_agg_join<<<gG, 256, 0, s>>>(BR, m, 0, A->blc_ptr, A->blc_idx, smap.p, lam.p, st.p, agg, agg);
        AMGT_LAUNCHED();
        AMGT_CUDA(cudaMemcpyAsync(aggA.p, agg, m * sizeof(int32_t), cudaMemcpyDeviceToDevice, s));
        k_agg_join<<<gG, 256, 0, s>>>(BR, m, 1, A->blc_ptr, A->blc_idx, smap.p, lam.p, st.p, aggA.p, agg);
        AMGT_LAUNCHED();
        k_flag<<<g256(m), 256, 0, s>>>(m, st.p, 0, agg, fl.p);
        AMGT_LAUNCHED();
    }
    AMGT_TRY(scan_exclusive(fl.p, pos.p, m, a, s));
    if (m > 0) {
        k_agg_singletons<<<g256(m), 256, 0, s>>>(m, nC, pos.p, agg);
        AMGT_LAUNCHED();
        if (is_c) {
            k_is_c<<<g256(m), 256, 0, s>>>(m, st.p, is_c);
            AMGT_LAUNCHED();
        }
    }
    const int64_t nS = read_i64(pos.p + m, s, rs);
    AMGT_TRY(rs);
    if (nagg_host) *nagg_host = nC + nS;
    if (rounds_host) *rounds_host = rounds;
    return AMGT_OK;
}

// Pt(i, agg_i) = 1 (the tentative interpolation of an aggregation), mBSR in `prec`
amgt_status aggregation_p_impl(int64_t m, int64_t nagg, const int32_t* agg, amgt_prec prec, amgt_mbsr* Pt, Alloc& a) {
    Scratch<int64_t> rp;
    Scratch<double> v;
    AMGT_TRY(rp.init(a, m + 1));
    AMGT_TRY(v.init(a, m + 1));
    k_pt_csr<<<g256(m + 1), 256, 0, a.s>>>(m, agg, rp.p, v.p);
    AMGT_LAUNCHED();
    return csr_to_mbsr_impl(m, nagg, m, rp.p, agg, v.p, prec, Pt, a, 0);
}

}  // namespace amgt

extern "C" {

amgt_status amgt_pmis_aggregate(const amgt_mbsr* A, double theta, double max_row_sum, const double* weights,
                                uint64_t seed, int level, int32_t* agg, int8_t* is_c, int64_t* n_agg_host,
                                int* rounds_host, void* stream) {
    if (!A || (A->m > 0 && !agg) || !n_agg_host) return fail(AMGT_ERR_ARG, "amgt_pmis_aggregate: bad argument");
    Alloc a{nullptr, (cudaStream_t)stream};
    return pmis_aggregate_impl(A, theta, max_row_sum, weights, seed, level, agg, is_c, n_agg_host, rounds_host, a);
}

amgt_status amgt_aggregation_p(int64_t m, int64_t n_agg, const int32_t* agg, amgt_prec prec, amgt_mbsr* Pt,
                               const amgt_allocator* al, void* stream) {
    if (m < 0 || n_agg < 0 || (m > 0 && !agg) || !Pt || !prec_valid(prec))
        return fail(AMGT_ERR_ARG, "amgt_aggregation_p: bad argument");
    Alloc a{al, (cudaStream_t)stream};
    return aggregation_p_impl(m, n_agg, agg, prec, Pt, a);
}

}  // extern "C"
