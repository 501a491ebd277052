// interp.cu — interpolation through one SpGEMM call (Alg. 1 line 4, L54; [35] L385; §8(f)
// NEXT-2), reading R31: smoothed aggregation P = (I - w D_F^-1 A_F) Pt, where
//   A_F  = the strength-filtered operator: off-diagonal a_ij is strong iff
//          -a_ij >= theta * max_{k != i}(-a_ik) > 0 (classical strength, str_thr = theta, L300);
//          weak entries are removed from the structure and added to the diagonal (ascending
//          column order, so the row sums are kept);
//   Pt   = the tentative interpolation (fixed aggregation, reading R19);
//   T    = A_F Pt by the mBSR SpGEMM (binning, two-step symbolic, numeric: spgemm.cu);
//   P_ij = Pt_ij - (w / (A_F)_ii) T_ij on T's structure (two roundings, no FMA contraction).
// Kernels:
//   k_filter<PASS>  4-lane group per block row, lane r = scalar row r.  Pass 0 counts the tiles
//                   that keep a bit; pass 1 writes them (tile columns, bitmaps, values with the
//                   lumped diagonal) and s_i = w / d_i.  Both passes recompute the same masks.
//   k_sa_combine    thread per tile of T: finds the Pt tile of the same (I, J) and rewrites the
//                   16 values in place.
#include <cstdint>

#include "common.cuh"

namespace amgt {

amgt_status mbsr_alloc(amgt_mbsr* M, int64_t m, int64_t n, int64_t T, amgt_prec prec, Alloc& a, bool structure,
                       bool values, int64_t* existing_ptr);
amgt_status mbsr_release(amgt_mbsr* M, Alloc& a);
amgt_status spgemm_symbolic_impl(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* Cout, amgt_spgemm_info* info,
                                 Alloc& a);
amgt_status spgemm_numeric_impl(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* C, Alloc& a);

template <typename T> struct FiltAcc { using type = float; };  // lumping arithmetic
template <> struct FiltAcc<double> { using type = double; };

template <typename T> __device__ __forceinline__ typename FiltAcc<T>::type facc(T v);
template <> __device__ __forceinline__ double facc<double>(double v) { return v; }
template <> __device__ __forceinline__ float facc<float>(float v) { return v; }
template <> __device__ __forceinline__ float facc<__half>(__half v) { return __half2float(v); }

// Strong-connection mask of row r (lane) for one tile: bit c set when entry (r, c) of the
// tile is kept (the diagonal always is).
// (strong iff the row has a negative off-diagonal, mx > 0, and -a_ij >= theta * mx)
template <typename T>
__device__ __forceinline__ uint32_t keep_nibble(const T* tile, uint32_t nib, int r, int64_t J, int64_t I, bool anyneg,
                                                typename FiltAcc<T>::type thr) {
    uint32_t keep = 0;
#pragma unroll
    for (int c = 0; c < 4; ++c) {
        if (!(nib & (1u << c))) continue;
        const bool diag = 4 * J + c == 4 * I + r;
        const auto v = facc(tile[4 * r + c]);
        if (diag || (anyneg && -v >= thr)) keep |= 1u << c;
    }
    return keep;
}

// PASS 0: cnt[I] = kept tiles of block row I.  PASS 1: write A_F's tiles from out_ptr[I] and
// s[i] = w / d_i.  flag |= 1 when a row drops entries but has no diagonal entry.
template <typename T, typename S, int PASS>
__global__ void __launch_bounds__(256) k_filter(int64_t BR, int64_t m, const int64_t* __restrict__ bptr,
                                                const int32_t* __restrict__ bidx, const uint16_t* __restrict__ bmap,
                                                const T* __restrict__ bval, double theta, double omega,
                                                int64_t* __restrict__ cnt, const int64_t* __restrict__ out_ptr,
                                                int32_t* __restrict__ oidx, uint16_t* __restrict__ omap,
                                                T* __restrict__ oval, S* __restrict__ s_out,
                                                uint32_t* __restrict__ flag) {
    using A = typename FiltAcc<T>::type;
    const int lane = threadIdx.x & 31, r = lane & 3;
    const unsigned gm = 0xFu << (lane & ~3);
    const int64_t I = (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 2);
    if ((((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5) * 8 >= BR) return;  // whole warp out of range
    const bool valid = I < BR;
    int64_t t0 = 0, t1 = 0;
    if (valid) {
        t0 = bptr[I];
        t1 = bptr[I + 1];
    }
    const int64_t i = 4 * I + r;
    // max_{k != i} (-a_ik) over the row
    A mx = A(0);
    for (int64_t t = t0; t < t1; ++t) {
        const uint32_t nib = (bmap[t] >> (4 * r)) & 0xFu;
        const int64_t J = bidx[t];
#pragma unroll
        for (int c = 0; c < 4; ++c)
            if ((nib & (1u << c)) && 4 * J + c != i) {
                const A v = -facc(bval[16 * t + 4 * r + c]);
                mx = v > mx ? v : mx;
            }
    }
    const bool anyneg = mx > A(0);
    const A thr = (A)theta * mx;
    if (PASS == 0) {
        int64_t kept = 0;
        bool dropped = false, hasdiag = false;
        for (int64_t t = t0; t < t1; ++t) {
            const uint32_t nib = (bmap[t] >> (4 * r)) & 0xFu;
            const int64_t J = bidx[t];
            const uint32_t k = keep_nibble(bval + 16 * t, nib, r, J, I, anyneg, thr);
            dropped |= (k != nib);
            if (J == I && (nib & (1u << r))) hasdiag = true;
            const uint32_t any = __reduce_or_sync(gm, k);  // group: does the tile keep a bit
            kept += any ? 1 : 0;
        }
        if (valid && r == 0) cnt[I] = kept;
        if (valid && i < m && dropped && !hasdiag) atomicOr(flag, 1u);
        return;
    }
    // PASS 1
    int64_t o = valid ? out_ptr[I] : 0;
    A d = A(0);
    bool hasdiag = false;
    // diagonal value first (lumping starts from a_ii), then the weak entries in column order
    for (int64_t t = t0; t < t1; ++t) {
        const uint32_t nib = (bmap[t] >> (4 * r)) & 0xFu;
        if (bidx[t] == I && (nib & (1u << r))) {
            d = facc(bval[16 * t + 5 * r]);
            hasdiag = true;
        }
    }
    for (int64_t t = t0; t < t1; ++t) {
        const uint32_t nib = (bmap[t] >> (4 * r)) & 0xFu;
        const int64_t J = bidx[t];
        const uint32_t k = keep_nibble(bval + 16 * t, nib, r, J, I, anyneg, thr);
#pragma unroll
        for (int c = 0; c < 4; ++c)
            if ((nib & ~k) & (1u << c)) d = d + facc(bval[16 * t + 4 * r + c]);
    }
    for (int64_t t = t0; t < t1; ++t) {
        const uint32_t nib = (bmap[t] >> (4 * r)) & 0xFu;
        const int64_t J = bidx[t];
        const uint32_t k = keep_nibble(bval + 16 * t, nib, r, J, I, anyneg, thr);
        const uint32_t tm = __reduce_or_sync(gm, k << (4 * r));
        if (!tm) continue;
        if (r == 0) {
            oidx[o] = (int32_t)J;
            omap[o] = (uint16_t)tm;
        }
#pragma unroll
        for (int c = 0; c < 4; ++c) {
            T v = T(0.0f);
            if (k & (1u << c)) v = (4 * J + c == i) ? from_acc<T>(d) : bval[16 * t + 4 * r + c];
            oval[16 * o + 4 * r + c] = v;
        }
        ++o;
    }
    if (valid) {
        const A dd = hasdiag ? d : A(0);
        s_out[i] = (S)(dd != A(0) ? (A)omega / dd : A(0));
    }
}

template <typename T> __device__ __forceinline__ T sa_value(T pt, T s, T t);
template <> __device__ __forceinline__ double sa_value<double>(double pt, double s, double t) {
    return __dsub_rn(pt, __dmul_rn(s, t));
}
template <> __device__ __forceinline__ float sa_value<float>(float pt, float s, float t) {
    return __fsub_rn(pt, __fmul_rn(s, t));
}

// In place on T = A_F Pt: T_ij <- Pt_ij - s_i T_ij (Pt_ij = 0 where Pt has no entry).
template <typename T, typename S>
__global__ void __launch_bounds__(256) k_sa_combine(int64_t BR, const int64_t* __restrict__ tptr,
                                                    const int32_t* __restrict__ tidx, const uint16_t* __restrict__ tmap,
                                                    T* __restrict__ tval, const int64_t* __restrict__ pptr,
                                                    const int32_t* __restrict__ pidx, const T* __restrict__ pval,
                                                    const S* __restrict__ s) {
    const int64_t I = (int64_t)blockIdx.x * blockDim.y + threadIdx.y;  // block row
    if (I >= BR) return;
    for (int64_t t = tptr[I] + threadIdx.x; t < tptr[I + 1]; t += blockDim.x) {
        const int32_t J = tidx[t];
        int64_t pt = -1;
        for (int64_t q = pptr[I]; q < pptr[I + 1]; ++q)
            if (pidx[q] == J) { pt = q; break; }
        const uint32_t mp = tmap[t];
#pragma unroll
        for (int e = 0; e < 16; ++e) {
            if (!(mp & (1u << e))) continue;
            const int rr = e >> 2;
            using C = typename FiltAcc<T>::type;
            const C pv = pt >= 0 ? facc(pval[16 * pt + e]) : C(0);
            const C sv = (C)s[4 * I + rr];
            const C tv = facc(tval[16 * t + e]);
            tval[16 * t + e] = from_acc<T>(sa_value<C>(pv, sv, tv));
        }
    }
}

// A_F and s (w / d_i, vector precision S) from A.
template <typename T, typename S>
static amgt_status filter_impl(const amgt_mbsr* A, double theta, double omega, amgt_mbsr* AF, S* s_out, Alloc& a) {
    cudaStream_t s = a.s;
    const int64_t BR = A->blc_row;
    Scratch<int64_t> cnt;
    Scratch<uint32_t> flag;
    AMGT_TRY(cnt.init(a, BR + 1));
    AMGT_TRY(flag.init(a, 1));
    AMGT_CUDA(cudaMemsetAsync(flag.p, 0, sizeof(uint32_t), s));
    const unsigned blocks = (unsigned)ceil_div(ceil_div(BR, 8) * 32, 256);
    if (BR > 0) {
        k_filter<T, S, 0><<<blocks, 256, 0, s>>>(BR, A->m, A->blc_ptr, A->blc_idx, A->blc_map, (const T*)A->blc_val,
                                                 theta, omega, cnt.p, nullptr, nullptr, nullptr, nullptr, nullptr,
                                                 flag.p);
        AMGT_LAUNCHED();
    }
    amgt_mbsr M{};
    M.blc_ptr = (int64_t*)a.get((BR + 1) * sizeof(int64_t));
    if (!M.blc_ptr) return fail(AMGT_ERR_ALLOC, "filter: row pointer allocation failed");
    AMGT_TRY(scan_exclusive(cnt.p, M.blc_ptr, BR, a, s));
    int64_t TF = 0;
    uint32_t hflag = 0;
    AMGT_CUDA(cudaMemcpyAsync(&TF, M.blc_ptr + BR, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaMemcpyAsync(&hflag, flag.p, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaStreamSynchronize(s));
    if (hflag) {
        a.put(M.blc_ptr, (BR + 1) * sizeof(int64_t));
        return fail(AMGT_ERR_ARG, "strength filter: a row with weak entries has no diagonal entry to lump into");
    }
    amgt_status st = mbsr_alloc(&M, A->m, A->n, TF, A->prec, a, true, true, M.blc_ptr);
    if (st != AMGT_OK) { mbsr_release(&M, a); return st; }
    if (BR > 0) {
        k_filter<T, S, 1><<<blocks, 256, 0, s>>>(BR, A->m, A->blc_ptr, A->blc_idx, A->blc_map, (const T*)A->blc_val,
                                                 theta, omega, nullptr, M.blc_ptr, M.blc_idx, M.blc_map,
                                                 (T*)M.blc_val, s_out, flag.p);
        AMGT_LAUNCHED();
    }
    *AF = M;
    return AMGT_OK;
}

template <typename T, typename S>
static amgt_status combine_impl(amgt_mbsr* Tm, const amgt_mbsr* Pt, const S* sv, cudaStream_t s) {
    const int64_t BR = Tm->blc_row;
    if (BR == 0) return AMGT_OK;
    const dim3 block(32, 8);
    k_sa_combine<T, S><<<(unsigned)ceil_div(BR, 8), block, 0, s>>>(BR, Tm->blc_ptr, Tm->blc_idx, Tm->blc_map,
                                                                  (T*)Tm->blc_val, Pt->blc_ptr, Pt->blc_idx,
                                                                  (const T*)Pt->blc_val, sv);
    AMGT_LAUNCHED();
    return AMGT_OK;
}

static amgt_status check_sa_args(const amgt_mbsr* A, const amgt_mbsr* Pt) {
    if (!A || !Pt) return fail(AMGT_ERR_ARG, "null matrix");
    if (A->m != A->n) return fail(AMGT_ERR_ARG, "interpolation: A must be square");
    if (Pt->m != A->m) return fail(AMGT_ERR_ARG, "interpolation: Pt has %lld rows, A %lld", (long long)Pt->m,
                                   (long long)A->m);
    if (Pt->prec != A->prec) return fail(AMGT_ERR_ARG, "interpolation: Pt and A precisions differ");
    return AMGT_OK;
}

// P = SA(A, Pt) in A's precision (lumping and the combine in FP64 for FP64 operators, FP32
// otherwise).
amgt_status sa_interp_impl(const amgt_mbsr* A, const amgt_mbsr* Pt, double theta, double omega, amgt_mbsr* P,
                           Alloc& a) {
    AMGT_TRY(check_sa_args(A, Pt));
    amgt_mbsr AF{};
    const int64_t n = 4 * A->blc_row;
    amgt_status st = AMGT_OK;
    if (A->prec == AMGT_FP64) {
        Scratch<double> sv;
        AMGT_TRY(sv.init(a, n > 0 ? n : 1));
        AMGT_TRY((filter_impl<double, double>(A, theta, omega, &AF, sv.p, a)));
        amgt_mbsr Tm{};
        st = spgemm_symbolic_impl(&AF, Pt, &Tm, nullptr, a);
        if (st == AMGT_OK) st = spgemm_numeric_impl(&AF, Pt, &Tm, a);
        if (st == AMGT_OK) st = combine_impl<double, double>(&Tm, Pt, sv.p, a.s);
        mbsr_release(&AF, a);
        if (st != AMGT_OK) { mbsr_release(&Tm, a); return st; }
        *P = Tm;
    } else {
        Scratch<float> sv;
        AMGT_TRY(sv.init(a, n > 0 ? n : 1));
        if (A->prec == AMGT_FP32) AMGT_TRY((filter_impl<float, float>(A, theta, omega, &AF, sv.p, a)));
        else AMGT_TRY((filter_impl<__half, float>(A, theta, omega, &AF, sv.p, a)));
        amgt_mbsr Tm{};
        st = spgemm_symbolic_impl(&AF, Pt, &Tm, nullptr, a);
        if (st == AMGT_OK) st = spgemm_numeric_impl(&AF, Pt, &Tm, a);
        if (st == AMGT_OK)
            st = A->prec == AMGT_FP32 ? combine_impl<float, float>(&Tm, Pt, sv.p, a.s)
                                      : combine_impl<__half, float>(&Tm, Pt, sv.p, a.s);
        mbsr_release(&AF, a);
        if (st != AMGT_OK) { mbsr_release(&Tm, a); return st; }
        *P = Tm;
    }
    return AMGT_OK;
}

}  // namespace amgt

using namespace amgt;

extern "C" {

amgt_status amgt_strength_filter(const amgt_mbsr* A, double theta, double omega, amgt_mbsr* AF, void* s_out,
                                 const amgt_allocator* al, void* stream) {
    if (!A || !AF || !s_out) return fail(AMGT_ERR_ARG, "amgt_strength_filter: null argument");
    if (A->m != A->n) return fail(AMGT_ERR_ARG, "amgt_strength_filter: A must be square");
    Alloc a{al, (cudaStream_t)stream};
    switch (A->prec) {
        case AMGT_FP64: return filter_impl<double, double>(A, theta, omega, AF, (double*)s_out, a);
        case AMGT_FP32: return filter_impl<float, float>(A, theta, omega, AF, (float*)s_out, a);
        default: return filter_impl<__half, float>(A, theta, omega, AF, (float*)s_out, a);
    }
}

amgt_status amgt_sa_interp(const amgt_mbsr* A, const amgt_mbsr* Pt, double theta, double omega, amgt_mbsr* P,
                           const amgt_allocator* al, void* stream) {
    if (!P) return fail(AMGT_ERR_ARG, "amgt_sa_interp: null output");
    Alloc a{al, (cudaStream_t)stream};
    return sa_interp_impl(A, Pt, theta, omega, P, a);
}

}  // extern "C"
