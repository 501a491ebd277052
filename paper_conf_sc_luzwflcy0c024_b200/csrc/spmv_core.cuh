// spmv_core.cuh — the per-row SpMV device code shared by the SpMV kernels (spmv.cu) and the
// persistent coarse-level V-cycle kernel (vcycle.cu).  See spmv.cu for the design notes.
#pragma once

#include <type_traits>

#include "common.cuh"

namespace amgt {

// ---------------------------------------------------------------- loads
__device__ __forceinline__ double2 ldg_stream(const double2* p) {
    double2 r;
    asm volatile("ld.global.nc.v2.f64 {%0, %1}, [%2];" : "=d"(r.x), "=d"(r.y) : "l"(p));
    return r;
}
__device__ __forceinline__ float4 ldg_stream(const float4* p) {
    float4 r;
    asm volatile("ld.global.nc.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
    return r;
}
__device__ __forceinline__ uint2 ldg_stream(const uint2* p) {
    uint2 r;
    asm volatile("ld.global.nc.v2.u32 {%0, %1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
    return r;
}

// four consecutive elements (16-byte aligned for float, 32-byte for double)
__device__ __forceinline__ void vload4(const double* p, double (&v)[4]) {
    const double2 a = reinterpret_cast<const double2*>(p)[0], b = reinterpret_cast<const double2*>(p)[1];
    v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
}
__device__ __forceinline__ void vload4(const float* p, float (&v)[4]) {
    const float4 a = *reinterpret_cast<const float4*>(p);
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
}
__device__ __forceinline__ void vstore4(double* p, const double (&v)[4]) {
    reinterpret_cast<double2*>(p)[0] = make_double2(v[0], v[1]);
    reinterpret_cast<double2*>(p)[1] = make_double2(v[2], v[3]);
}
__device__ __forceinline__ void vstore4(float* p, const float (&v)[4]) {
    *reinterpret_cast<float4*>(p) = make_float4(v[0], v[1], v[2], v[3]);
}

// x pair (elements 2h, 2h+1 of the 4-segment at 4J) as doubles.
__device__ __forceinline__ double2 x_pair(const double* x, int64_t J, int h) {
    return __ldg(reinterpret_cast<const double2*>(x + 4 * J + 2 * h));
}
__device__ __forceinline__ double2 x_pair(const float* x, int64_t J, int h) {
    float2 f = __ldg(reinterpret_cast<const float2*>(x + 4 * J + 2 * h));
    return make_double2(f.x, f.y);
}
// x quad as floats.
__device__ __forceinline__ float4 x_quad(const float* x, int64_t J) { return __ldg(reinterpret_cast<const float4*>(x + 4 * J)); }
__device__ __forceinline__ float4 x_quad(const double* x, int64_t J) {
    double2 a = __ldg(reinterpret_cast<const double2*>(x + 4 * J));
    double2 b = __ldg(reinterpret_cast<const double2*>(x + 4 * J + 2));
    return make_float4((float)a.x, (float)a.y, (float)b.x, (float)b.y);
}

// Epilogue applied to each (A x)_i (the Alg. 2 vector steps fused into the SpMV, NEXT-1):
//   EPI_Y        y_i = (A x)_i
//   EPI_JACOBI   y_i = xs_i + w dinv_i (b_i - (A x)_i)       (out-of-place weighted Jacobi, R21)
//   EPI_RESIDUAL y_i = b_i - (A x)_i                          (Alg. 2 line 3)
//   EPI_ACCUM    y_i = y_i + (A x)_i                          (interpolation + correction, lines 8-9)
//   EPI_JACOBI_RES  as EPI_JACOBI, and r_i = b_i - (A x)_i   (the residual of the sweep's input:
//                   after a V-cycle it is the Alg. 2 / L308 residual, so the first pre-smoothing
//                   sweep of the next cycle also delivers the previous cycle's residual)
// Vector arithmetic is done in the y precision, as the separate vector kernels did.
// MODE >= 0 fixes the epilogue at compile time (the row kernels); -1 reads `mode` at run time.
template <typename XT, typename YT, int MODE = -1>
struct Epi {
    YT* y;
    const YT* b;
    const YT* dinv;
    const XT* xs;
    YT omega;
    int mode;
    YT* r = nullptr;   // EPI_JACOBI_RES only
    YT* x1 = nullptr;  // EPI_RES_X0 only
    double* nws = nullptr;  // EPI_JACOBI_NORM only
    __device__ __forceinline__ int md() const { return MODE >= 0 ? MODE : mode; }
    // operands of row i, loaded before the tile loop so their latency overlaps it
    struct Pre {
        YT a = YT(0), c = YT(0), d = YT(0);
    };
    __device__ __forceinline__ Pre prefetch(int64_t i) const {
        Pre p;
        switch (md()) {
            case AMGT_EPI_JACOBI:
            case EPI_JACOBI_NORM:
            case AMGT_EPI_JACOBI_RES: p.a = b[i]; p.c = dinv[i]; p.d = (YT)xs[i]; break;
            case AMGT_EPI_RESIDUAL: p.a = b[i]; break;
            case AMGT_EPI_ACCUM: p.a = y[i]; break;
            case EPI_RES_X0: p.a = b[i]; p.c = dinv[i]; break;
            default: break;
        }
        return p;
    }
    // returns b_i - (A x)_i for EPI_JACOBI_NORM (0 otherwise)
    template <typename V>
    __device__ __forceinline__ YT finish(int64_t i, V v, const Pre& p) const {
        const YT t = (YT)v;
        switch (md()) {
            case AMGT_EPI_JACOBI: y[i] = p.d + omega * p.c * (p.a - t); break;
            case EPI_JACOBI_NORM: {
                const YT res = p.a - t;
                y[i] = p.d + omega * p.c * res;
                return res;
            }
            case AMGT_EPI_JACOBI_RES: {
                const YT res = p.a - t;
                y[i] = p.d + omega * p.c * res;
                r[i] = res;
                break;
            }
            case AMGT_EPI_RESIDUAL: y[i] = p.a - t; break;
            case AMGT_EPI_ACCUM: y[i] = p.a + t; break;
            case EPI_RES_X0: {
                y[i] = p.a - t;
                const YT zero = YT(0), t0 = YT(0);
                x1[i] = zero + omega * p.c * (p.a - t0);
                break;
            }
            default: y[i] = t;
        }
        return YT(0);
    }
    // four consecutive rows i0..i0+3 with 16/32-byte vector accesses (all vectors aligned to
    // 4 elements: the caller checks)
    __device__ __forceinline__ void prefetch4(int64_t i0, Pre (&p)[4]) const {
        YT a[4], c[4], d[4];
        switch (md()) {
            case AMGT_EPI_JACOBI:
            case AMGT_EPI_JACOBI_RES:
                vload4(b + i0, a);
                vload4(dinv + i0, c);
                if constexpr (std::is_same<XT, YT>::value) vload4(xs + i0, d);
                else
                    for (int k = 0; k < 4; ++k) d[k] = (YT)xs[i0 + k];
                for (int k = 0; k < 4; ++k) { p[k].a = a[k]; p[k].c = c[k]; p[k].d = d[k]; }
                break;
            case AMGT_EPI_RESIDUAL:
                vload4(b + i0, a);
                for (int k = 0; k < 4; ++k) p[k].a = a[k];
                break;
            case AMGT_EPI_ACCUM:
                vload4(y + i0, a);
                for (int k = 0; k < 4; ++k) p[k].a = a[k];
                break;
            default: break;
        }
    }
    template <typename V>
    __device__ __forceinline__ void finish4(int64_t i0, const V (&v)[4], const Pre (&p)[4]) const {
        YT o[4], rr[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const YT t = (YT)v[k];
            switch (md()) {
                case AMGT_EPI_JACOBI: o[k] = p[k].d + omega * p[k].c * (p[k].a - t); break;
                case AMGT_EPI_JACOBI_RES:
                    rr[k] = p[k].a - t;
                    o[k] = p[k].d + omega * p[k].c * rr[k];
                    break;
                case AMGT_EPI_RESIDUAL: o[k] = p[k].a - t; break;
                case AMGT_EPI_ACCUM: o[k] = p[k].a + t; break;
                default: o[k] = t;
            }
        }
        vstore4(y + i0, o);
        if (md() == AMGT_EPI_JACOBI_RES) vstore4(r + i0, rr);
    }
    __device__ __forceinline__ void apply(int64_t i, double v) const { put(i, (YT)v); }
    __device__ __forceinline__ void apply(int64_t i, float v) const { put(i, (YT)v); }
    __device__ __forceinline__ void put(int64_t i, YT t) const {
        switch (md()) {
            case AMGT_EPI_JACOBI: y[i] = (YT)xs[i] + omega * dinv[i] * (b[i] - t); break;
            case AMGT_EPI_JACOBI_RES: {
                const YT res = b[i] - t;
                y[i] = (YT)xs[i] + omega * dinv[i] * res;
                r[i] = res;
                break;
            }
            case AMGT_EPI_RESIDUAL: y[i] = b[i] - t; break;
            case AMGT_EPI_ACCUM: y[i] = y[i] + t; break;
            default: y[i] = t;
        }
    }
};

// ---------------------------------------------------------------- FP64 tile step
// Lane q of the group: elements e0 = 2q, 2q+1 (row q>>1) and e1 = 8+2q, 9+2q (row 2+(q>>1)),
// columns 2(q&1), 2(q&1)+1.
struct F64Lane {
    double acc0 = 0.0, acc1 = 0.0;
    __device__ __forceinline__ void step(const double* tile, uint32_t mp, double2 xv, int q) {
        const double2 a = ldg_stream(reinterpret_cast<const double2*>(tile) + q);
        const double2 b = ldg_stream(reinterpret_cast<const double2*>(tile) + 4 + q);
        const uint32_t s0 = mp >> (2 * q), s1 = mp >> (8 + 2 * q);
        acc0 = (s0 & 1u) ? fma(a.x, xv.x, acc0) : acc0;
        acc0 = (s0 & 2u) ? fma(a.y, xv.y, acc0) : acc0;
        acc1 = (s1 & 1u) ? fma(b.x, xv.x, acc1) : acc1;
        acc1 = (s1 & 2u) ? fma(b.y, xv.y, acc1) : acc1;
    }
};

// DMMA m8n8k4 (FP64 tensor core) on two tiles: fragA rows 0-3 = tile a, rows 4-7 = tile b;
// fragB cols 0-3 = x_a (every column), cols 4-7 = x_b.  fragC[g][*] for g<4 = (A_a x_a)[g],
// g>=4 = (A_b x_b)[g-4]  ("diagonal of fragY", L228).
__device__ __forceinline__ void dmma_884(double& c0, double& c1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};"
                 : "+d"(c0), "+d"(c1)
                 : "d"(a), "d"(b));
}

// ---------------------------------------------------------------- row kernel
// MatT = double / float / __half; XT, YT = double / float.
// FP64 CUDA-core tile loop, U tiles per iteration: all U tiles' column indices, bitmaps and
// values are requested before any x segment (one dependent round trip per U tiles).
template <int U, typename XT>
__device__ __forceinline__ void f64_tile_loop(F64Lane& L, int64_t t0, int64_t t1, const int32_t* __restrict__ bidx,
                                              const uint16_t* __restrict__ bmap, const double* __restrict__ bval,
                                              const XT* __restrict__ x, int q) {
    for (int64_t t = t0; t < t1; t += U) {
        int32_t J[U];
        uint32_t mp[U];
        double2 a[U], b[U], xv[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const bool v = t + u < t1;
            J[u] = v ? __ldg(bidx + t + u) : 0;
            mp[u] = v ? __ldg(bmap + t + u) : 0u;
            if (v) {
                a[u] = ldg_stream(reinterpret_cast<const double2*>(bval + 16 * (t + u)) + q);
                b[u] = ldg_stream(reinterpret_cast<const double2*>(bval + 16 * (t + u)) + 4 + q);
            } else {
                a[u] = make_double2(0.0, 0.0);
                b[u] = a[u];
            }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) xv[u] = mp[u] ? x_pair(x, J[u], q & 1) : make_double2(0.0, 0.0);
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint32_t s0 = mp[u] >> (2 * q), s1 = mp[u] >> (8 + 2 * q);
            L.acc0 = (s0 & 1u) ? fma(a[u].x, xv[u].x, L.acc0) : L.acc0;
            L.acc0 = (s0 & 2u) ? fma(a[u].y, xv[u].y, L.acc0) : L.acc0;
            L.acc1 = (s1 & 1u) ? fma(b[u].x, xv[u].x, L.acc1) : L.acc1;
            L.acc1 = (s1 & 2u) ? fma(b[u].y, xv[u].y, L.acc1) : L.acc1;
        }
    }
}


// One warp, 8 block rows [I0 + 8*octet, +8): 4-lane group per block row, U tiles per
// iteration, fused epilogue.  (The k_spmv_rows non-tensor-core path, without long rows.)
template <typename MatT, typename XT, typename YT, int MODE, int U>
__device__ __forceinline__ void spmv_octet(int64_t I0, int64_t octet, int64_t BR, const int64_t* __restrict__ bptr,
                                           const int32_t* __restrict__ bidx, const uint16_t* __restrict__ bmap,
                                           const MatT* __restrict__ bval, const XT* __restrict__ x,
                                           const Epi<XT, YT, MODE>& epi, int lane) {
    const int g = lane >> 2, q = lane & 3;
    const int64_t I = I0 + octet * 8 + g;
    int64_t t0 = 0, t1 = 0;
    const bool write = I < BR;
    if (write) {
        t0 = __ldg(bptr + I);
        t1 = __ldg(bptr + I + 1);
    }
    const int64_t out_i = 4 * I + (sizeof(MatT) == 8 ? ((q == 0) ? 0 : (q == 1) ? 2 : (q == 2) ? 1 : 3) : q);
    typename Epi<XT, YT, MODE>::Pre pre;
    if (write) pre = epi.prefetch(out_i);
    if constexpr (sizeof(MatT) == 8) {
        F64Lane L;
        f64_tile_loop<U>(L, t0, t1, bidx, bmap, (const double*)bval, x, q);
        const double s0 = L.acc0 + __shfl_xor_sync(0xffffffffu, L.acc0, 1);
        const double s1 = L.acc1 + __shfl_xor_sync(0xffffffffu, L.acc1, 1);
        if (write) epi.finish(out_i, (q & 1) ? s1 : s0, pre);
    } else {
        float acc = 0.f;
        for (int64_t t = t0; t < t1; t += U) {
            int32_t J[U];
            uint32_t nib[U];
            float4 a[U], xv[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const bool v = t + u < t1;
                J[u] = v ? __ldg(bidx + t + u) : 0;
                nib[u] = v ? (__ldg(bmap + t + u) >> (4 * q)) & 0xFu : 0u;
                a[u] = make_float4(0.f, 0.f, 0.f, 0.f);
                if (v) {
                    if constexpr (sizeof(MatT) == 4) {
                        a[u] = ldg_stream(reinterpret_cast<const float4*>(bval + 16 * (t + u)) + q);
                    } else {
                        const uint2 w = ldg_stream(reinterpret_cast<const uint2*>(bval + 16 * (t + u)) + q);
                        const float2 lo = __half22float2(*reinterpret_cast<const __half2*>(&w.x));
                        const float2 hi = __half22float2(*reinterpret_cast<const __half2*>(&w.y));
                        a[u] = make_float4(lo.x, lo.y, hi.x, hi.y);
                    }
                }
            }
#pragma unroll
            for (int u = 0; u < U; ++u) xv[u] = nib[u] ? x_quad(x, J[u]) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
            for (int u = 0; u < U; ++u) {
                acc = (nib[u] & 1u) ? fmaf(a[u].x, xv[u].x, acc) : acc;
                acc = (nib[u] & 2u) ? fmaf(a[u].y, xv[u].y, acc) : acc;
                acc = (nib[u] & 4u) ? fmaf(a[u].z, xv[u].z, acc) : acc;
                acc = (nib[u] & 8u) ? fmaf(a[u].w, xv[u].w, acc) : acc;
            }
        }
        if (write) epi.finish(out_i, acc, pre);
    }
}

}  // namespace amgt
