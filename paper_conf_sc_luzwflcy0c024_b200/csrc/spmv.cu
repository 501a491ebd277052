// spmv.cu — y = A x over mBSR (§IV.D; Alg. 5; Fig. 5).
//
// B200 design (HBM-bound: 134 B per FP64 tile, <=1 flop/B):
//  * Row kernel: a 4-lane group owns one block row, 8 block rows per warp (no cross-group
//    reduction).  Per tile, each lane issues 128-bit loads only: FP64 lane q loads the
//    16-B halves {16q, 64+16q} of the 128-B tile (so every load instruction of the
//    group covers one contiguous 64-B span) plus one 16-B x segment; FP32 lane q loads
//    its row (16 B); FP16 lane q loads its row (8 B).  Each lane multiplies only the
//    entries whose bitmap bit is set (Alg. 5 lines 9-11, GETBIT).  FP64: 8 tiles per
//    iteration (all indices/bitmaps/values requested before the x gathers: one dependent
//    round trip per 8 tiles) under a 64-register budget (4 blocks of 256 per SM).
//  * Load balancing (L220, Fig. 5): with a plan (amgt_spmv_analyze), block rows longer
//    than WARP_CAPACITY = 64 tiles are split into 64-tile warp chunks (8 groups x 8
//    tiles, Alg. 5 lines 4-6 with reading R12); each chunk reduces its 8 groups with
//    shuffles and writes a partial; a combine kernel sums the partials of a row in chunk
//    order (deterministic, no atomics).
//  * Tensor-core route (L222-228, R14): tiles with popcount >= the SpMV threshold are
//    multiplied with DMMA m8n8k4 two at a time inside the row kernel (FP64 only).  Off by
//    default on B200 (DMMA rate == DFMA rate), enabled by
//    amgt_set_tc_threshold.
#include <algorithm>
#include <climits>
#include <type_traits>
#include <cstdlib>

#include <mutex>
#include <unordered_map>

#include "common.cuh"
#include "spmv_core.cuh"

namespace amgt {

// resident 256-thread CTAs per SM of a kernel, queried once per kernel (the level-1 SpMVs of the
// V-cycle loop are launched directly: no host-side occupancy query per launch)
static int occupancy_256(const void* kern) {
    static std::mutex mu;
    static std::unordered_map<const void*, int> cache;
    std::lock_guard<std::mutex> lk(mu);
    auto it = cache.find(kern);
    if (it != cache.end()) return it->second;
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 256, 0) != cudaSuccess) {
        cudaGetLastError();
        per_sm = 0;
    }
    cache[kern] = per_sm;
    return per_sm;
}


constexpr int WARP_CAPACITY = 64;  // tiles per warp chunk (L220)

struct SpmvPlan {
    int64_t nlong = 0, nchunks = 0;
    int32_t* long_rows = nullptr;  // [nlong]
    int64_t* chunk_ptr = nullptr;  // [nlong+1]
    int32_t* chunk_lr = nullptr;   // [nchunks] -> index into long_rows
    double* partial = nullptr;     // [nchunks*4] (double or float accumulators)
    amgt_spmv_stats st{};
    bool stats_ready = false;  // st computed (the fast path defers it to amgt_spmv_get_stats)
    double mean_row = 0.0;     // tiles per block row
};

void spmv_plan_free(void* aux, Alloc& a) {
    SpmvPlan* p = (SpmvPlan*)aux;
    if (!p) return;
    a.put(p->long_rows, p->nlong * sizeof(int32_t));
    a.put(p->chunk_ptr, (p->nlong + 1) * sizeof(int64_t));
    a.put(p->chunk_lr, p->nchunks * sizeof(int32_t));
    a.put(p->partial, p->nchunks * 4 * sizeof(double));
    delete p;
}

// One warp, row octet `wid` (block rows I0 + 8 wid + g, one 4-lane group each).
template <typename MatT, typename XT, typename YT, int MODE, int U, bool TC>
__device__ __forceinline__ void spmv_rows_octet(int64_t wid, int64_t I0, int64_t BR, const int64_t* __restrict__ bptr,
                                                const int32_t* __restrict__ bidx, const uint16_t* __restrict__ bmap,
                                                const MatT* __restrict__ bval, const XT* __restrict__ x,
                                                const Epi<XT, YT, MODE>& epi, int64_t long_thr, int tc_thr) {
    const int lane = threadIdx.x & 31, g = lane >> 2, q = lane & 3;
    const int64_t I = I0 + wid * 8 + g;  // block rows [I0, BR)
    int64_t t0 = 0, t1 = 0;
    bool write = false;
    if (I < BR) {
        t0 = __ldg(bptr + I);
        t1 = __ldg(bptr + I + 1);
        write = t1 - t0 <= long_thr;
        if (!write) t1 = t0;  // long row: handled by the chunk kernel
    }
    // output element of this lane (FP64 layout: rows {0,2,1,3} for q = 0..3)
    const int64_t out_i = 4 * I + (sizeof(MatT) == 8 ? ((q == 0) ? 0 : (q == 1) ? 2 : (q == 2) ? 1 : 3) : q);
    typename Epi<XT, YT, MODE>::Pre pre;
    if (write) pre = epi.prefetch(out_i);
    if constexpr (sizeof(MatT) == 8) {
        F64Lane L;
        if constexpr (!TC) {
            f64_tile_loop<U>(L, t0, t1, bidx, bmap, (const double*)bval, x, q);
        } else {
            // Per-tile routing: each iteration the 8 groups hold one tile each; tiles with
            // popcount >= tc_thr are paired and multiplied with DMMA, the rest use CUDA cores.
            const int64_t len = t1 - t0;
            int64_t maxlen = len;
#pragma unroll
            for (int d = 4; d < 32; d <<= 1) maxlen = max(maxlen, __shfl_xor_sync(0xffffffffu, maxlen, d));
            double tcacc = 0.0;  // lane q of group g: row q contribution from the TC route
            for (int64_t k = 0; k < maxlen; ++k) {
                const bool have = k < len;
                const int64_t t = t0 + k;
                const uint32_t mp = have ? __ldg(bmap + t) : 0u;
                const int32_t J = have ? __ldg(bidx + t) : 0;
                const bool dense = have && __popc(mp) >= tc_thr;
                if (have && !dense) L.step((const double*)bval + 16 * t, mp, x_pair(x, J, q & 1), q);
                uint32_t dm = __ballot_sync(0xffffffffu, dense && q == 0);  // bit 4g per dense group
                while (dm) {
                    const int ga = __ffs(dm) - 1;
                    dm &= dm - 1;
                    int gb = -1;
                    if (dm) { gb = __ffs(dm) - 1; dm &= dm - 1; }
                    const int gA = ga >> 2, gB = gb >= 0 ? (gb >> 2) : -1;
                    // fragment coordinates: lane = 4*row8 + k4 for A (row row8, col k4);
                    // B: row k4, col row8.
                    const int row8 = lane >> 2, k4 = lane & 3;
                    const int src = row8 < 4 ? gA : gB;  // tile owner for this lane's A element
                    const int64_t ta = __shfl_sync(0xffffffffu, t, 4 * gA);
                    const int64_t tb = gB >= 0 ? __shfl_sync(0xffffffffu, t, 4 * gB) : ta;
                    const int32_t Ja = __shfl_sync(0xffffffffu, J, 4 * gA);
                    const int32_t Jb = gB >= 0 ? __shfl_sync(0xffffffffu, J, 4 * gB) : Ja;
                    const uint32_t ma = __shfl_sync(0xffffffffu, mp, 4 * gA);
                    const uint32_t mb = gB >= 0 ? __shfl_sync(0xffffffffu, mp, 4 * gB) : 0u;
                    double av = 0.0, bv = 0.0;
                    if (src >= 0) {
                        const int64_t tt = row8 < 4 ? ta : tb;
                        const uint32_t mm = row8 < 4 ? ma : mb;
                        const int e = 4 * (row8 & 3) + k4;
                        av = ((mm >> e) & 1u) ? ((const double*)bval)[16 * tt + e] : 0.0;
                    }
                    {
                        const bool first = row8 < 4;
                        const int32_t JJ = first ? Ja : Jb;
                        if (first || gB >= 0) bv = (double)x[4 * (int64_t)JJ + k4];
                    }
                    double c0 = 0.0, c1 = 0.0;
                    dmma_884(c0, c1, av, bv);
                    // C[row8][2*k4'] lives in lane 4*row8 + k4'; column 0 of rows 0-3 -> tile a,
                    // column 4 of rows 4-7 -> tile b.  Lane (gA, q) takes row q of tile a.
                    const double ya = __shfl_sync(0xffffffffu, c0, 4 * q + 0);
                    const double yb = __shfl_sync(0xffffffffu, c0, 4 * (4 + q) + 2);
                    if (g == gA) tcacc += ya;
                    if (gB >= 0 && g == gB) tcacc += yb;
                }
            }
            // fold the TC contribution (row q) into the FP64 lane layout: lane q adds it to
            // the row it will write (rowmap below) — gather via shuffles inside the group.
            const int myrow = (q == 0) ? 0 : (q == 1) ? 2 : (q == 2) ? 1 : 3;
            const double tcmine = __shfl_sync(0xffffffffu, tcacc, 4 * g + myrow);
            const double s0 = L.acc0 + __shfl_xor_sync(0xffffffffu, L.acc0, 1);
            const double s1 = L.acc1 + __shfl_xor_sync(0xffffffffu, L.acc1, 1);
            if (write) epi.finish(out_i, ((q & 1) ? s1 : s0) + tcmine, pre);
            return;
        }
        const double s0 = L.acc0 + __shfl_xor_sync(0xffffffffu, L.acc0, 1);
        const double s1 = L.acc1 + __shfl_xor_sync(0xffffffffu, L.acc1, 1);
        if constexpr (MODE == EPI_JACOBI_NORM) {  // per-warp partial of the residual norm
            double sq = 0.0;
            if (write) {
                const double res = (double)epi.finish(out_i, (q & 1) ? s1 : s0, pre);
                sq = res * res;
            }
            for (int d = 16; d; d >>= 1) sq += __shfl_xor_sync(0xffffffffu, sq, d);
            if (lane == 0) epi.nws[wid] = sq;
        } else {
            if (write) epi.finish(out_i, (q & 1) ? s1 : s0, pre);
        }
    } else {
        // FP32 / FP16 tiles: lane q owns tile row q; U tiles' indices, bitmaps and row values
        // are requested before the x gathers (one dependent round trip per U tiles).
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
            if constexpr (MODE == EPI_RES_X0) {  // x1_J = 0 + w dinv_J (b_J - 0), the k_jacobi0 expression
                const float om = (float)epi.omega;
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    xv[u] = make_float4(0.f, 0.f, 0.f, 0.f);
                    if (nib[u]) {
                        const float4 bq = x_quad((const float*)epi.b, J[u]), dq = x_quad((const float*)epi.dinv, J[u]);
                        const float zero = 0.f, t0 = 0.f;
                        xv[u] = make_float4(zero + om * dq.x * (bq.x - t0), zero + om * dq.y * (bq.y - t0),
                                            zero + om * dq.z * (bq.z - t0), zero + om * dq.w * (bq.w - t0));
                    }
                }
            } else {
#pragma unroll
                for (int u = 0; u < U; ++u) xv[u] = nib[u] ? x_quad(x, J[u]) : make_float4(0.f, 0.f, 0.f, 0.f);
            }
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

// Row kernel: warps take row octets in a grid-stride loop (one octet per warp when the grid
// covers the rows, AMGT_SPMV_PERSIST=0; by default a grid of exactly the resident CTAs while
// the launch is <= kPersistMaxWaves waves, so no partial last wave: 386.8 vs 399.8 us per
// config-2 V-cycle; longer launches keep the full grid: config-3 A_1 2.42 vs 2.53 ms).
template <typename MatT, typename XT, typename YT, int MODE, int U = 2, int MINB = 1, bool TC = false>
__global__ void __launch_bounds__(256, MINB) k_spmv_rows(int64_t I0, int64_t BR, const int64_t* __restrict__ bptr,
                                                   const int32_t* __restrict__ bidx,
                                                   const uint16_t* __restrict__ bmap, const MatT* __restrict__ bval,
                                                   const XT* __restrict__ x, const Epi<XT, YT, MODE> epi,
                                                   int64_t long_thr, int tc_thr) {
    pdl_wait();
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; I0 + wid * 8 < BR; wid += nw)
        spmv_rows_octet<MatT, XT, YT, MODE, U, TC>(wid, I0, BR, bptr, bidx, bmap, bval, x, epi, long_thr, tc_thr);
}

// ---------------------------------------------------------------- warp-per-row kernel
// FP32 / FP16 coarse operators of up to AMGT_SPMV_WROW block columns (default 65,536: config 3's
// levels 3-5) with >= 16 tiles per block row on average (~27 there): a warp per block row, the 8 four-lane groups take tiles
// g, g + 8, g + 16, g + 24 of the row (32 per iteration: one dependent round trip for the tiles
// and one for x, where the octet kernel needs four pairs for a 27-tile row), lane q of a group
// accumulates tile row q; the 8 group partials are added by a fixed 3-step xor tree
// (deterministic).  The small levels are latency-bound, so fewer round trips per row is the gain.
template <typename MatT, typename XT, typename YT, int MODE>
__global__ void __launch_bounds__(256) k_spmv_wrow(int64_t I0, int64_t BR, const int64_t* __restrict__ bptr,
                                                   const int32_t* __restrict__ bidx, const uint16_t* __restrict__ bmap,
                                                   const MatT* __restrict__ bval, const XT* __restrict__ x,
                                                   const Epi<XT, YT, MODE> epi, int64_t long_thr) {
    pdl_wait();
    const int lane = threadIdx.x & 31, g = lane >> 2, q = lane & 3;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t I = I0 + (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5); I < BR; I += nw) {
        const int64_t t0 = __ldg(bptr + I);
        int64_t t1 = __ldg(bptr + I + 1);
        if (t1 - t0 > long_thr) continue;  // warp-uniform: the chunk kernel takes long rows
        const int64_t out_i = 4 * I + q;
        typename Epi<XT, YT, MODE>::Pre pre;
        if (g == 0) pre = epi.prefetch(out_i);
        constexpr int U = 4;
        float acc = 0.f;
        for (int64_t t = t0 + g; t < t1; t += 8 * U) {
            int32_t J[U];
            uint32_t nib[U];
            float4 a[U], xv[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const int64_t tt = t + 8 * u;
                const bool v = tt < t1;
                J[u] = v ? __ldg(bidx + tt) : 0;
                nib[u] = v ? (__ldg(bmap + tt) >> (4 * q)) & 0xFu : 0u;
                a[u] = make_float4(0.f, 0.f, 0.f, 0.f);
                if (v) {
                    if constexpr (sizeof(MatT) == 4) {
                        a[u] = ldg_stream(reinterpret_cast<const float4*>(bval + 16 * tt) + q);
                    } else {
                        const uint2 w = ldg_stream(reinterpret_cast<const uint2*>(bval + 16 * tt) + q);
                        const float2 lo = __half22float2(*reinterpret_cast<const __half2*>(&w.x));
                        const float2 hi = __half22float2(*reinterpret_cast<const __half2*>(&w.y));
                        a[u] = make_float4(lo.x, lo.y, hi.x, hi.y);
                    }
                }
            }
            if constexpr (MODE == EPI_RES_X0) {  // x1_J = 0 + w dinv_J (b_J - 0), the k_jacobi0 expression
                const float om = (float)epi.omega;
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    xv[u] = make_float4(0.f, 0.f, 0.f, 0.f);
                    if (nib[u]) {
                        const float4 bq = x_quad((const float*)epi.b, J[u]), dq = x_quad((const float*)epi.dinv, J[u]);
                        const float zero = 0.f, z0 = 0.f;
                        xv[u] = make_float4(zero + om * dq.x * (bq.x - z0), zero + om * dq.y * (bq.y - z0),
                                            zero + om * dq.z * (bq.z - z0), zero + om * dq.w * (bq.w - z0));
                    }
                }
            } else {
#pragma unroll
                for (int u = 0; u < U; ++u) xv[u] = nib[u] ? x_quad(x, J[u]) : make_float4(0.f, 0.f, 0.f, 0.f);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                acc = (nib[u] & 1u) ? fmaf(a[u].x, xv[u].x, acc) : acc;
                acc = (nib[u] & 2u) ? fmaf(a[u].y, xv[u].y, acc) : acc;
                acc = (nib[u] & 4u) ? fmaf(a[u].z, xv[u].z, acc) : acc;
                acc = (nib[u] & 8u) ? fmaf(a[u].w, xv[u].w, acc) : acc;
            }
        }
        acc += __shfl_xor_sync(0xffffffffu, acc, 4);
        acc += __shfl_xor_sync(0xffffffffu, acc, 8);
        acc += __shfl_xor_sync(0xffffffffu, acc, 16);
        if (g == 0) epi.finish(out_i, acc, pre);
    }
}

static int64_t wrow_max_br() {
    static int64_t v = -1;
    if (v < 0) {
        const char* e = getenv("AMGT_SPMV_WROW");
        v = e ? atoll(e) : 65536;
    }
    return v;
}

// ---------------------------------------------------------------- lane-per-row kernel
// For operators with ~1 tile per block row (interpolation P, L262/Alg. 2 line 8): one lane
// owns a whole block row (its tiles' 16 values, its x segment, its 4 outputs), 32 block rows
// per warp, so every dependent round trip moves 32 tiles instead of 8.
template <typename MatT, typename XT, typename YT, int MODE>
__global__ void __launch_bounds__(256) k_spmv_lanerow(int64_t I0, int64_t BR, const int64_t* __restrict__ bptr,
                                                      const int32_t* __restrict__ bidx,
                                                      const uint16_t* __restrict__ bmap,
                                                      const MatT* __restrict__ bval, const XT* __restrict__ x,
                                                      const Epi<XT, YT, MODE> epi, bool vec) {
    pdl_wait();
    using Acc = typename AccOf<MatT>::type;
    const int64_t I = I0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (I >= BR) return;
    const int64_t t0 = __ldg(bptr + I), t1 = __ldg(bptr + I + 1);
    typename Epi<XT, YT, MODE>::Pre pre[4];
    if (vec) {
        epi.prefetch4(4 * I, pre);
    } else {
#pragma unroll
        for (int r = 0; r < 4; ++r) pre[r] = epi.prefetch(4 * I + r);
    }
    Acc acc[4] = {Acc(0), Acc(0), Acc(0), Acc(0)};
    for (int64_t t = t0; t < t1; ++t) {
        const int32_t J = __ldg(bidx + t);
        const uint32_t mp = __ldg(bmap + t);
        Acc v[16];  // one lane reads the whole tile: L1-allocating loads (sectors re-used)
        if constexpr (sizeof(MatT) == 8) {
#pragma unroll
            for (int k = 0; k < 8; ++k) {
                const double2 d = __ldg(reinterpret_cast<const double2*>(bval + 16 * t) + k);
                v[2 * k] = d.x;
                v[2 * k + 1] = d.y;
            }
        } else if constexpr (sizeof(MatT) == 4) {
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const float4 d = __ldg(reinterpret_cast<const float4*>(bval + 16 * t) + k);
                v[4 * k] = d.x; v[4 * k + 1] = d.y; v[4 * k + 2] = d.z; v[4 * k + 3] = d.w;
            }
        } else {
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const uint2 w = __ldg(reinterpret_cast<const uint2*>(bval + 16 * t) + k);
                const float2 lo = __half22float2(*reinterpret_cast<const __half2*>(&w.x));
                const float2 hi = __half22float2(*reinterpret_cast<const __half2*>(&w.y));
                v[4 * k] = lo.x; v[4 * k + 1] = lo.y; v[4 * k + 2] = hi.x; v[4 * k + 3] = hi.y;
            }
        }
        Acc xv[4];
        if constexpr (sizeof(Acc) == 8) {
            const double2 a = x_pair(x, J, 0), b = x_pair(x, J, 1);
            xv[0] = a.x; xv[1] = a.y; xv[2] = b.x; xv[3] = b.y;
        } else {
            const float4 a = x_quad(x, J);
            xv[0] = a.x; xv[1] = a.y; xv[2] = a.z; xv[3] = a.w;
        }
#pragma unroll
        for (int r = 0; r < 4; ++r)
#pragma unroll
            for (int c = 0; c < 4; ++c)
                acc[r] = ((mp >> (4 * r + c)) & 1u) ? fma(v[4 * r + c], xv[c], acc[r]) : acc[r];
    }
    if (vec) {
        epi.finish4(4 * I, acc, pre);
    } else {
#pragma unroll
        for (int r = 0; r < 4; ++r) epi.finish(4 * I + r, acc[r], pre[r]);
    }
}

// FP64 operators with ~1 tile per block row (the level-1 interpolation P): LPR lanes per block
// row (2 by default), lane h owning tile rows [h 4/LPR, (h+1) 4/LPR) (contiguous 16-B loads).
// The lane-per-row kernel's loads touch 32 lines per warp instruction (8 instructions per
// tile: L1-wavefront bound, ncu 82% L1/TEX); with 2 lanes each tile line is touched by 4.  Same
// per-row accumulation order as k_spmv_lanerow (tiles in order, columns in order).
template <typename XT, typename YT, int MODE, int LPR>
__global__ void __launch_bounds__(256) k_spmv_lanepair(int64_t I0, int64_t BR, const int64_t* __restrict__ bptr,
                                                       const int32_t* __restrict__ bidx,
                                                       const uint16_t* __restrict__ bmap,
                                                       const double* __restrict__ bval, const XT* __restrict__ x,
                                                       const Epi<XT, YT, MODE> epi) {
    constexpr int RPL = 4 / LPR;  // tile rows per lane
    pdl_wait();
    const int64_t gt = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t I = I0 + gt / LPR;
    const int h = (int)(gt % LPR);
    if (I >= BR) return;  // all lanes of the row
    const int64_t t0 = __ldg(bptr + I), t1 = __ldg(bptr + I + 1);
    typename Epi<XT, YT, MODE>::Pre pre[RPL];
#pragma unroll
    for (int rr = 0; rr < RPL; ++rr) pre[rr] = epi.prefetch(4 * I + RPL * h + rr);
    double acc[RPL];
#pragma unroll
    for (int rr = 0; rr < RPL; ++rr) acc[rr] = 0.0;
    for (int64_t t = t0; t < t1; ++t) {
        const int32_t J = __ldg(bidx + t);
        const uint32_t mp = __ldg(bmap + t);
        double v[4 * RPL];
        const double2* tp = reinterpret_cast<const double2*>(bval + 16 * t + 4 * RPL * h);
#pragma unroll
        for (int k = 0; k < 2 * RPL; ++k) {
            const double2 d = __ldg(tp + k);
            v[2 * k] = d.x;
            v[2 * k + 1] = d.y;
        }
        const double2 xa = x_pair(x, J, 0), xb = x_pair(x, J, 1);
        const double xv[4] = {xa.x, xa.y, xb.x, xb.y};
#pragma unroll
        for (int rr = 0; rr < RPL; ++rr) {
            const int r = RPL * h + rr;
#pragma unroll
            for (int c = 0; c < 4; ++c)
                acc[rr] = ((mp >> (4 * r + c)) & 1u) ? fma(v[4 * rr + c], xv[c], acc[rr]) : acc[rr];
        }
    }
#pragma unroll
    for (int rr = 0; rr < RPL; ++rr) epi.finish(4 * I + RPL * h + rr, acc[rr], pre[rr]);
}

// ---------------------------------------------------------------- chunk kernel (long rows)
template <typename MatT, typename XT>
__global__ void __launch_bounds__(256) k_spmv_chunks(int64_t nchunks, const int64_t* __restrict__ bptr,
                                                     const int32_t* __restrict__ bidx,
                                                     const uint16_t* __restrict__ bmap,
                                                     const MatT* __restrict__ bval, const XT* __restrict__ x,
                                                     const int32_t* __restrict__ long_rows,
                                                     const int64_t* __restrict__ chunk_ptr,
                                                     const int32_t* __restrict__ chunk_lr,
                                                     typename AccOf<MatT>::type* __restrict__ partial) {
    pdl_wait();
    using Acc = typename AccOf<MatT>::type;
    const int lane = threadIdx.x & 31, g = lane >> 2, q = lane & 3;
    const int64_t c = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (c >= nchunks) return;
    const int32_t lr = chunk_lr[c];
    const int64_t row = long_rows[lr];
    const int64_t k = c - chunk_ptr[lr];
    const int64_t a = bptr[row] + k * WARP_CAPACITY;
    const int64_t b = min(a + WARP_CAPACITY, bptr[row + 1]);
    Acc out;
    if constexpr (sizeof(MatT) == 8) {
        F64Lane L;
        for (int64_t t = a + g; t < b; t += 8) {
            const int32_t J = __ldg(bidx + t);
            L.step((const double*)bval + 16 * t, __ldg(bmap + t), x_pair(x, J, q & 1), q);
        }
        double s0 = L.acc0 + __shfl_xor_sync(0xffffffffu, L.acc0, 1);
        double s1 = L.acc1 + __shfl_xor_sync(0xffffffffu, L.acc1, 1);
        double v = (q & 1) ? s1 : s0;  // row rowmap(q)
        v += __shfl_xor_sync(0xffffffffu, v, 4);
        v += __shfl_xor_sync(0xffffffffu, v, 8);
        v += __shfl_xor_sync(0xffffffffu, v, 16);
        const int myrow = (q == 0) ? 0 : (q == 1) ? 2 : (q == 2) ? 1 : 3;
        if (g == 0) partial[4 * c + myrow] = v;
        (void)out;
    } else {
        float acc = 0.f;
        for (int64_t t = a + g; t < b; t += 8) {
            const int32_t J = __ldg(bidx + t);
            const uint32_t nib = (__ldg(bmap + t) >> (4 * q)) & 0xFu;
            const float4 xv = x_quad(x, J);
            float a0, a1, a2, a3;
            if constexpr (sizeof(MatT) == 4) {
                const float4 av = ldg_stream(reinterpret_cast<const float4*>(bval + 16 * t) + q);
                a0 = av.x; a1 = av.y; a2 = av.z; a3 = av.w;
            } else {
                const uint2 u = ldg_stream(reinterpret_cast<const uint2*>(bval + 16 * t) + q);
                const float2 lo = __half22float2(*reinterpret_cast<const __half2*>(&u.x));
                const float2 hi = __half22float2(*reinterpret_cast<const __half2*>(&u.y));
                a0 = lo.x; a1 = lo.y; a2 = hi.x; a3 = hi.y;
            }
            acc = (nib & 1u) ? fmaf(a0, xv.x, acc) : acc;
            acc = (nib & 2u) ? fmaf(a1, xv.y, acc) : acc;
            acc = (nib & 4u) ? fmaf(a2, xv.z, acc) : acc;
            acc = (nib & 8u) ? fmaf(a3, xv.w, acc) : acc;
        }
        acc += __shfl_xor_sync(0xffffffffu, acc, 4);
        acc += __shfl_xor_sync(0xffffffffu, acc, 8);
        acc += __shfl_xor_sync(0xffffffffu, acc, 16);
        if (g == 0) partial[4 * c + q] = acc;
    }
}

template <typename Acc, typename XT, typename YT>
__global__ void k_spmv_combine(int64_t nlong, const int32_t* __restrict__ long_rows,
                               const int64_t* __restrict__ chunk_ptr, const Acc* __restrict__ partial,
                               const Epi<XT, YT> epi) {
    pdl_wait();
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= 4 * nlong) return;
    const int64_t lr = i >> 2;
    const int r = (int)(i & 3);
    Acc s = 0;
    for (int64_t c = chunk_ptr[lr]; c < chunk_ptr[lr + 1]; ++c) s += partial[4 * c + r];
    epi.apply(4 * (int64_t)long_rows[lr] + r, s);
}

// ---------------------------------------------------------------- analysis kernels
__global__ void k_plan_rows(int64_t BR, const int64_t* __restrict__ bptr, int64_t* __restrict__ islong,
                            int64_t* __restrict__ nch, double* __restrict__ sums /*[2]: sum len, sum len^2*/) {
    double s1 = 0, s2 = 0;
    for (int64_t I = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; I < BR; I += (int64_t)gridDim.x * blockDim.x) {
        const int64_t len = bptr[I + 1] - bptr[I];
        const bool lg = len > WARP_CAPACITY;
        islong[I] = lg;
        nch[I] = lg ? (len + WARP_CAPACITY - 1) / WARP_CAPACITY : 0;
        s1 += (double)len;
        s2 += (double)len * (double)len;
    }
    for (int d = 16; d; d >>= 1) {
        s1 += __shfl_xor_sync(0xffffffffu, s1, d);
        s2 += __shfl_xor_sync(0xffffffffu, s2, d);
    }
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(sums, s1);
        atomicAdd(sums + 1, s2);
    }
}

__global__ void k_plan_fill(int64_t BR, const int64_t* __restrict__ bptr, const int64_t* __restrict__ lpos,
                            const int64_t* __restrict__ cpos, int32_t* __restrict__ long_rows,
                            int64_t* __restrict__ chunk_ptr, int32_t* __restrict__ chunk_lr) {
    for (int64_t I = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; I < BR; I += (int64_t)gridDim.x * blockDim.x) {
        if (lpos[I + 1] == lpos[I]) continue;
        const int64_t lr = lpos[I];
        long_rows[lr] = (int32_t)I;
        chunk_ptr[lr] = cpos[I];
        for (int64_t c = cpos[I]; c < cpos[I + 1]; ++c) chunk_lr[c] = (int32_t)lr;
    }
}

__global__ void k_count_tc(int64_t T, const uint16_t* __restrict__ bmap, int thr, unsigned long long* __restrict__ out) {
    int64_t s = 0, nz = 0;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < T; t += (int64_t)gridDim.x * blockDim.x) {
        const int p = __popc(bmap[t]);
        s += p >= thr;
        nz += p;
    }
    for (int d = 16; d; d >>= 1) {
        s += __shfl_xor_sync(0xffffffffu, s, d);
        nz += __shfl_xor_sync(0xffffffffu, nz, d);
    }
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(out, (unsigned long long)s);
        atomicAdd(out + 1, (unsigned long long)nz);
    }
}

static unsigned grid_cap(int64_t work, int threads) {
    int64_t b = ceil_div(work, threads);
    int64_t cap = (int64_t)num_sms() * 16;
    return (unsigned)(b < 1 ? 1 : (b > cap ? cap : b));
}

// The reported statistics of a plan (amgt_spmv_get_stats; no effect on the SpMV): mean and
// coefficient of variation of tiles per block row (R11), popcount sum, tensor-core tiles.
static amgt_status plan_stats(const amgt_mbsr* A, SpmvPlan* P, cudaStream_t s) {
    Alloc a{nullptr, s};
    const int64_t BR = A->blc_row;
    Scratch<int64_t> islong, nch;
    Scratch<double> sums;
    Scratch<unsigned long long> tcc;
    AMGT_TRY(islong.init(a, BR + 1));
    AMGT_TRY(nch.init(a, BR + 1));
    AMGT_TRY(sums.init(a, 2));
    AMGT_TRY(tcc.init(a, 2));
    AMGT_CUDA(cudaMemsetAsync(sums.p, 0, 2 * sizeof(double), s));
    AMGT_CUDA(cudaMemsetAsync(tcc.p, 0, 2 * sizeof(unsigned long long), s));
    if (BR > 0) {
        k_plan_rows<<<grid_cap(BR, 256), 256, 0, s>>>(BR, A->blc_ptr, islong.p, nch.p, sums.p);
        AMGT_LAUNCHED();
    }
    if (A->blc_num > 0) {
        k_count_tc<<<grid_cap(A->blc_num, 256), 256, 0, s>>>(A->blc_num, A->blc_map, g_tc_thr_spmv, tcc.p);
        AMGT_LAUNCHED();
    }
    double hs[2];
    unsigned long long ht[2];
    AMGT_CUDA(cudaMemcpyAsync(hs, sums.p, sizeof(hs), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaMemcpyAsync(ht, tcc.p, sizeof(ht), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaStreamSynchronize(s));
    const double mean = BR ? hs[0] / BR : 0.0;
    const double var = BR ? hs[1] / BR - mean * mean : 0.0;
    P->st.avg_nnz_blc = A->blc_num ? (double)ht[1] / (double)A->blc_num : 0.0;
    P->st.variation = mean > 0 ? sqrt(var > 0 ? var : 0) / mean : 0.0;
    P->st.long_rows = P->nlong;
    P->st.chunks = P->nchunks;
    P->st.tc_tiles = (int64_t)ht[0];
    P->stats_ready = true;
    return AMGT_OK;
}

amgt_status spmv_analyze_impl(amgt_mbsr* A, Alloc& a) {
    cudaStream_t s = a.s;
    if (A->aux) { spmv_plan_free(A->aux, a); A->aux = nullptr; }
    const int64_t BR = A->blc_row;
    if (A->row_max > 0 && A->row_max <= WARP_CAPACITY) {
        // longest block row known (conversion / SpGEMM / transpose) and within one warp chunk:
        // no long rows, nothing to split, no device work and no synchronisation; the reported
        // statistics are computed on first request
        SpmvPlan* P = new SpmvPlan();
        P->mean_row = BR ? (double)A->blc_num / (double)BR : 0.0;
        A->aux = P;
        return AMGT_OK;
    }
    Scratch<int64_t> islong, nch, lpos, cpos;
    Scratch<double> sums;
    Scratch<unsigned long long> tcc;
    AMGT_TRY(islong.init(a, BR + 1));
    AMGT_TRY(nch.init(a, BR + 1));
    AMGT_TRY(lpos.init(a, BR + 1));
    AMGT_TRY(cpos.init(a, BR + 1));
    AMGT_TRY(sums.init(a, 2));
    AMGT_TRY(tcc.init(a, 2));
    AMGT_CUDA(cudaMemsetAsync(sums.p, 0, 2 * sizeof(double), s));
    AMGT_CUDA(cudaMemsetAsync(tcc.p, 0, 2 * sizeof(unsigned long long), s));
    if (BR > 0) {
        k_plan_rows<<<grid_cap(BR, 256), 256, 0, s>>>(BR, A->blc_ptr, islong.p, nch.p, sums.p);
        AMGT_LAUNCHED();
    }
    if (A->blc_num > 0) {
        k_count_tc<<<grid_cap(A->blc_num, 256), 256, 0, s>>>(A->blc_num, A->blc_map, g_tc_thr_spmv, tcc.p);
        AMGT_LAUNCHED();
    }
    AMGT_TRY(scan_exclusive(islong.p, lpos.p, BR, a, s));
    AMGT_TRY(scan_exclusive(nch.p, cpos.p, BR, a, s));
    int64_t nl = 0, ncx = 0;
    double hs[2];
    unsigned long long ht[2];
    AMGT_CUDA(cudaMemcpyAsync(&nl, lpos.p + BR, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaMemcpyAsync(&ncx, cpos.p + BR, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaMemcpyAsync(hs, sums.p, sizeof(hs), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaMemcpyAsync(ht, tcc.p, sizeof(ht), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaStreamSynchronize(s));
    SpmvPlan* P = new SpmvPlan();
    P->nlong = nl;
    P->nchunks = ncx;
    if (nl > 0) {
        P->long_rows = (int32_t*)a.get(nl * sizeof(int32_t));
        P->chunk_ptr = (int64_t*)a.get((nl + 1) * sizeof(int64_t));
        P->chunk_lr = (int32_t*)a.get(ncx * sizeof(int32_t));
        P->partial = (double*)a.get(ncx * 4 * sizeof(double));
        if (!P->long_rows || !P->chunk_ptr || !P->chunk_lr || !P->partial) {
            spmv_plan_free(P, a);
            return fail(AMGT_ERR_ALLOC, "SpMV plan allocation failed");
        }
        k_plan_fill<<<grid_cap(BR, 256), 256, 0, s>>>(BR, A->blc_ptr, lpos.p, cpos.p, P->long_rows, P->chunk_ptr,
                                                     P->chunk_lr);
        AMGT_LAUNCHED();
        AMGT_CUDA(cudaMemcpyAsync(P->chunk_ptr + nl, &ncx, sizeof(int64_t), cudaMemcpyHostToDevice, s));
        AMGT_CUDA(cudaStreamSynchronize(s));  // ncx is a host stack value
    }
    const double mean = BR ? hs[0] / BR : 0.0;
    const double var = BR ? hs[1] / BR - mean * mean : 0.0;
    P->st.avg_nnz_blc = A->blc_num ? (double)ht[1] / (double)A->blc_num : 0.0;
    P->st.variation = mean > 0 ? sqrt(var > 0 ? var : 0) / mean : 0.0;
    P->st.long_rows = nl;
    P->st.chunks = ncx;
    P->st.tc_tiles = (int64_t)ht[0];
    P->stats_ready = true;
    P->mean_row = mean;
    A->aux = P;
    return AMGT_OK;
}

// FP64 SpMV kernel variant (tiles per iteration U, minimum resident blocks MINB of 256
// threads — i.e. the register budget): 0 = U8/4 (default; measured best on B200, see
// DESIGN.md §7), 1 = U4/5, 2 = U4/6, 3 = U2/6.
// The environment variable AMGT_SPMV_VARIANT selects another for tuning.
// AMGT_SPMV_PERSIST: 0 = one warp per row octet over a full grid, 1 = grid of exactly the
// resident CTAs while the launch is at most kPersistMaxWaves waves (default), 2 = always.
static constexpr unsigned kPersistMaxWaves = 32;

static int spmv_variant() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("AMGT_SPMV_VARIANT");
        v = e ? atoi(e) : 0;
        if (v < 0 || v > 3) v = 0;
    }
    return v;
}

// lanes per block row of k_spmv_lanepair for FP64 ~1-tile-per-row operators (AMGT_LANEPAIR:
// 2 default, 4, or 0 = the lane-per-row kernel; measurement knob)
static int lanepair_lanes() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("AMGT_LANEPAIR");
        v = e ? atoi(e) : 2;
    }
    return v;
}

// AMGT_LANEROW=0: ~1-tile-per-row matrices take the group kernel too (measurement knob)
static bool lanerow_enabled() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("AMGT_LANEROW");
        v = (e && e[0] == '0') ? 0 : 1;
    }
    return v == 1;
}

bool spmv_warp_norm_ok(const amgt_mbsr* A) {
    const SpmvPlan* P = (const SpmvPlan*)A->aux;
    return A->prec == AMGT_FP64 && g_tc_thr_spmv > 16 && P && P->nlong == 0 &&
           !(P->mean_row <= 2.0 && lanerow_enabled());
}
int64_t spmv_warp_norm_count(const amgt_mbsr* A) { return ceil_div(A->blc_row, 8); }

// ---------------------------------------------------------------- tensor-core routes (L222-228)
// FP64 (DMMA m8n8k4): one warp per block row walks its tiles in consecutive pairs (t, t+1).  The
// A fragment [A_t; A_t+1] is ONE coalesced 256-byte load: lane l holds element l % 16 of tile
// t + l / 16, i.e. row l / 4, column l % 4 of the 8x4 fragment (a[row8][k4], lane = 4 row8 + k4).
// The B fragment is [x_J | x_J' | 0 ...] (lane 4n + k holds B[k][n]).  C accumulates over the whole
// row; y_r = C[r][0] + C[4 + r][1] ("diagonal of fragY", L228).  Per-tile routing (R10): a tile
// with POPCOUNT(map) < tc_thr is multiplied by the CUDA cores of the 16 lanes that loaded it
// (bitmap-predicated FMAs) and enters the mma with a zero B column; a pair without a dense tile
// skips the mma.  Values: route-independent up to rounding.  Rows longer than long_thr are the
// chunk kernel's.
__device__ __forceinline__ double ldg_f64(const double* p) {
    double r;
    asm volatile("ld.global.nc.f64 %0, [%1];" : "=d"(r) : "l"(p));
    return r;
}

template <typename XT, typename YT, int MODE, int UP>
__global__ void __launch_bounds__(256) k_spmv_tc64(int64_t I0, int64_t BR, const int64_t* __restrict__ bptr,
                                                   const int32_t* __restrict__ bidx, const uint16_t* __restrict__ bmap,
                                                   const double* __restrict__ bval, const XT* __restrict__ x,
                                                   Epi<XT, YT, MODE> epi, int64_t long_thr, int tc_thr) {
    pdl_wait();
    constexpr unsigned FULL = 0xffffffffu;
    const int lane = threadIdx.x & 31, h = lane >> 4, e = lane & 15, n = lane >> 2, k = lane & 3;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t I = I0 + (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5); I < BR; I += nw) {
        const int64_t t0 = __ldg(bptr + I), t1 = __ldg(bptr + I + 1);
        if (t1 - t0 > long_thr) continue;  // warp-uniform
        typename Epi<XT, YT, MODE>::Pre pre;
        if (lane < 4) pre = epi.prefetch(4 * I + lane);
        double c0 = 0.0, c1 = 0.0, cc = 0.0;
        for (int64_t p = t0; p < t1; p += 2 * UP) {
            double a[UP];
            uint32_t mp[UP];
            int32_t J[UP];
            bool v[UP];
#pragma unroll
            for (int u = 0; u < UP; ++u) {  // every load of the UP pairs in flight together
                const int64_t t = p + 2 * u + h;
                v[u] = t < t1;
                a[u] = v[u] ? ldg_f64(bval + 16 * t + e) : 0.0;
                mp[u] = v[u] ? __ldg(bmap + t) : 0u;
                J[u] = v[u] ? __ldg(bidx + t) : 0;
            }
            // x operands of all UP pairs requested before any mma (one dependent round trip)
            double xb[UP], xc[UP];
            bool dn[UP], any[UP];
#pragma unroll
            for (int u = 0; u < UP; ++u) {
                dn[u] = v[u] && __popc(mp[u]) >= tc_thr;
                const int32_t Jb = __shfl_sync(FULL, J[u], n == 1 ? 16 : 0);
                const bool db = __shfl_sync(FULL, dn[u] ? 1 : 0, n == 1 ? 16 : 0) != 0;
                any[u] = __any_sync(FULL, dn[u]);
                xb[u] = (n < 2 && db) ? (double)__ldg(x + 4 * (int64_t)Jb + k) : 0.0;
                xc[u] = (v[u] && !dn[u] && ((mp[u] >> e) & 1u)) ? (double)__ldg(x + 4 * (int64_t)J[u] + (e & 3)) : 0.0;
            }
#pragma unroll
            for (int u = 0; u < UP; ++u) {
                if (v[u] && !dn[u]) cc = fma(a[u], xc[u], cc);  // xc = 0 at the clear bits
                if (any[u]) dmma_884(c0, c1, dn[u] ? a[u] : 0.0, xb[u]);
            }
        }
        double cs = cc + __shfl_xor_sync(FULL, cc, 1);
        cs += __shfl_xor_sync(FULL, cs, 2);
        cs += __shfl_xor_sync(FULL, cs, 16);  // lanes 4r.. and 16+4r..: the CUDA-core sum of row r
        const int r = lane & 3;
        const double ya = __shfl_sync(FULL, c0, 4 * r), yb = __shfl_sync(FULL, c1, 16 + 4 * r);
        const double yc = __shfl_sync(FULL, cs, 4 * r);
        if (lane < 4) epi.finish(4 * I + lane, ya + yb + yc, pre);
    }
}

// FP16 (HMMA m16n8k16, FP16 operands, FP32 accumulation, R18): a warp takes FOUR block rows g =
// 0..3 and their tiles four at a time: A[4g + r][4i + c] = tile i of row g (row r, column c),
// B[4i + c][g] = x_J(g,i)[c] (x rounded to FP16 for the mma), so C[4g + r][g] = the four tiles'
// contribution to row r of block row g — 16 tile products per instruction, the diagonal column
// blocks of C kept.  Tiles with POPCOUNT < tc_thr go through CUDA-core FMAs (FP32, x in FP32) of
// the lanes that hold them and enter the mma as zeros.
__device__ __forceinline__ void hmma_16816(float (&c)[4], const uint32_t (&a)[4], const uint32_t (&b)[2]) {
    asm volatile(
        "mma.sync.aligned.m16n8k16.row.col.f32.f16.f16.f32 {%0, %1, %2, %3}, {%4, %5, %6, %7}, {%8, %9}, "
        "{%0, %1, %2, %3};"
        : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
}

template <typename XT, typename YT, int MODE>
__global__ void __launch_bounds__(256) k_spmv_tc16(int64_t I0, int64_t BR, const int64_t* __restrict__ bptr,
                                                   const int32_t* __restrict__ bidx, const uint16_t* __restrict__ bmap,
                                                   const __half* __restrict__ bval, const XT* __restrict__ x,
                                                   Epi<XT, YT, MODE> epi, int64_t long_thr, int tc_thr) {
    pdl_wait();
    constexpr unsigned FULL = 0xffffffffu;
    const int lane = threadIdx.x & 31, gid = lane >> 2, tig = lane & 3;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t Q = I0 + 4 * (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5); Q < BR; Q += 4 * nw) {
        // this lane's two A rows: (g0 = gid / 4, r = gid % 4) and (g0 + 2, r); its B column gid (< 4)
        const int r = gid & 3, gA = gid >> 2, gB = gA + 2;
        int64_t ta0 = 0, ta1 = 0, tb0 = 0, tb1 = 0, tn0 = 0, tn1 = 0;
        auto range = [&](int g, int64_t& lo, int64_t& hi) {
            const int64_t I = Q + g;
            lo = hi = 0;
            if (I < BR) {
                lo = __ldg(bptr + I);
                hi = __ldg(bptr + I + 1);
                if (hi - lo > long_thr) hi = lo;  // chunk kernel's row
            }
        };
        range(gA, ta0, ta1);
        range(gB, tb0, tb1);
        if (gid < 4) range(gid, tn0, tn1);
        int64_t len = max(ta1 - ta0, tb1 - tb0);
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) len = max(len, __shfl_xor_sync(FULL, len, d));
        typename Epi<XT, YT, MODE>::Pre pre;
        const int64_t out_i = 4 * (Q + (lane >> 2 & 3)) + (lane & 3);  // lanes 0-15: rows of the quad
        const bool writer = lane < 16 && Q + (lane >> 2) < BR;
        if (writer) pre = epi.prefetch(out_i);
        float c[4] = {0.f, 0.f, 0.f, 0.f};
        float ccA = 0.f, ccB = 0.f;  // CUDA-core sums of rows (gA, r) and (gB, r)
        for (int64_t w = 0; w < len; w += 4) {
            // phase 1: the A side (tile values of this lane's two rows, 4 tile slots) and the B
            // side (bitmaps and columns of block row gid's tiles), all requested together
            uint32_t raw[4], mpA[4], mpB[2];
            int64_t tA[4], JA[4], JB[2];
            bool vA[4], vB[2];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const bool rowB = q & 1;
                const int i = (tig >> 1) + ((q >> 1) << 1);
                const int64_t lo = rowB ? tb0 : ta0, hi = rowB ? tb1 : ta1;
                tA[q] = lo + w + i;
                vA[q] = tA[q] < hi;
                raw[q] = vA[q] ? __ldg(reinterpret_cast<const uint32_t*>(bval + 16 * tA[q] + 4 * r) + (tig & 1)) : 0u;
                mpA[q] = vA[q] ? (uint32_t)__ldg(bmap + tA[q]) : 0u;
                JA[q] = vA[q] ? (int64_t)__ldg(bidx + tA[q]) : 0;
            }
#pragma unroll
            for (int q = 0; q < 2; ++q) {
                const int64_t t = tn0 + w + (tig >> 1) + 2 * q;
                vB[q] = gid < 4 && t < tn1;
                mpB[q] = vB[q] ? (uint32_t)__ldg(bmap + t) : 0u;
                JB[q] = vB[q] ? (int64_t)__ldg(bidx + t) : 0;
            }
            // phase 2: x operands (B fragment in FP16; the sparse tiles' entries in FP32)
            const int cb = 2 * (tig & 1);
            uint32_t a[4], b[2];
            float2 xs[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const bool dense = vA[q] && __popc(mpA[q]) >= tc_thr;
                a[q] = dense ? raw[q] : 0u;
                const uint32_t bits = (vA[q] && !dense) ? (mpA[q] >> (4 * r + cb)) & 3u : 0u;
                xs[q] = make_float2(bits & 1u ? (float)__ldg(x + 4 * JA[q] + cb) : 0.f,
                                    bits & 2u ? (float)__ldg(x + 4 * JA[q] + cb + 1) : 0.f);
            }
#pragma unroll
            for (int q = 0; q < 2; ++q) {
                b[q] = 0u;
                if (vB[q] && __popc(mpB[q]) >= tc_thr) {
                    const __half2 xv = __floats2half2_rn((float)__ldg(x + 4 * JB[q] + cb), (float)__ldg(x + 4 * JB[q] + cb + 1));
                    b[q] = *reinterpret_cast<const uint32_t*>(&xv);
                }
            }
            // phase 3: the sparse tiles on CUDA cores, the dense ones through the mma
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                if (a[q] == 0u && vA[q]) {
                    const float2 av = __half22float2(*reinterpret_cast<const __half2*>(&raw[q]));
                    const float sv = fmaf(av.y, xs[q].y, av.x * xs[q].x);
                    if (q & 1) ccB += sv; else ccA += sv;
                }
            }
            hmma_16816(c, a, b);
        }
        // C[4g + r][g]: g = 0 -> c[0] of lanes 4r (tig 0), g = 1 -> c[1] of lanes 16 + 4r, g = 2 ->
        // c[2] of lanes 4r + 1, g = 3 -> c[3] of lanes 16 + 4r + 1
        float sA = ccA + __shfl_xor_sync(FULL, ccA, 1);
        sA += __shfl_xor_sync(FULL, sA, 2);
        float sB = ccB + __shfl_xor_sync(FULL, ccB, 1);
        sB += __shfl_xor_sync(FULL, sB, 2);  // group gid: rows (gA, r) and (gB, r) summed over tig
        const int g = lane >> 2 & 3, rr = lane & 3;  // this writer lane's block row g and row rr
        const int srcC = (g & 1 ? 16 : 0) + 4 * rr + (g >> 1);
        const float v0 = __shfl_sync(FULL, c[0], srcC), v1 = __shfl_sync(FULL, c[1], srcC);
        const float v2 = __shfl_sync(FULL, c[2], srcC), v3 = __shfl_sync(FULL, c[3], srcC);
        const float cv = g == 0 ? v0 : g == 1 ? v1 : g == 2 ? v2 : v3;
        // CUDA-core part of (g, rr): group gid' = 4 (g & 1) + rr holds it in sA (g < 2) or sB (g >= 2)
        const int srcS = 4 * (4 * (g & 1) + rr);
        const float vA = __shfl_sync(FULL, sA, srcS), vB = __shfl_sync(FULL, sB, srcS);
        if (writer) epi.finish(out_i, cv + (g < 2 ? vA : vB), pre);
    }
}

template <typename MatT, typename XT, typename YT, int MODE>
static void launch_rows(const amgt_mbsr* A, const void* x, void* y, const EpiArgs& ea, int64_t I0, int64_t BR,
                        int64_t long_thr, cudaStream_t s) {
    const Epi<XT, YT, MODE> epi{(YT*)y, (const YT*)ea.b, (const YT*)ea.dinv, (const XT*)ea.xs, (YT)ea.omega, MODE,
                                (YT*)ea.r, (YT*)ea.x1, ea.nws};
    const SpmvPlan* P = (const SpmvPlan*)A->aux;
    if (MODE != EPI_RES_X0 && P && P->nlong == 0 && P->mean_row <= 2.0 && g_tc_thr_spmv > 16 &&
        lanerow_enabled()) {  // ~1 tile per block row
        // vector epilogue when every vector it touches is 4-element aligned
        const uintptr_t al = 4 * sizeof(YT) - 1;
        auto ok = [&](const void* p) { return (reinterpret_cast<uintptr_t>(p) & al) == 0; };
        const bool vec = ok(y) && ok(ea.b) && ok(ea.dinv) && ok(ea.r) &&
                         (reinterpret_cast<uintptr_t>(ea.xs) & (4 * sizeof(XT) - 1)) == 0;
        if constexpr (sizeof(MatT) == 8) {
            const int lpr = lanepair_lanes();
            if (lpr == 2 || lpr == 4) {
                auto kern = lpr == 2 ? k_spmv_lanepair<XT, YT, MODE, 2> : k_spmv_lanepair<XT, YT, MODE, 4>;
                pdl_launch(kern, dim3((unsigned)ceil_div(lpr * (BR - I0), 256)), dim3(256), 0, s, I0, BR, A->blc_ptr,
                           A->blc_idx, A->blc_map, (const double*)A->blc_val, (const XT*)x, epi);
                return;
            }
        }
        pdl_launch(k_spmv_lanerow<MatT, XT, YT, MODE>, dim3((unsigned)ceil_div(BR - I0, 256)), dim3(256), 0, s, I0, BR,
                   A->blc_ptr, A->blc_idx, A->blc_map, (const MatT*)A->blc_val, (const XT*)x, epi, vec);
        return;
    }
    const unsigned blocks = (unsigned)ceil_div(ceil_div(BR - I0, 8) * 32, 256);
    const int tc = sizeof(MatT) != 4 ? g_tc_thr_spmv : 17;  // FP32: CUDA cores (no TF32, R17)
    if constexpr (sizeof(MatT) <= 4 && MODE != EPI_JACOBI_NORM) {
        // small coarse levels with long rows (decided per operator — block columns, mean row
        // length — so a row range of a distributed operator takes the same arithmetic)
        const double mean = A->blc_row > 0 ? (double)A->blc_num / (double)A->blc_row : 0.0;
        if (tc > 16 && A->blc_col <= wrow_max_br() && mean >= 16.0) {
            auto kern = k_spmv_wrow<MatT, XT, YT, MODE>;
            const int per_sm = occupancy_256(reinterpret_cast<const void*>(kern));
            const int64_t cap = (int64_t)num_sms() * std::max(per_sm, 1);
            const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(BR - I0, 8), cap));
            pdl_launch(kern, dim3(g), dim3(256), 0, s, I0, BR, A->blc_ptr, A->blc_idx, A->blc_map,
                       (const MatT*)A->blc_val, (const XT*)x, epi, long_thr);
            return;
        }
    }
    if (tc <= 16 && MODE != EPI_JACOBI_NORM && MODE != EPI_RES_X0) {  // tensor-core routes (L222-228)
        const int per_sm_cap = 8;  // 256-thread CTAs: persistent grid over the rows
        if constexpr (sizeof(MatT) == 8) {
            const unsigned g = (unsigned)std::min<int64_t>(ceil_div((BR - I0) * 32, 256), (int64_t)num_sms() * per_sm_cap);
            pdl_launch(k_spmv_tc64<XT, YT, MODE, 4>, dim3(std::max(g, 1u)), dim3(256), 0, s, I0, BR, A->blc_ptr,
                       A->blc_idx, A->blc_map, (const double*)A->blc_val, (const XT*)x, epi, long_thr, tc);
            return;
        } else if constexpr (sizeof(MatT) == 2) {
            const unsigned g =
                (unsigned)std::min<int64_t>(ceil_div(ceil_div(BR - I0, 4) * 32, 256), (int64_t)num_sms() * per_sm_cap);
            pdl_launch(k_spmv_tc16<XT, YT, MODE>, dim3(std::max(g, 1u)), dim3(256), 0, s, I0, BR, A->blc_ptr,
                       A->blc_idx, A->blc_map, (const __half*)A->blc_val, (const XT*)x, epi, long_thr, tc);
            return;
        }
    }
    static const int persist = [] { const char* e = getenv("AMGT_SPMV_PERSIST"); return e ? atoi(e) : 1; }();
    auto go = [&](auto kern) {
        unsigned g = blocks;
        if (persist > 0) {  // exactly the resident CTAs (no partial last wave)
            const int per_sm = occupancy_256(reinterpret_cast<const void*>(kern));
            const unsigned cap = (unsigned)num_sms() * (unsigned)std::max(per_sm, 1);
            // auto (1): only while the partial last wave is a visible share of the launch; over
            // many waves a grid-stride loop lets the warps drift apart in the address space
            // (config-3 A_1, ~110 octets per warp: 2.53 ms vs 2.37 ms for the full grid)
            if (persist > 1 || g <= kPersistMaxWaves * cap) g = std::min(g, cap);
        }
        pdl_launch(kern, dim3(g), dim3(256), 0, s, I0, BR, A->blc_ptr, A->blc_idx, A->blc_map,
                   (const MatT*)A->blc_val, (const XT*)x, epi, long_thr, tc);
    };
    if constexpr (sizeof(MatT) == 8) {
        switch (spmv_variant()) {  // tuning knob AMGT_SPMV_VARIANT: tiles per iteration x min blocks/SM
            case 1: go(k_spmv_rows<MatT, XT, YT, MODE, 4, 5>); break;
            case 2: go(k_spmv_rows<MatT, XT, YT, MODE, 4, 6>); break;
            case 3: go(k_spmv_rows<MatT, XT, YT, MODE, 2, 6>); break;
            default: go(k_spmv_rows<MatT, XT, YT, MODE, 8, 4>);
        }
    } else {
        go(k_spmv_rows<MatT, XT, YT, MODE, 8, 4>);
    }
}

template <typename MatT, typename XT, typename YT>
static amgt_status launch_spmv(const amgt_mbsr* A, const void* x, void* y, const EpiArgs& ea, cudaStream_t s) {
    const SpmvPlan* P = (const SpmvPlan*)A->aux;
    const bool ranged = ea.I1 >= 0;
    if (ranged && P && P->nlong > 0) return fail(AMGT_ERR_UNSUPPORTED, "row-range SpMV on a matrix with split long rows");
    const int64_t long_thr = (P && P->nlong > 0) ? WARP_CAPACITY : INT64_MAX;
    const int64_t I0 = ranged ? ea.I0 : 0, BR = ranged ? ea.I1 : A->blc_row;
    if (BR > I0) {
        switch (ea.mode) {
            case AMGT_EPI_JACOBI: launch_rows<MatT, XT, YT, AMGT_EPI_JACOBI>(A, x, y, ea, I0, BR, long_thr, s); break;
            case AMGT_EPI_JACOBI_RES:
                launch_rows<MatT, XT, YT, AMGT_EPI_JACOBI_RES>(A, x, y, ea, I0, BR, long_thr, s);
                break;
            case AMGT_EPI_RESIDUAL: launch_rows<MatT, XT, YT, AMGT_EPI_RESIDUAL>(A, x, y, ea, I0, BR, long_thr, s); break;
            case AMGT_EPI_ACCUM: launch_rows<MatT, XT, YT, AMGT_EPI_ACCUM>(A, x, y, ea, I0, BR, long_thr, s); break;
            case EPI_JACOBI_NORM:
                if constexpr (sizeof(MatT) == 8 && std::is_same<XT, double>::value && std::is_same<YT, double>::value) {
                    if (!spmv_warp_norm_ok(A) || ranged) return fail(AMGT_ERR_UNSUPPORTED, "warp-partial norm");
                    launch_rows<MatT, XT, YT, EPI_JACOBI_NORM>(A, x, y, ea, I0, BR, long_thr, s);
                } else {
                    return fail(AMGT_ERR_UNSUPPORTED, "warp-partial norm: FP64 only");
                }
                break;
            case EPI_RES_X0:
                if constexpr (sizeof(MatT) < 8 && std::is_same<XT, float>::value && std::is_same<YT, float>::value) {
                    if (P && P->nlong > 0) return fail(AMGT_ERR_UNSUPPORTED, "zero-guess residual with split long rows");
                    launch_rows<MatT, XT, YT, EPI_RES_X0>(A, x, y, ea, I0, BR, long_thr, s);
                } else {
                    return fail(AMGT_ERR_UNSUPPORTED, "zero-guess residual: FP32 vectors, FP32/FP16 operator only");
                }
                break;
            default: launch_rows<MatT, XT, YT, AMGT_EPI_Y>(A, x, y, ea, I0, BR, long_thr, s);
        }
        AMGT_LAUNCHED();
    }
    if (!ranged && P && P->nlong > 0) {
        using Acc = typename AccOf<MatT>::type;
        const Epi<XT, YT> epi{(YT*)y, (const YT*)ea.b, (const YT*)ea.dinv, (const XT*)ea.xs, (YT)ea.omega, ea.mode,
                              (YT*)ea.r};
        pdl_launch(k_spmv_chunks<MatT, XT>, dim3((unsigned)ceil_div(P->nchunks * 32, 256)), dim3(256), 0, s,
                   P->nchunks, A->blc_ptr, A->blc_idx, A->blc_map, (const MatT*)A->blc_val, (const XT*)x,
                   P->long_rows, P->chunk_ptr, P->chunk_lr, (Acc*)P->partial);
        AMGT_LAUNCHED();
        pdl_launch(k_spmv_combine<Acc, XT, YT>, dim3((unsigned)ceil_div(4 * P->nlong, 256)), dim3(256), 0, s,
                   P->nlong, P->long_rows, P->chunk_ptr, (const Acc*)P->partial, epi);
        AMGT_LAUNCHED();
    }
    return AMGT_OK;
}

template <typename MatT>
static amgt_status dispatch_xy(const amgt_mbsr* A, const void* x, amgt_prec xp, void* y, amgt_prec yp,
                               const EpiArgs& ea, cudaStream_t s) {
    if (xp == AMGT_FP64 && yp == AMGT_FP64) return launch_spmv<MatT, double, double>(A, x, y, ea, s);
    if (xp == AMGT_FP64 && yp == AMGT_FP32) return launch_spmv<MatT, double, float>(A, x, y, ea, s);
    if (xp == AMGT_FP32 && yp == AMGT_FP64) return launch_spmv<MatT, float, double>(A, x, y, ea, s);
    return launch_spmv<MatT, float, float>(A, x, y, ea, s);
}

double spmv_bytes(const amgt_mbsr* A, amgt_prec xp, amgt_prec yp) {
    // T(16s + 4 + 2) + (BR+1) 8 + 4 BC s_x + 4 BR s_y
    return A->blc_num * (16.0 * prec_bytes(A->prec) + 6.0) + (A->blc_row + 1) * 8.0 +
           4.0 * A->blc_col * prec_bytes(xp) + 4.0 * A->blc_row * prec_bytes(yp);
}

amgt_status spmv_ex_impl(const amgt_mbsr* A, const void* x, amgt_prec xp, void* y, amgt_prec yp, const EpiArgs& ea,
                         cudaStream_t s, int timer_class) {
    const double vec = 4.0 * A->blc_row * prec_bytes(yp);
    // epilogue operands read once each: Jacobi b, dinv (+ r written); residual b; accumulate y
    const double extra = (ea.mode == AMGT_EPI_JACOBI || ea.mode == EPI_JACOBI_NORM) ? 2 * vec
                         : (ea.mode == AMGT_EPI_JACOBI_RES || ea.mode == EPI_RES_X0) ? 3 * vec
                         : (ea.mode == AMGT_EPI_Y ? 0.0 : vec);
    // a block-row range (the distributed path's interior / boundary launches) counts its share
    const double frac = (ea.I1 >= 0 && A->blc_row > 0)
                            ? (double)(std::min<int64_t>(ea.I1, A->blc_row) - ea.I0) / (double)A->blc_row
                            : 1.0;
    TimerScope ts(timer_class, (spmv_bytes(A, xp, yp) + extra) * frac, s);
    switch (A->prec) {
        case AMGT_FP64: return dispatch_xy<double>(A, x, xp, y, yp, ea, s);
        case AMGT_FP32: return dispatch_xy<float>(A, x, xp, y, yp, ea, s);
        default: return dispatch_xy<__half>(A, x, xp, y, yp, ea, s);
    }
}

amgt_status spmv_impl(const amgt_mbsr* A, const void* x, amgt_prec xp, void* y, amgt_prec yp, cudaStream_t s,
                      int timer_class) {
    return spmv_ex_impl(A, x, xp, y, yp, EpiArgs{AMGT_EPI_Y, nullptr, nullptr, nullptr, 0.0, 0, -1}, s, timer_class);
}

}  // namespace amgt

using namespace amgt;

extern "C" {

amgt_status amgt_spmv_analyze(amgt_mbsr* A, const amgt_allocator* al, void* stream) {
    if (!A) return fail(AMGT_ERR_ARG, "amgt_spmv_analyze: NULL matrix");
    Alloc a{al, (cudaStream_t)stream};
    return spmv_analyze_impl(A, a);
}

amgt_status amgt_spmv_get_stats(const amgt_mbsr* A, amgt_spmv_stats* st) {
    if (!A || !st) return fail(AMGT_ERR_ARG, "amgt_spmv_get_stats: NULL argument");
    if (!A->aux) return fail(AMGT_ERR_ARG, "amgt_spmv_get_stats: matrix not analysed");
    SpmvPlan* P = (SpmvPlan*)A->aux;
    if (!P->stats_ready) AMGT_TRY(plan_stats(A, P, (cudaStream_t)0));  // legacy stream: ordered after prior work
    *st = P->st;
    return AMGT_OK;
}

amgt_status amgt_spmv(const amgt_mbsr* A, const void* x, amgt_prec xprec, void* y, amgt_prec yprec, void* stream) {
    if (!A || (!x && A->blc_col > 0) || (!y && A->blc_row > 0)) return fail(AMGT_ERR_ARG, "amgt_spmv: NULL argument");
    if ((xprec != AMGT_FP64 && xprec != AMGT_FP32) || (yprec != AMGT_FP64 && yprec != AMGT_FP32))
        return fail(AMGT_ERR_ARG, "amgt_spmv: x/y precision must be FP64 or FP32");
    if (!prec_valid(A->prec)) return fail(AMGT_ERR_ARG, "amgt_spmv: bad matrix precision");
    return spmv_impl(A, x, xprec, y, yprec, (cudaStream_t)stream, TC_SPMV);
}

amgt_status amgt_spmv_fused_r(const amgt_mbsr* A, const void* x, amgt_prec xprec, void* y, amgt_prec yprec,
                              const void* b, const void* dinv, double omega, void* r, void* stream) {
    if (!A || (!x && A->blc_col > 0) || (!y && A->blc_row > 0) || (!r && A->blc_row > 0))
        return fail(AMGT_ERR_ARG, "amgt_spmv_fused_r: NULL argument");
    if ((xprec != AMGT_FP64 && xprec != AMGT_FP32) || xprec != yprec)
        return fail(AMGT_ERR_ARG, "amgt_spmv_fused_r: x/y must share one precision, FP64 or FP32");
    if (!b || !dinv || A->m != A->n || x == y || r == x || r == y)
        return fail(AMGT_ERR_ARG, "amgt_spmv_fused_r: needs b, dinv, a square A and distinct x, y, r");
    EpiArgs ea{AMGT_EPI_JACOBI_RES, b, dinv, x, omega, 0, -1};
    ea.r = r;
    return spmv_ex_impl(A, x, xprec, y, yprec, ea, (cudaStream_t)stream, TC_SPMV);
}

amgt_status amgt_spmv_fused(const amgt_mbsr* A, const void* x, amgt_prec xprec, void* y, amgt_prec yprec, int mode,
                            const void* b, const void* dinv, double omega, void* stream) {
    if (!A || (!x && A->blc_col > 0) || (!y && A->blc_row > 0)) return fail(AMGT_ERR_ARG, "amgt_spmv_fused: NULL argument");
    if ((xprec != AMGT_FP64 && xprec != AMGT_FP32) || (yprec != AMGT_FP64 && yprec != AMGT_FP32))
        return fail(AMGT_ERR_ARG, "amgt_spmv_fused: x/y precision must be FP64 or FP32");
    if (mode < AMGT_EPI_Y || mode > AMGT_EPI_ACCUM) return fail(AMGT_ERR_ARG, "amgt_spmv_fused: bad mode");
    if ((mode == AMGT_EPI_JACOBI || mode == AMGT_EPI_RESIDUAL) && !b) return fail(AMGT_ERR_ARG, "amgt_spmv_fused: b is NULL");
    if (mode == AMGT_EPI_JACOBI && (!dinv || xprec != yprec || A->m != A->n || x == y))
        return fail(AMGT_ERR_ARG, "amgt_spmv_fused: Jacobi needs dinv, a square A, x/y of one precision, x != y");
    return spmv_ex_impl(A, x, xprec, y, yprec, EpiArgs{mode, b, dinv, x, omega, 0, -1}, (cudaStream_t)stream, TC_SPMV);
}

amgt_status amgt_spmv_fused_range(const amgt_mbsr* A, int64_t blk_begin, int64_t blk_end, const void* x,
                                  amgt_prec xprec, void* y, amgt_prec yprec, int mode, const void* b, const void* dinv,
                                  const void* xs, double omega, void* stream) {
    if (!A || blk_begin < 0 || blk_end < blk_begin || blk_end > A->blc_row)
        return fail(AMGT_ERR_ARG, "amgt_spmv_fused_range: bad block-row range");
    if ((xprec != AMGT_FP64 && xprec != AMGT_FP32) || (yprec != AMGT_FP64 && yprec != AMGT_FP32))
        return fail(AMGT_ERR_ARG, "amgt_spmv_fused_range: x/y precision must be FP64 or FP32");
    if (mode < AMGT_EPI_Y || mode > AMGT_EPI_ACCUM) return fail(AMGT_ERR_ARG, "amgt_spmv_fused_range: bad mode");
    if ((mode == AMGT_EPI_JACOBI || mode == AMGT_EPI_RESIDUAL) && !b)
        return fail(AMGT_ERR_ARG, "amgt_spmv_fused_range: b is NULL");
    if (mode == AMGT_EPI_JACOBI && (!dinv || !xs || xprec != yprec))
        return fail(AMGT_ERR_ARG, "amgt_spmv_fused_range: Jacobi needs dinv, xs and x/y of one precision");
    if (blk_end == blk_begin) return AMGT_OK;
    return spmv_ex_impl(A, x, xprec, y, yprec, EpiArgs{mode, b, dinv, xs, omega, blk_begin, blk_end},
                        (cudaStream_t)stream, TC_SPMV);
}

}  // extern "C"
