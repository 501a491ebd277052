// sweep.cu — consecutive Alg. 2 SpMV steps on one FP64 operator in ONE pass over HBM
// (§8(f) NEXT-1: fused solve-phase kernels).
//
// On level 1 of the V-cycle, the post-smoothing sweep of cycle c (Alg. 2 line 10), the
// pre-smoothing sweep of cycle c+1 (line 2; it also yields the residual of cycle c, L308)
// and the residual of cycle c+1 (line 3) are three back-to-back SpMVs with A_1 whose only
// dependencies are through neighbouring rows.  A_1 of config 2 is 488 MB and the B200 L2 is
// 126 MB, so three separate kernels read it from HBM three times.  Here one persistent kernel
// runs the stages as a wavefront over chunks of 64 block rows: work item w (claimed in order
// from a global counter) does stage 0 on chunk w, stage 1 on chunk w - D, stage 2 on chunk
// w - 2D (consecutive items interleave the stages: item 3k + s = stage s of chunk k - sD).
// Stage s of chunk c waits until stage s-1 is done on every chunk its columns touch
// (completion counters per group of 8 chunks, release/acquire); D = forward bandwidth + 1 +
// about the items in flight, so the tiles a later stage re-reads were streamed by stage 0 only
// ~2D chunks earlier and are still in L2: A_1 comes from HBM about once per three SpMVs.
// Latency hiding per item: the next item is claimed while this one runs, and a later stage
// issues all its A-side loads (row pointers, tile columns, bitmaps, values, b, dinv) before it
// waits for the previous stage; only the x gathers come after the wait.
//
// Arithmetic per row is exactly that of k_spmv_rows with the matching epilogue (same tile
// order, same FMA sequence, same shuffles, same epilogue expression), so the iterates are
// bit-identical to the unfused kernels; only the residual norm is summed in a different
// fixed order (per-chunk partials, then a fixed tree in the last CTA): deterministic.
//
// Deadlock freedom: items are claimed in increasing order by running CTAs; an item waits only
// for items with smaller indices (D > forward bandwidth), which are held by running CTAs that
// never wait on larger items.
#include <cstdlib>
#include <cstring>

#include "common.cuh"
#include "spmv_core.cuh"

namespace amgt {

constexpr int SW_THREADS = 128;
constexpr int SW_CHUNK = 32;  // block rows per chunk: 4 warps x 8 four-lane groups
constexpr int SW_GROUP = 8;   // chunks per completion counter
#ifndef SW_MINB
#define SW_MINB 4  // resident CTAs per SM the register budget is sized for
#endif
#ifndef SW_STATS
#define SW_STATS 0  // 1: per-item cycle accounting into SweepDev::stats (diagnostics)
#endif
#ifndef SW_PRELOAD
#define SW_PRELOAD 0  // 1: tile loads issued before the wait (needs ~100 registers)
#endif

struct SweepDev {       // device-resident plan scalars
    int64_t D;          // stage lag in items
    int32_t bw_fwd;     // max over chunks of (last column chunk - chunk)
    uint32_t pad;
    uint32_t ctr[2];    // [0] item counter, [1] exit ticket (re-armed by the last CTA)
    unsigned long long stats[6];  // SW_STATS builds: cycles/count of stage-0 items, of later
                                  // items, cycles waiting, unready polls (amgt_sweep_plan_stats)
};

struct SweepPlanImpl {
    int64_t m = 0, BR = 0, nchunks = 0, T = 0;
    int grid = 0;
    bool tma = true;  // k_sweep_tma (default) or the register-staged k_sweep (AMGT_SWEEP_IMPL=ldg)
    uint32_t ep[AMGT_SWEEP_MAX_STAGES] = {0, 0, 0, 0};
    int64_t ngroups = 0;
    int32_t* clo = nullptr;     // [nchunks] first column GROUP read by the chunk's rows
    int32_t* chi = nullptr;     // [nchunks] last column group
    uint32_t* cnt = nullptr;    // [AMGT_SWEEP_MAX_STAGES * ngroups] completed chunk-stages (monotonic)
    double* partial = nullptr;  // [nchunks] squared-residual partial sums
    int64_t* chunk_t = nullptr; // [nchunks+1] first tile of each chunk (TMA variant)
    int32_t* xr = nullptr;      // [nchunks * TM_XR] x runs per chunk (TMA variant)
    SweepDev* dev = nullptr;
    amgt_allocator al{};
    bool has_al = false;
};

struct SweepStageDev {
    const double* x;
    double* y;
    int mode;
};

struct SweepArgs {
    int64_t BR, nchunks;
    const int64_t* __restrict__ bptr;
    const int32_t* __restrict__ bidx;
    const uint16_t* __restrict__ bmap;
    const double* __restrict__ bval;
    const double* __restrict__ b;
    const double* __restrict__ dinv;
    double omega;
    int nst;
    SweepStageDev st[AMGT_SWEEP_MAX_STAGES];
    const int32_t* __restrict__ clo;
    const int32_t* __restrict__ chi;
    uint32_t* cnt;
    int64_t ngroups;
    uint32_t ep[AMGT_SWEEP_MAX_STAGES];  // launches so far (this one included) that ran stage s
    SweepDev* dev;
    double* partial;
    double* norm_out;
};

__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void red_release_add(uint32_t* p, uint32_t v) {
#if SW_RELAXED_SIGNAL  // timing experiment only: NOT a correct signal
    asm volatile("red.relaxed.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
#else
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
#endif
}
__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }

// x pair of column block J (elements 2h, 2h+1); COH = produced inside this kernel: L2 only
template <bool COH>
__device__ __forceinline__ double2 sw_x_pair(const double* x, int64_t J, int h) {
    const double2* p = reinterpret_cast<const double2*>(x + 4 * J + 2 * h);
    if constexpr (COH) return __ldcg(p);
    else return __ldg(p);
}
template <bool COH>
__device__ __forceinline__ double sw_ld(const double* p) {
    if constexpr (COH) return __ldcg(p);
    else return __ldg(p);
}

constexpr int SW_U = 8;  // tiles per load batch (7-point rows: 6.9 tiles per block row)

// A-side operands of one batch of SW_U tiles (read-only data: may be loaded before the wait)
struct SwBatch {
    int32_t J[SW_U];
    uint32_t mp[SW_U];
    double2 a[SW_U], b[SW_U];
};
__device__ __forceinline__ void sw_load_batch(SwBatch& B, int64_t t, int64_t t1, const SweepArgs& a, int q) {
#pragma unroll
    for (int u = 0; u < SW_U; ++u) {
        const bool v = t + u < t1;
        B.J[u] = v ? __ldg(a.bidx + t + u) : 0;
        B.mp[u] = v ? __ldg(a.bmap + t + u) : 0u;
        if (v) {
            B.a[u] = ldg_stream(reinterpret_cast<const double2*>(a.bval + 16 * (t + u)) + q);
            B.b[u] = ldg_stream(reinterpret_cast<const double2*>(a.bval + 16 * (t + u)) + 4 + q);
        } else {
            B.a[u] = make_double2(0.0, 0.0);
            B.b[u] = B.a[u];
        }
    }
}
// x gathers and FMAs of a batch: the FMA order of f64_tile_loop (spmv_core.cuh)
template <bool COH>
__device__ __forceinline__ void sw_fma_batch(F64Lane& L, const SwBatch& B, const double* x, int q) {
    double2 xv[SW_U];
#pragma unroll
    for (int u = 0; u < SW_U; ++u) xv[u] = B.mp[u] ? sw_x_pair<COH>(x, B.J[u], q & 1) : make_double2(0.0, 0.0);
#pragma unroll
    for (int u = 0; u < SW_U; ++u) {
        const uint32_t s0 = B.mp[u] >> (2 * q), s1 = B.mp[u] >> (8 + 2 * q);
        L.acc0 = (s0 & 1u) ? fma(B.a[u].x, xv[u].x, L.acc0) : L.acc0;
        L.acc0 = (s0 & 2u) ? fma(B.a[u].y, xv[u].y, L.acc0) : L.acc0;
        L.acc1 = (s1 & 1u) ? fma(B.b[u].x, xv[u].x, L.acc1) : L.acc1;
        L.acc1 = (s1 & 2u) ? fma(B.b[u].y, xv[u].y, L.acc1) : L.acc1;
    }
}

// kernel-parameter arrays indexed with a run-time stage: select, so they stay in param space
__device__ __forceinline__ SweepStageDev sw_st(const SweepArgs& a, int s) {
    return s == 0 ? a.st[0] : s == 1 ? a.st[1] : s == 2 ? a.st[2] : a.st[3];
}
__device__ __forceinline__ uint32_t sw_ep(const SweepArgs& a, int s) {
    return s == 0 ? a.ep[0] : s == 1 ? a.ep[1] : s == 2 ? a.ep[2] : a.ep[3];
}

// Block until stage s-1 has completed every chunk in column groups [g0, g1] (warp 0 polls the
// group counters with relaxed loads in parallel, then one acquire fence; bar.sync extends it
// to the CTA).  Must be called by all threads.
__device__ __forceinline__ void sw_wait(const SweepArgs& a, int s, int64_t c, unsigned long long* wst) {
#if SW_STATS
    const long long w0 = clock64();
    unsigned polls = 0;
#endif
    if (threadIdx.x < 32) {
        const int64_t g0 = a.clo[c], g1 = a.chi[c];
        const uint32_t* cnt = a.cnt + (int64_t)(s - 1) * a.ngroups;
        for (int64_t gb = g0; gb <= g1; gb += 32) {
            const int64_t g = gb + threadIdx.x;
            bool ok = g > g1;
            if (!ok) {
                const int64_t gs = min((int64_t)SW_GROUP, a.nchunks - g * SW_GROUP);
                const uint32_t target = sw_ep(a, s - 1) * (uint32_t)gs;
                while (!(ok = ld_relaxed_u32(cnt + g) >= target)) {
#if SW_STATS
                    ++polls;
#endif
                    __nanosleep(20);
                }
            }
        }
        fence_acq_rel_gpu();
    }
    __syncthreads();
#if SW_STATS
    if (threadIdx.x == 0) { wst[0] += clock64() - w0; wst[1] += polls; }
#else
    (void)wst;
#endif
}

// One stage on one chunk; returns this thread's squared residual (norm stages) or 0.
template <bool COH>
__device__ __forceinline__ double sw_stage(const SweepArgs& a, int s, int64_t c, unsigned long long* wst) {
    const SweepStageDev st = sw_st(a, s);
    const int lane = threadIdx.x & 31, g = lane >> 2, q = lane & 3, warp = threadIdx.x >> 5;
    const int64_t I = c * SW_CHUNK + warp * 8 + g;
    int64_t t0 = 0, t1 = 0;
    const bool write = I < a.BR;
    if (write) {
        t0 = __ldg(a.bptr + I);
        t1 = __ldg(a.bptr + I + 1);
    }
    const int64_t out_i = 4 * I + ((q == 0) ? 0 : (q == 1) ? 2 : (q == 2) ? 1 : 3);
    const int mode = st.mode;
    const bool jac = mode == AMGT_SWEEP_J || mode == AMGT_SWEEP_JR;
    double pb = 0.0, pd = 0.0, px = 0.0;  // b_i, dinv_i, x_i
    if (write) {
        pb = __ldg(a.b + out_i);
        if (jac) pd = __ldg(a.dinv + out_i);
    }
    SwBatch B;
#if SW_PRELOAD
    sw_load_batch(B, t0, t1, a, q);  // A-side loads in flight across the wait
    if constexpr (COH) sw_wait(a, s, c, wst);
#else
    if constexpr (COH) sw_wait(a, s, c, wst);  // row pointers, b, dinv in flight across the wait
    sw_load_batch(B, t0, t1, a, q);
#endif
    if (write && jac) px = sw_ld<COH>(st.x + out_i);
    F64Lane L;
    sw_fma_batch<COH>(L, B, st.x, q);
    for (int64_t t = t0 + SW_U; t < t1; t += SW_U) {  // rows longer than one batch
        sw_load_batch(B, t, t1, a, q);
        sw_fma_batch<COH>(L, B, st.x, q);
    }
    const double s0 = L.acc0 + __shfl_xor_sync(0xffffffffu, L.acc0, 1);
    const double s1 = L.acc1 + __shfl_xor_sync(0xffffffffu, L.acc1, 1);
    if (!write) return 0.0;
    const double t = (q & 1) ? s1 : s0;
    double y, nrm = 0.0;
    switch (mode) {
        case AMGT_SWEEP_J: y = px + a.omega * pd * (pb - t); break;  // Epi JACOBI
        case AMGT_SWEEP_JR: {                                         // Epi JACOBI_RES
            const double res = pb - t;
            y = px + a.omega * pd * res;
            nrm = res * res;
            break;
        }
        case AMGT_SWEEP_RN:
            y = pb - t;
            nrm = y * y;
            break;
        default: y = pb - t;  // AMGT_SWEEP_R (Epi RESIDUAL)
    }
    st.y[out_i] = y;
    return nrm;
}

// fixed-order block sum of one double per thread (xor tree per warp, warps in order)
__device__ __forceinline__ double sw_block_sum(double v, double* sh) {
    for (int d = 16; d; d >>= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
    __syncthreads();
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = v;
    __syncthreads();
    double s = 0.0;
    if (threadIdx.x == 0)
        for (int w = 0; w < SW_THREADS / 32; ++w) s += sh[w];
    return s;
}

__global__ void __launch_bounds__(SW_THREADS, SW_MINB) k_sweep(SweepArgs a) {
    __shared__ int64_t s_item[2];
    __shared__ double s_red[SW_THREADS / 32];
    __shared__ bool s_last;
    const int64_t D = a.dev->D;
    const int64_t total = (a.nchunks + (int64_t)(a.nst - 1) * D) * a.nst;
    unsigned long long st6[6] = {0, 0, 0, 0, 0, 0};
    if (threadIdx.x == 0) s_item[0] = (int64_t)atomicAdd(&a.dev->ctr[0], 1u);
    for (int it = 0;; ++it) {
        __syncthreads();  // s_item[it & 1] visible; everyone is done with the other slot
        const int64_t w = s_item[it & 1];
        if (w >= total) break;
        // claim the next item now; its value is only stored at the end of this one
        unsigned nxt = 0;
        if (threadIdx.x == 0) nxt = atomicAdd(&a.dev->ctr[0], 1u);
        // item w = stage s of chunk k - s D, k = w / nst: consecutive items interleave the
        // stages, so HBM-streaming stage-0 work and L2-served later stages run side by side
        const int64_t k = w / a.nst;
        const int s = (int)(w - k * a.nst);
        const int64_t c = k - (int64_t)s * D;
        if (c >= 0 && c < a.nchunks) {
#if SW_STATS
            const long long t_item = clock64();
#endif
            const double nrm = s == 0 ? sw_stage<false>(a, 0, c, st6 + 4) : sw_stage<true>(a, s, c, st6 + 4);
            const int md = sw_st(a, s).mode;
            if (md == AMGT_SWEEP_JR || md == AMGT_SWEEP_RN) {
                const double part = sw_block_sum(nrm, s_red);
                if (threadIdx.x == 0) a.partial[c] = part;
            }
            __syncthreads();  // every row of chunk c written
            if (threadIdx.x == 0) red_release_add(a.cnt + (int64_t)s * a.ngroups + c / SW_GROUP, 1u);
#if SW_STATS
            if (threadIdx.x == 0) { st6[s ? 2 : 0] += clock64() - t_item; st6[s ? 3 : 1] += 1; }
#endif
        }
        if (threadIdx.x == 0) s_item[(it + 1) & 1] = (int64_t)nxt;
    }
#if SW_STATS
    if (threadIdx.x == 0)
        for (int i = 0; i < 6; ++i) atomicAdd(&a.dev->stats[i], st6[i]);
#endif
    // exit ticket: the last CTA re-arms the counters and sums the norm partials in order
    if (threadIdx.x == 0) {
        __threadfence();
        s_last = atomicAdd(&a.dev->ctr[1], 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    if (a.norm_out) {
        double v = 0.0;
        for (int64_t k = threadIdx.x; k < a.nchunks; k += SW_THREADS) v += __ldcg(a.partial + k);
        const double tot = sw_block_sum(v, s_red);
        if (threadIdx.x == 0) *a.norm_out = tot;
    }
    if (threadIdx.x == 0) {
        a.dev->ctr[0] = 0u;
        a.dev->ctr[1] = 0u;
    }
}

// ======================================================================================
// TMA-pipelined variant (default).  Measured on B200 (tools/sweep_bench.py): the register-
// staged kernel above reaches only ~1/3 of the L2 and HBM throughput — each CTA has one item
// in flight and stalls on the claim, the dependency poll, the row pointers and the release
// between items.  Here the memory side is decoupled from the arithmetic:
//   * one CTA per SM: a producer warp and TM_NG consumer groups of TM_GW warps (one chunk);
//   * the producer claims chunk steps k (one claim: stages 0..nst-1 of chunks k - sD), two
//     claims ahead, prefetches the plan's per-chunk descriptors (tile range, x runs), polls
//     the dependencies of a later stage, and moves everything the chunk's rows read into one
//     of TM_NS shared-memory slots with cp.async.bulk: tile values, tile columns, bitmaps,
//     row pointers, and the x segments ("runs": the chunk's column blocks merged into <= 8
//     contiguous ranges by the plan) — signalled by the slot's mbarrier with the byte count;
//   * consumer groups take the slots in turn (group g: items g, g+NG, ...), compute from
//     shared memory only, store y, and the group leader publishes the chunk (release
//     counter) and frees the slot (mbarrier).
// Chunks whose tiles or x runs exceed a slot fall back to global loads for that part.
constexpr int TM_NG = 4;                       // consumer groups
constexpr int TM_GW = SW_CHUNK / 8;            // warps per group (one chunk: 8 block rows per warp)
constexpr int TM_NS = 5;                       // slots
constexpr int TM_THREADS = 32 * (1 + TM_GW * TM_NG);
constexpr int TM_CAP = 224;                    // tiles per slot (7-point: <= 32 x 7)
constexpr int TM_XCAP = 208;                   // x blocks per slot (7-point 128^3: 192)
constexpr int TM_NRUN = 8;                     // x runs per chunk
constexpr int TM_XR = 1 + 2 * TM_NRUN;         // plan record per chunk: n, start[8], len[8]
constexpr int TM_VAL_BYTES = TM_CAP * 128;
constexpr int TM_IDX_BYTES = TM_CAP * 4 + 32;
constexpr int TM_MAP_BYTES = TM_CAP * 2 + 32;
constexpr int TM_PTR_BYTES = (SW_CHUNK + 2) * 8;
constexpr int TM_X_BYTES = TM_XCAP * 32;
constexpr int TM_V_BYTES = 4 * SW_CHUNK * 8;   // b or dinv of the chunk's rows
constexpr int TM_SLOT_BYTES = TM_VAL_BYTES + TM_IDX_BYTES + TM_MAP_BYTES + TM_PTR_BYTES + TM_X_BYTES + 2 * TM_V_BYTES;
constexpr int TM_SMEM = TM_NS * TM_SLOT_BYTES + 128;
static_assert(TM_SLOT_BYTES % 16 == 0, "slot layout must keep 16-byte alignment");
static_assert(TM_SMEM <= 227 * 1024, "slots exceed shared memory");

struct TmMeta {        // per slot, written by the producer before its arrive
    int64_t c;         // chunk (-1: stop)
    int64_t tbase;     // first tile of the chunk
    int32_t s;         // stage
    int32_t nrows;
    int32_t direct;    // tiles exceed the slot: consumers read tiles from global memory
    int32_t idx_off;   // byte offset of tile tbase inside the slot's idx area
    int32_t map_off;
    int32_t nrun;      // x runs in the slot (0: x from global memory)
    int32_t rs[TM_NRUN], rl[TM_NRUN], ro[TM_NRUN];  // run start block, length, slot offset
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
    asm volatile("{ .reg .b64 st; mbarrier.arrive.shared::cta.b64 st, [%0]; }" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* b, uint32_t bytes) {
    asm volatile("{ .reg .b64 st; mbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1; }" ::"r"(smem_u32(b)),
                 "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
    uint32_t done = 0;
    while (!done) {
        asm volatile(
            "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
            : "=r"(done)
            : "r"(smem_u32(b)), "r"(parity)
            : "memory");
    }
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void bar_named(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }

struct TmSlot {
    double* val;
    int32_t* idx;   // base of the idx area (byte offset idx_off applies)
    uint16_t* map;
    int64_t* ptr;
    double* x;
    double* b;      // b of the chunk's rows
    double* dinv;   // dinv of the chunk's rows (Jacobi stages)
};
__device__ __forceinline__ TmSlot tm_slot(char* base, int i) {
    char* p = base + (size_t)i * TM_SLOT_BYTES;
    TmSlot s;
    s.val = reinterpret_cast<double*>(p);
    p += TM_VAL_BYTES;
    s.idx = reinterpret_cast<int32_t*>(p);
    p += TM_IDX_BYTES;
    s.map = reinterpret_cast<uint16_t*>(p);
    p += TM_MAP_BYTES;
    s.ptr = reinterpret_cast<int64_t*>(p);
    p += TM_PTR_BYTES;
    s.x = reinterpret_cast<double*>(p);
    p += TM_X_BYTES;
    s.b = reinterpret_cast<double*>(p);
    p += TM_V_BYTES;
    s.dinv = reinterpret_cast<double*>(p);
    return s;
}

// Producer prefetch of the items of chunk step k into a shared-memory ring entry with
// cp.async (no register staging, so nothing waits until the entry is used two steps later):
// desc[s][f] = field f of stage s's item: 0/1 first/end tile, 2/3 clo/chi, 4 x-run count,
// 5..12 run starts, 13..20 run lengths.
constexpr int TM_DF = 4 + TM_XR;  // 21 fields
__device__ __forceinline__ void cp_async4(void* dst, const void* src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void tm_prefetch(const SweepArgs& a, const int64_t* __restrict__ chunk_t,
                                            const int32_t* __restrict__ xr, int64_t k, int64_t D, int lane,
                                            int32_t (*desc)[32]) {
    for (int s = 0; s < a.nst; ++s) {
        const int64_t c = k - (int64_t)s * D;
        if (c < 0 || c >= a.nchunks || lane >= TM_DF) continue;
        // tile offsets: low words of the int64 chunk_t entries (< 2^31, checked by the plan)
        const void* src = lane < 2 ? (const void*)(chunk_t + c + lane)
                        : lane == 2 ? (const void*)(a.clo + c)
                        : lane == 3 ? (const void*)(a.chi + c)
                        : (const void*)(xr + c * TM_XR + (lane - 4));
        cp_async4(&desc[s][lane], src);
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
}

// consumer: x pair (elements 2h, 2h+1) of column block J, from the slot's runs when present
template <bool COH>
__device__ __forceinline__ double2 tm_x_pair(const TmMeta& m, const double* xs, const double* xg, int32_t J, int h) {
    for (int r = 0; r < m.nrun; ++r) {
        const uint32_t d = (uint32_t)(J - m.rs[r]);
        if (d < (uint32_t)m.rl[r]) return reinterpret_cast<const double2*>(xs + 4 * (m.ro[r] + (int32_t)d) + 2 * h)[0];
    }
    return sw_x_pair<COH>(xg, J, h);
}

// f64_tile_loop (spmv_core.cuh) with the x loads of a stage (same FMA order)
template <bool COH>
__device__ __forceinline__ void f64_tile_loop_x(F64Lane& L, int64_t t0, int64_t t1, const int32_t* __restrict__ bidx,
                                                const uint16_t* __restrict__ bmap, const double* __restrict__ bval,
                                                const double* x, int q) {
    for (int64_t t = t0; t < t1; t += SW_U) {
        int32_t J[SW_U];
        uint32_t mp[SW_U];
        double2 av[SW_U], bv[SW_U], xv[SW_U];
#pragma unroll
        for (int u = 0; u < SW_U; ++u) {
            const bool v = t + u < t1;
            J[u] = v ? __ldg(bidx + t + u) : 0;
            mp[u] = v ? __ldg(bmap + t + u) : 0u;
            av[u] = v ? ldg_stream(reinterpret_cast<const double2*>(bval + 16 * (t + u)) + q) : make_double2(0.0, 0.0);
            bv[u] = v ? ldg_stream(reinterpret_cast<const double2*>(bval + 16 * (t + u)) + 4 + q) : make_double2(0.0, 0.0);
        }
#pragma unroll
        for (int u = 0; u < SW_U; ++u) xv[u] = mp[u] ? sw_x_pair<COH>(x, J[u], q & 1) : make_double2(0.0, 0.0);
#pragma unroll
        for (int u = 0; u < SW_U; ++u) {
            const uint32_t s0 = mp[u] >> (2 * q), s1 = mp[u] >> (8 + 2 * q);
            L.acc0 = (s0 & 1u) ? fma(av[u].x, xv[u].x, L.acc0) : L.acc0;
            L.acc0 = (s0 & 2u) ? fma(av[u].y, xv[u].y, L.acc0) : L.acc0;
            L.acc1 = (s1 & 1u) ? fma(bv[u].x, xv[u].x, L.acc1) : L.acc1;
            L.acc1 = (s1 & 2u) ? fma(bv[u].y, xv[u].y, L.acc1) : L.acc1;
        }
    }
}

// consumer fallback for chunks with more tiles than a slot: tiles from global memory (kept
// out of line so its batch registers do not raise the consumer's register budget)
template <bool COH>
__device__ __noinline__ void tm_direct(F64Lane& L, const int32_t* __restrict__ bidx, const uint16_t* __restrict__ bmap,
                                       const double* __restrict__ bval, const double* x, int64_t t0, int64_t t1,
                                       int q) {
    // (pointers by value: a reference to the kernel parameters would force them to local memory)
    f64_tile_loop_x<COH>(L, t0, t1, bidx, bmap, bval, x, q);
}

// consumer: one block row (4-lane group) of a slot's chunk; returns the squared residual
template <bool COH>
__device__ __forceinline__ double tm_row(const SweepArgs& a, const SweepStageDev& st, const TmMeta& m,
                                         const TmSlot& sl, int r, int q) {
    const int64_t I = m.c * SW_CHUNK + r;
    const bool write = r < m.nrows;
    int64_t t0 = 0, t1 = 0;
    if (write) {
        t0 = sl.ptr[r];
        t1 = sl.ptr[r + 1];
    }
    const int64_t out_i = 4 * I + ((q == 0) ? 0 : (q == 1) ? 2 : (q == 2) ? 1 : 3);
    const int mode = st.mode;
    const bool jac = mode == AMGT_SWEEP_J || mode == AMGT_SWEEP_JR;
    double pb = 0.0, pd = 0.0, px = 0.0;
    if (write) {
        const int li = (int)(out_i - 4 * m.c * SW_CHUNK);  // row within the chunk
        pb = sl.b[li];
        if (jac) {
            pd = sl.dinv[li];
            const double2 xp = tm_x_pair<COH>(m, sl.x, st.x, (int32_t)I, (int)((out_i & 3) >> 1));
            px = (out_i & 1) ? xp.y : xp.x;
        }
    }
    F64Lane L;
    if (m.direct) {
        tm_direct<COH>(L, a.bidx, a.bmap, a.bval, st.x, t0, t1, q);
    } else {
        const int32_t* sidx = reinterpret_cast<const int32_t*>(reinterpret_cast<const char*>(sl.idx) + m.idx_off);
        const uint16_t* smap = reinterpret_cast<const uint16_t*>(reinterpret_cast<const char*>(sl.map) + m.map_off);
        const int64_t b0 = t0 - m.tbase, b1 = t1 - m.tbase;
        for (int64_t t = b0; t < b1; t += SW_U) {
            int32_t J[SW_U];
            uint32_t mp[SW_U];
            double2 xv[SW_U];
#pragma unroll
            for (int u = 0; u < SW_U; ++u) {
                const bool v = t + u < b1;
                J[u] = v ? sidx[t + u] : 0;
                mp[u] = v ? smap[t + u] : 0u;
            }
#pragma unroll
            for (int u = 0; u < SW_U; ++u)
                xv[u] = mp[u] ? tm_x_pair<COH>(m, sl.x, st.x, J[u], q & 1) : make_double2(0.0, 0.0);
#pragma unroll
            for (int u = 0; u < SW_U; ++u) {
                double2 av = make_double2(0.0, 0.0), bv = av;
                if (t + u < b1) {
                    av = reinterpret_cast<const double2*>(sl.val + 16 * (t + u))[q];
                    bv = reinterpret_cast<const double2*>(sl.val + 16 * (t + u))[4 + q];
                }
                const uint32_t s0 = mp[u] >> (2 * q), s1 = mp[u] >> (8 + 2 * q);
                L.acc0 = (s0 & 1u) ? fma(av.x, xv[u].x, L.acc0) : L.acc0;
                L.acc0 = (s0 & 2u) ? fma(av.y, xv[u].y, L.acc0) : L.acc0;
                L.acc1 = (s1 & 1u) ? fma(bv.x, xv[u].x, L.acc1) : L.acc1;
                L.acc1 = (s1 & 2u) ? fma(bv.y, xv[u].y, L.acc1) : L.acc1;
            }
        }
    }
    const double s0 = L.acc0 + __shfl_xor_sync(0xffffffffu, L.acc0, 1);
    const double s1 = L.acc1 + __shfl_xor_sync(0xffffffffu, L.acc1, 1);
    if (!write) return 0.0;
    const double t = (q & 1) ? s1 : s0;
    double y, nrm = 0.0;
    switch (mode) {
        case AMGT_SWEEP_J: y = px + a.omega * pd * (pb - t); break;
        case AMGT_SWEEP_JR: {
            const double res = pb - t;
            y = px + a.omega * pd * res;
            nrm = res * res;
            break;
        }
        case AMGT_SWEEP_RN:
            y = pb - t;
            nrm = y * y;
            break;
        default: y = pb - t;
    }
    st.y[out_i] = y;
    return nrm;
}

struct TmPlan {
    const int64_t* chunk_t;  // [nchunks+1] first tile of each chunk
    const int32_t* xr;       // [nchunks * TM_XR] x runs
};

// producer: one chunk step k (its items into slots; P: the step's descriptors, loaded earlier)
__device__ __forceinline__ void tm_produce(const SweepArgs& a, unsigned k, const int32_t (*desc)[32], int64_t& i, char* slots,
                                           uint64_t* full, uint64_t* empty, TmMeta* meta, int64_t D, int lane,
                                           unsigned long long* pst) {
#pragma unroll 1
        for (int s = 0; s < AMGT_SWEEP_MAX_STAGES; ++s) {
            const int64_t c = (int64_t)k - (int64_t)s * D;
            if (s >= a.nst || c < 0 || c >= a.nchunks) continue;
            const int32_t* f = desc[s];
            const int64_t tb = f[0], te = f[1];
#if SW_STATS
            const long long tw0 = clock64();
#endif
            if (s > 0) {  // stage s-1 done on the column groups [clo, chi] of chunk c
                const int64_t g0 = f[2], g1 = f[3];
                const uint32_t* cnt = a.cnt + (int64_t)(s - 1) * a.ngroups;
                const uint32_t ep = sw_ep(a, s - 1);
                for (int64_t g = g0 + lane; g <= g1; g += 32) {
                    const uint32_t target = ep * (uint32_t)min((int64_t)SW_GROUP, a.nchunks - g * SW_GROUP);
                    while (ld_relaxed_u32(cnt + g) < target) __nanosleep(32);
                }
                fence_acq_rel_gpu();
                asm volatile("fence.proxy.async.global;" ::: "memory");  // x is read by the bulk copies
                __syncwarp();
            }
#if SW_STATS
            const long long tw1 = clock64();
#endif
            const int slot = (int)(i % TM_NS);
            if (i >= TM_NS) mbar_wait(&empty[slot], (uint32_t)(((i / TM_NS) & 1) ^ 1));
#if SW_STATS
            const long long tw2 = clock64();
            pst[2] += tw1 - tw0;
            pst[1] += tw2 - tw1;
#endif
            const TmSlot sl = tm_slot(slots, slot);
            const int nrows = (int)min((int64_t)SW_CHUNK, a.BR - c * SW_CHUNK);
            const int64_t nt = te - tb;
            const int nrun = f[4];
            const int lr = lane < TM_NRUN ? lane : TM_NRUN - 1;  // lane r: run r
            const int32_t rs = f[5 + lr];
            const int32_t rl = f[5 + TM_NRUN + lr];
            // slot offsets of the runs: exclusive prefix over the lanes < nrun
            int32_t ro = lane < nrun ? rl : 0;
            for (int d = 1; d < 32; d <<= 1) {
                const int32_t o = __shfl_up_sync(0xffffffffu, ro, d);
                if (lane >= d) ro += o;
            }
            ro -= lane < nrun ? rl : 0;
            const bool direct = nt > TM_CAP;
            const bool xin = nrun > 0;  // the plan only keeps runs that fit TM_XCAP
            uint32_t bytes = 0;
#if SW_STATS
            const long long tw3 = clock64();
#endif
            if (lane < nrun && xin) {
                meta[slot].rs[lane] = rs;
                meta[slot].rl[lane] = rl;
                meta[slot].ro[lane] = ro;
                bulk_g2s(sl.x + 4 * ro, sw_st(a, s).x + 4 * (int64_t)rs, (uint32_t)rl * 32u, &full[slot]);
                bytes += (uint32_t)rl * 32u;
            }
            for (int d = 16; d; d >>= 1) bytes += __shfl_xor_sync(0xffffffffu, bytes, d);
            if (lane == 0) {
                TmMeta& m = meta[slot];
                m.c = c;
                m.tbase = tb;
                m.s = s;
                m.nrows = nrows;
                m.direct = direct;
                m.nrun = xin ? nrun : 0;
                m.idx_off = m.map_off = 0;
                // row pointers: the first (nrows+1) rounded down to an even count by bulk
                // copy (16-byte granules, never past the array), the last one from the plan
                bulk_g2s(sl.b, a.b + 4 * SW_CHUNK * c, (uint32_t)(4 * nrows * 8), &full[slot]);
                bytes += (uint32_t)(4 * nrows * 8);
                const int md = sw_st(a, s).mode;
                if (md == AMGT_SWEEP_J || md == AMGT_SWEEP_JR) {
                    bulk_g2s(sl.dinv, a.dinv + 4 * SW_CHUNK * c, (uint32_t)(4 * nrows * 8), &full[slot]);
                    bytes += (uint32_t)(4 * nrows * 8);
                }
                const int np = (nrows + 1) & ~1;
                bulk_g2s(sl.ptr, a.bptr + c * SW_CHUNK, (uint32_t)np * 8u, &full[slot]);
                bytes += (uint32_t)np * 8u;
                sl.ptr[nrows] = te;
                if (!direct && nt > 0) {
                    const uintptr_t i0 = reinterpret_cast<uintptr_t>(a.bidx + tb) & ~uintptr_t(15);
                    const uintptr_t i1 = (reinterpret_cast<uintptr_t>(a.bidx + te) + 15) & ~uintptr_t(15);
                    const uintptr_t m0 = reinterpret_cast<uintptr_t>(a.bmap + tb) & ~uintptr_t(15);
                    const uintptr_t m1 = (reinterpret_cast<uintptr_t>(a.bmap + te) + 15) & ~uintptr_t(15);
                    m.idx_off = (int32_t)(reinterpret_cast<uintptr_t>(a.bidx + tb) - i0);
                    m.map_off = (int32_t)(reinterpret_cast<uintptr_t>(a.bmap + tb) - m0);
                    bulk_g2s(sl.val, a.bval + 16 * tb, (uint32_t)(nt * 128), &full[slot]);
                    bulk_g2s(sl.idx, reinterpret_cast<const void*>(i0), (uint32_t)(i1 - i0), &full[slot]);
                    bulk_g2s(sl.map, reinterpret_cast<const void*>(m0), (uint32_t)(m1 - m0), &full[slot]);
                    bytes += (uint32_t)(nt * 128 + (i1 - i0) + (m1 - m0));
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive_tx(&full[slot], bytes);
            __syncwarp();
#if SW_STATS
            pst[0] += clock64() - tw3;  // issue time (copies, meta, arrive)
#endif
            ++i;
        }
}

__global__ void __launch_bounds__(TM_THREADS, 1) k_sweep_tma(SweepArgs a, TmPlan tp) {
    extern __shared__ __align__(128) char smem[];
    __shared__ uint64_t full[TM_NS], empty[TM_NS];
    __shared__ TmMeta meta[TM_NS];
    __shared__ int32_t desc[3][AMGT_SWEEP_MAX_STAGES][32];  // producer descriptor ring
    __shared__ double red[TM_NG][TM_GW];
    __shared__ bool s_last;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    char* slots = reinterpret_cast<char*>((reinterpret_cast<uintptr_t>(smem) + 127) & ~uintptr_t(127));
    if (threadIdx.x == 0) {
        for (int i = 0; i < TM_NS; ++i) {
            mbar_init(&full[i], 1);
            mbar_init(&empty[i], 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const int64_t D = a.dev->D;
    const int64_t K = a.nchunks + (int64_t)(a.nst - 1) * D;
    if (warp == 0) {
        // ------------------------------------------------------------ producer
        int64_t i = 0;  // items produced
        unsigned k = 0, kn = 0;
        if (lane == 0) {
            k = atomicAdd(&a.dev->ctr[0], 1u);
            kn = atomicAdd(&a.dev->ctr[0], 1u);
        }
        k = __shfl_sync(0xffffffffu, k, 0);
        unsigned long long pst[3] = {0, 0, 0};  // SW_STATS: total, empty waits, dependency waits
#if SW_STATS
        const long long tp0 = clock64();
#endif
        // three claims and two descriptor sets ahead: ring of three shared-memory entries
        // filled by cp.async; the entry of step n is waited for (wait_group 1) two steps after
        // it was requested
        unsigned k1 = kn, k2 = 0;
        if (lane == 0) k2 = atomicAdd(&a.dev->ctr[0], 1u);
        k1 = __shfl_sync(0xffffffffu, k1, 0);
        k2 = __shfl_sync(0xffffffffu, k2, 0);
        tm_prefetch(a, tp.chunk_t, tp.xr, (int64_t)k, D, lane, desc[0]);
        tm_prefetch(a, tp.chunk_t, tp.xr, (int64_t)k1, D, lane, desc[1]);
        for (int r = 0; (int64_t)k < K; r = (r == 2) ? 0 : r + 1) {
            tm_prefetch(a, tp.chunk_t, tp.xr, (int64_t)k2, D, lane, desc[r == 0 ? 2 : r - 1]);
            unsigned k3 = 0xffffffffu;
            if (lane == 0 && (int64_t)k2 < K) k3 = atomicAdd(&a.dev->ctr[0], 1u);
            asm volatile("cp.async.wait_group 2;" ::: "memory");  // entry r (two groups older) landed
            __syncwarp();
            tm_produce(a, k, desc[r], i, slots, full, empty, meta, D, lane, pst);
            __syncwarp();  // entry r is refilled two steps later
            k = k1;
            k1 = k2;
            k2 = __shfl_sync(0xffffffffu, k3, 0);
        }
        asm volatile("cp.async.wait_all;" ::: "memory");
#if SW_STATS
        atomicAdd(&a.dev->stats[5], lane == 0 ? (unsigned long long)(clock64() - tp0) : 0ull);
        if (lane == 0)
            for (int j = 0; j < 3; ++j) atomicAdd(&a.dev->stats[j], pst[j]);
#endif
        // one stop item per consumer group
        for (int g = 0; g < TM_NG; ++g) {
            const int slot = (int)(i % TM_NS);
            if (i >= TM_NS) mbar_wait(&empty[slot], (uint32_t)(((i / TM_NS) & 1) ^ 1));
            if (lane == 0) {
                meta[slot].c = -1;
                mbar_arrive_tx(&full[slot], 0);
            }
            __syncwarp();
            ++i;
        }
    } else {
        // ------------------------------------------------------------ consumers
        const int cw = warp - 1;
        const int g = cw / TM_GW, wg = cw % TM_GW;    // group, warp within the group
        const int r = wg * 8 + (lane >> 2), q = lane & 3;
        unsigned long long cst[3] = {0, 0, 0};  // SW_STATS: full waits, compute, items
        for (int64_t i = g;; i += TM_NG) {
            const int slot = (int)(i % TM_NS);
#if SW_STATS
            const long long tc0 = clock64();
#endif
            mbar_wait(&full[slot], (uint32_t)((i / TM_NS) & 1));
#if SW_STATS
            const long long tc1 = clock64();
            cst[0] += tc1 - tc0;
#endif
            const TmMeta& m = meta[slot];
            if (m.c < 0) break;
            const TmSlot sl = tm_slot(slots, slot);
            const SweepStageDev st = sw_st(a, m.s);
            // one instantiation (L2-coherent loads for the rare global fallbacks): code size
            const double nrm = tm_row<true>(a, st, m, sl, r, q);
            const bool norm = st.mode == AMGT_SWEEP_JR || st.mode == AMGT_SWEEP_RN;
            if (norm) {
                double v = nrm;
                for (int d = 16; d; d >>= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
                if (lane == 0) red[g][wg] = v;
            }
            const int64_t mc = m.c;
            const int ms = m.s;
            bar_named(1 + g, 32 * TM_GW);  // the group's rows written, slot no longer read
            // the publishing lane rotates over the group's warps: its release fence waits for
            // the group's stores, and rotating spreads that stall over TM_GW items
            if (wg == (int)((i / TM_NG) % TM_GW) && lane == 0) {
                mbar_arrive(&empty[slot]);
                if (norm) {
                    double p = 0.0;
                    for (int w = 0; w < TM_GW; ++w) p += red[g][w];
                    a.partial[mc] = p;
                }
                red_release_add(a.cnt + (int64_t)ms * a.ngroups + mc / SW_GROUP, 1u);
            }
#if SW_STATS
            cst[1] += clock64() - tc1;
            cst[2] += 1;
#endif
        }
#if SW_STATS
        if (wg == 0 && lane == 0)
            for (int j = 0; j < 2; ++j) atomicAdd(&a.dev->stats[3 + j], cst[j]);
#endif
    }
    __syncthreads();
    // exit ticket: the last CTA re-arms the counters and sums the norm partials in order
    if (threadIdx.x == 0) {
        __threadfence();
        s_last = atomicAdd(&a.dev->ctr[1], 1u) == gridDim.x - 1;
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    if (a.norm_out && threadIdx.x < 256) {
        __shared__ double sh[8];
        double v = 0.0;
        for (int64_t k = threadIdx.x; k < a.nchunks; k += 256) v += __ldcg(a.partial + k);
        for (int d = 16; d; d >>= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
        if (lane == 0) sh[warp] = v;
        bar_named(1, 256);
        if (threadIdx.x == 0) {
            double tot = 0.0;
            for (int w = 0; w < 8; ++w) tot += sh[w];
            *a.norm_out = tot;
        }
    }
    if (threadIdx.x == 0) {
        a.dev->ctr[0] = 0u;
        a.dev->ctr[1] = 0u;
    }
}

// Plan: first tile of every chunk and its x runs (column blocks of the chunk's tiles, sorted,
// runs separated by gaps of <= 16 blocks merged; kept when <= TM_NRUN runs of <= TM_XCAP
// blocks in total, else n = 0: x read from global memory).  One CTA per chunk.
__global__ void __launch_bounds__(256) k_sweep_xruns(int64_t BR, int64_t nchunks, const int64_t* __restrict__ bptr,
                                                     const int32_t* __restrict__ bidx, int64_t* __restrict__ chunk_t,
                                                     int32_t* __restrict__ xr) {
    constexpr int WIN = 1 << 15;  // column-block window of the bitmap
    __shared__ uint32_t bm[WIN / 32];
    __shared__ int32_t smin, smax;
    const int64_t c = blockIdx.x;
    const int64_t r0 = c * SW_CHUNK, r1 = min(BR, r0 + SW_CHUNK);
    const int64_t t0 = bptr[r0], t1 = bptr[r1];
    if (threadIdx.x == 0) {
        chunk_t[c] = t0;
        if (c == nchunks - 1) chunk_t[nchunks] = t1;
        smin = INT32_MAX;
        smax = -1;
    }
    __syncthreads();
    int32_t lo = INT32_MAX, hi = -1;
    for (int64_t t = t0 + threadIdx.x; t < t1; t += blockDim.x) {
        const int32_t J = bidx[t];
        lo = min(lo, J);
        hi = max(hi, J);
    }
    atomicMin(&smin, lo);
    atomicMax(&smax, hi);
    __syncthreads();
    int32_t* rec = xr + c * TM_XR;
    const int32_t mn = smin, mx = smax;
    if (mx < 0 || mx - mn >= WIN) {
        if (threadIdx.x == 0) rec[0] = 0;
        return;
    }
    const int nw = (mx - mn) / 32 + 1;
    for (int w = threadIdx.x; w < nw; w += blockDim.x) bm[w] = 0u;
    __syncthreads();
    for (int64_t t = t0 + threadIdx.x; t < t1; t += blockDim.x) {
        const int32_t d = bidx[t] - mn;
        atomicOr(&bm[d >> 5], 1u << (d & 31));
    }
    __syncthreads();
    if (threadIdx.x != 0) return;
    int n = 0, total = 0;
    int32_t cs = -1, ce = -1;  // current run [cs, ce]
    bool ok = true;
    for (int w = 0; w < nw && ok; ++w) {
        uint32_t bits = bm[w];
        while (bits) {
            const int32_t J = mn + 32 * w + __ffs(bits) - 1;
            bits &= bits - 1;
            if (cs >= 0 && J - ce <= 17) {
                ce = J;
            } else {
                if (cs >= 0) {
                    if (n == TM_NRUN) { ok = false; break; }
                    rec[1 + n] = cs;
                    rec[1 + TM_NRUN + n] = ce - cs + 1;
                    total += ce - cs + 1;
                    ++n;
                }
                cs = ce = J;
            }
        }
    }
    if (ok && cs >= 0) {
        if (n == TM_NRUN) ok = false;
        else {
            rec[1 + n] = cs;
            rec[1 + TM_NRUN + n] = ce - cs + 1;
            total += ce - cs + 1;
            ++n;
        }
    }
    rec[0] = (ok && total <= TM_XCAP) ? n : 0;
}

// column-chunk range of each chunk and the forward bandwidth
__global__ void k_sweep_plan(int64_t BR, int64_t nchunks, const int64_t* __restrict__ bptr,
                             const int32_t* __restrict__ bidx, int32_t* __restrict__ clo, int32_t* __restrict__ chi,
                             SweepDev* dev) {
    const int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= nchunks) return;
    int64_t lo = INT64_MAX, hi = -1;
    for (int64_t I = c * SW_CHUNK; I < (c + 1) * SW_CHUNK && I < BR; ++I) {
        const int64_t t0 = bptr[I], t1 = bptr[I + 1];
        if (t1 > t0) {
            lo = min(lo, (int64_t)bidx[t0]);
            hi = max(hi, (int64_t)bidx[t1 - 1]);
        }
    }
    if (hi < 0) {  // no tiles: reads nothing
        clo[c] = 1;
        chi[c] = 0;
        return;
    }
    clo[c] = (int32_t)(lo / SW_CHUNK / SW_GROUP);
    chi[c] = (int32_t)(hi / SW_CHUNK / SW_GROUP);
    const int fwd = (int)(hi / SW_CHUNK - c);
    if (fwd > 0) atomicMax(&dev->bw_fwd, fwd);
}

// D = forward bandwidth + SW_GROUP + extra, at most the chunk count (beyond it the stages simply run
// one after another)
__global__ void k_sweep_lag(SweepDev* dev, int64_t extra, int64_t nchunks) {
    // waits are per group of SW_GROUP chunks: a wait may cover up to SW_GROUP - 1 chunks past
    // the bandwidth, so D > bw_fwd + SW_GROUP - 1 keeps every awaited item earlier
    const int64_t Dmin = (int64_t)dev->bw_fwd + SW_GROUP;
    const int64_t D = Dmin + extra;
    dev->D = D < nchunks ? D : (nchunks > Dmin ? nchunks : Dmin);
}

static int sweep_ctas_per_sm() {
    const char* e = getenv("AMGT_SWEEP_CTAS");
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_sweep, SW_THREADS, 0);
    int want = e ? atoi(e) : 4;
    if (want < 1) want = 1;
    return occ > 0 ? (want < occ ? want : occ) : 1;
}

// extra lag beyond the bandwidth: about the items in flight (one per resident CTA, nst
// items per chunk step) so later stages rarely wait, small enough that the A tiles of the
// 2 D chunks between stage 0 and the last stage stay in L2
static int64_t sweep_lag_extra(int grid, bool tma) {
    const char* e = getenv("AMGT_SWEEP_LAG");
    return e ? (int64_t)atoll(e) : (int64_t)(tma ? 3 * grid : grid / 2);
}

static bool sweep_use_tma() {
    const char* e = getenv("AMGT_SWEEP_IMPL");
    return !(e && !strcmp(e, "ldg"));
}

}  // namespace amgt

using namespace amgt;

struct amgt_sweep_plan {
    SweepPlanImpl p;
};

static void sweep_plan_release(amgt_sweep_plan* P, cudaStream_t s) {
    if (!P) return;
    SweepPlanImpl& p = P->p;
    Alloc a{p.has_al ? &p.al : nullptr, s};
    a.put(p.clo, p.nchunks * sizeof(int32_t));
    a.put(p.chi, p.nchunks * sizeof(int32_t));
    a.put(p.cnt, AMGT_SWEEP_MAX_STAGES * p.ngroups * sizeof(uint32_t));
    a.put(p.partial, p.nchunks * sizeof(double));
    a.put(p.chunk_t, (p.nchunks + 1) * sizeof(int64_t));
    a.put(p.xr, p.nchunks * TM_XR * sizeof(int32_t));
    a.put(p.dev, sizeof(SweepDev));
    delete P;
}

extern "C" {

amgt_status amgt_sweep_plan_create(const amgt_mbsr* A, const amgt_allocator* al, void* stream,
                                   amgt_sweep_plan** out) {
    if (!A || !out) return fail(AMGT_ERR_ARG, "amgt_sweep_plan_create: null argument");
    *out = nullptr;
    if (A->prec != AMGT_FP64) return fail(AMGT_ERR_UNSUPPORTED, "amgt_sweep_plan_create: FP64 operators only");
    if (A->m != A->n) return fail(AMGT_ERR_ARG, "amgt_sweep_plan_create: operator must be square");
    cudaStream_t s = (cudaStream_t)stream;
    amgt_sweep_plan* P = new amgt_sweep_plan();
    SweepPlanImpl& p = P->p;
    if (al) { p.al = *al; p.has_al = true; }
    Alloc a{p.has_al ? &p.al : nullptr, s};
    p.m = A->m;
    p.BR = A->blc_row;
    p.T = A->blc_num;
    p.nchunks = ceil_div(A->blc_row, SW_CHUNK);
    p.tma = sweep_use_tma() && A->blc_num < ((int64_t)1 << 31);  // 32-bit tile offsets in the TMA descriptors
    if (p.tma) {
        AMGT_CUDA(dyn_smem(k_sweep_tma, TM_SMEM));
        p.grid = num_sms();
    } else {
        p.grid = num_sms() * sweep_ctas_per_sm();
    }
    const int64_t nc = p.nchunks > 0 ? p.nchunks : 1;
    p.clo = (int32_t*)a.get(nc * sizeof(int32_t));
    p.chi = (int32_t*)a.get(nc * sizeof(int32_t));
    p.ngroups = ceil_div(nc, SW_GROUP);
    p.cnt = (uint32_t*)a.get(AMGT_SWEEP_MAX_STAGES * p.ngroups * sizeof(uint32_t));
    p.partial = (double*)a.get(nc * sizeof(double));
    if (p.tma) {
        p.chunk_t = (int64_t*)a.get((nc + 1) * sizeof(int64_t));
        p.xr = (int32_t*)a.get(nc * TM_XR * sizeof(int32_t));
        if (!p.chunk_t || !p.xr) {
            sweep_plan_release(P, s);
            return fail(AMGT_ERR_ALLOC, "amgt_sweep_plan_create: allocation failed");
        }
    }
    p.dev = (SweepDev*)a.get(sizeof(SweepDev));
    p.nchunks = nc;
    if (!p.clo || !p.chi || !p.cnt || !p.partial || !p.dev) {
        sweep_plan_release(P, s);
        return fail(AMGT_ERR_ALLOC, "amgt_sweep_plan_create: allocation failed");
    }
    cudaMemsetAsync(p.cnt, 0, AMGT_SWEEP_MAX_STAGES * p.ngroups * sizeof(uint32_t), s);
    cudaMemsetAsync(p.partial, 0, nc * sizeof(double), s);
    cudaMemsetAsync(p.dev, 0, sizeof(SweepDev), s);
    cudaMemsetAsync(p.clo, 0, nc * sizeof(int32_t), s);
    cudaMemsetAsync(p.chi, 0, nc * sizeof(int32_t), s);
    if (A->blc_row > 0) {
        k_sweep_plan<<<(unsigned)ceil_div(p.nchunks, 128), 128, 0, s>>>(A->blc_row, p.nchunks, A->blc_ptr, A->blc_idx,
                                                                       p.clo, p.chi, p.dev);
        count_launch();
        if (p.tma) {
            k_sweep_xruns<<<(unsigned)p.nchunks, 256, 0, s>>>(A->blc_row, p.nchunks, A->blc_ptr, A->blc_idx, p.chunk_t,
                                                            p.xr);
            count_launch();
        }
    }
    k_sweep_lag<<<1, 1, 0, s>>>(p.dev, sweep_lag_extra(p.grid, p.tma), p.nchunks);
    count_launch();
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        sweep_plan_release(P, s);
        return fail(AMGT_ERR_CUDA, "amgt_sweep_plan_create: %s", cudaGetErrorString(e));
    }
    *out = P;
    return AMGT_OK;
}

amgt_status amgt_sweep_plan_stats(amgt_sweep_plan* P, uint64_t* out6_host, void* stream) {
    if (!P || !out6_host) return fail(AMGT_ERR_ARG, "amgt_sweep_plan_stats: null argument");
    cudaStream_t s = (cudaStream_t)stream;
    AMGT_CUDA(cudaMemcpyAsync(out6_host, P->p.dev->stats, 6 * sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaMemsetAsync(P->p.dev->stats, 0, 6 * sizeof(uint64_t), s));
    AMGT_CUDA(cudaStreamSynchronize(s));
    return AMGT_OK;
}

amgt_status amgt_sweep_plan_destroy(amgt_sweep_plan* P, void* stream) {
    sweep_plan_release(P, (cudaStream_t)stream);
    return AMGT_OK;
}

amgt_status amgt_spmv_sweeps(amgt_sweep_plan* P, const amgt_mbsr* A, int nstages, const amgt_sweep_stage* st,
                             const void* b, const void* dinv, double omega, double* norm_dev, void* stream) {
    if (!P || !A || !st || !b) return fail(AMGT_ERR_ARG, "amgt_spmv_sweeps: null argument");
    SweepPlanImpl& p = P->p;
    if (A->prec != AMGT_FP64 || A->blc_row != p.BR || A->blc_num != p.T || A->m != p.m)
        return fail(AMGT_ERR_ARG, "amgt_spmv_sweeps: operator does not match the plan");
    if (nstages < 1 || nstages > AMGT_SWEEP_MAX_STAGES)
        return fail(AMGT_ERR_ARG, "amgt_spmv_sweeps: 1..%d stages", AMGT_SWEEP_MAX_STAGES);
    int nnorm = 0;
    SweepArgs a{};
    for (int s = 0; s < nstages; ++s) {
        const int md = st[s].mode;
        if (md != AMGT_SWEEP_J && md != AMGT_SWEEP_JR && md != AMGT_SWEEP_R && md != AMGT_SWEEP_RN)
            return fail(AMGT_ERR_ARG, "amgt_spmv_sweeps: stage %d has mode %d", s, md);
        if (!st[s].x || !st[s].y || st[s].x == st[s].y)
            return fail(AMGT_ERR_ARG, "amgt_spmv_sweeps: stage %d needs distinct x and y", s);
        if ((md == AMGT_SWEEP_J || md == AMGT_SWEEP_JR) && !dinv)
            return fail(AMGT_ERR_ARG, "amgt_spmv_sweeps: Jacobi stage without dinv");
        if (md == AMGT_SWEEP_JR || md == AMGT_SWEEP_RN) ++nnorm;
        for (int r = 0; r < s; ++r)  // no stage may overwrite what an earlier stage still reads
            if (st[s].y == st[r].x || st[s].y == st[r].y)
                return fail(AMGT_ERR_ARG, "amgt_spmv_sweeps: stage %d output aliases stage %d", s, r);
        if (s > 0 && st[s].x != st[s - 1].y)
            return fail(AMGT_ERR_ARG, "amgt_spmv_sweeps: stage %d must read stage %d's output", s, s - 1);
        a.st[s] = SweepStageDev{(const double*)st[s].x, (double*)st[s].y, md};
    }
    if (nnorm > 1) return fail(AMGT_ERR_ARG, "amgt_spmv_sweeps: at most one norm stage");
    if (nnorm == 1 && !norm_dev) return fail(AMGT_ERR_ARG, "amgt_spmv_sweeps: norm stage without norm_dev");
    cudaStream_t s = (cudaStream_t)stream;
    if (A->blc_row == 0) return AMGT_OK;
    if (p.ep[0] >= (1u << 28)) {  // keep ep * SW_GROUP below 2^32: restart the counters
        cudaMemsetAsync(p.cnt, 0, AMGT_SWEEP_MAX_STAGES * p.ngroups * sizeof(uint32_t), s);
        for (uint32_t& e : p.ep) e = 0;
    }
    for (int k = 0; k < nstages; ++k) a.ep[k] = ++p.ep[k];
    a.BR = A->blc_row;
    a.nchunks = p.nchunks;
    a.bptr = A->blc_ptr;
    a.bidx = A->blc_idx;
    a.bmap = A->blc_map;
    a.bval = (const double*)A->blc_val;
    a.b = (const double*)b;
    a.dinv = (const double*)dinv;
    a.omega = omega;
    a.nst = nstages;
    a.clo = p.clo;
    a.chi = p.chi;
    a.cnt = p.cnt;
    a.ngroups = p.ngroups;
    a.dev = p.dev;
    a.partial = p.partial;
    a.norm_out = nnorm ? norm_dev : nullptr;
    // algorithmic HBM bytes of the pass: A once, stage 0's x, b, dinv once, every stage's output
    const double bytes = (double)A->blc_num * (16 * 8 + 6) + (double)(A->blc_row + 1) * 8 +
                         8.0 * 4 * A->blc_row * (3 + nstages);
    TimerScope ts(TC_SPMV_L1, bytes, s);
    if (p.tma) k_sweep_tma<<<p.grid, TM_THREADS, TM_SMEM, s>>>(a, TmPlan{p.chunk_t, p.xr});
    else k_sweep<<<p.grid, SW_THREADS, 0, s>>>(a);
    AMGT_LAUNCHED();
    return AMGT_OK;
}

}  // extern "C"
