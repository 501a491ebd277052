// runtime.cu — error reporting, allocator glue, device prefix sum, timing/launch counters.
#include <atomic>
#include <ctime>
#include <cstdlib>
#include <cstdarg>
#include <mutex>
#include <unordered_map>
#include <vector>

#include "common.cuh"

namespace amgt {

static thread_local char g_err[1024] = "";

void set_error(const char* fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
}

amgt_status fail(amgt_status st, const char* fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return st;
}

void* Alloc::get(size_t bytes) {
    if (bytes == 0) bytes = 16;
    if (al && al->alloc) return al->alloc(bytes, (void*)s, al->ctx);
    void* p = nullptr;
    if (cudaMallocAsync(&p, bytes, s) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    return p;
}

void Alloc::put(void* p, size_t bytes) {
    if (!p) return;
    if (bytes == 0) bytes = 16;
    if (al && al->free) {
        al->free(p, bytes, (void*)s, al->ctx);
        return;
    }
    cudaFreeAsync(p, s);
}

// Scratch comes from a library-owned stream-ordered pool (not the device default pool, which
// torch or the caller may configure).  Freed scratch stays cached up to a release threshold
// (AMGT_SCRATCH_CACHE_MB, default 4096 MB); beyond it the pool returns memory to the device at
// the next synchronisation, so large transient buffers (SpGEMM candidate lists, hash tables)
// do not stay reserved for the life of the process.
static cudaMemPool_t scratch_pool() {
    static std::mutex mu;
    static cudaMemPool_t pools[64] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) return nullptr;
    std::lock_guard<std::mutex> lk(mu);
    if (!pools[dev]) {
        cudaMemPoolProps props = {};
        props.allocType = cudaMemAllocationTypePinned;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = dev;
        cudaMemPool_t p = nullptr;
        if (cudaMemPoolCreate(&p, &props) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        const char* e = getenv("AMGT_SCRATCH_CACHE_MB");
        uint64_t thr = (uint64_t)(e ? atoll(e) : 4096) << 20;
        cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
        pools[dev] = p;
    }
    return pools[dev];
}

void* scratch_get(size_t bytes, cudaStream_t s) {
    void* p = nullptr;
    cudaMemPool_t pool = scratch_pool();
    const cudaError_t e = pool ? cudaMallocFromPoolAsync(&p, bytes ? bytes : 16, pool, s)
                               : cudaMallocAsync(&p, bytes ? bytes : 16, s);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    return p;
}

void scratch_put(void* p, cudaStream_t s) {
    if (p) cudaFreeAsync(p, s);
}

size_t prec_bytes(amgt_prec p) { return p == AMGT_FP64 ? 8 : (p == AMGT_FP32 ? 4 : 2); }

int num_sms() {
    static int n = 0;
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

cudaError_t dyn_smem_optin(const void* kern, size_t bytes) {
    // (no shortcut at <= 48 KB: the default limit counts the kernel's static shared memory too)
    if (bytes == 0) return cudaSuccess;
    static std::mutex mu;
    static std::unordered_map<const void*, size_t> cur;
    std::lock_guard<std::mutex> g(mu);
    size_t& c = cur[kern];
    if (c >= bytes) return cudaSuccess;
    const cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
    if (e == cudaSuccess) c = bytes;
    return e;
}

// Tensor-core routing thresholds on POPCOUNT(mapA).  The paper uses 10 (L157); north_star asks
// for the mma route only where it beats CUDA cores.  Measured on B200 (R9/R10;
// tools/spgemm_bench.py): DMMA m8n8k4 issues at the FP64 FMA rate and both kernels are
// memory/latency bound, so the route is slower at every threshold (FP64 SpGEMM +6..150%,
// FP16 HMMA +0..15%, SpMV ~same) -> default 17 (CUDA cores); amgt_set_tc_threshold(10, 10)
// restores the paper's routing.
int g_tc_thr_spgemm = 17;
int g_tc_thr_spmv = 17;

// ------------------------------------------------------------------ scan
// Block-wide exclusive scan: 1024 threads x 8 items = 8192 items per block.
#ifndef AMGT_SCAN_T  // experiments: -DAMGT_SCAN_T=.. -DAMGT_SCAN_I=.. (AMGT_NVCC_EXTRA)
#define AMGT_SCAN_T 256
#endif
#ifndef AMGT_SCAN_I
#define AMGT_SCAN_I 8
#endif
constexpr int SCAN_T = AMGT_SCAN_T, SCAN_I = AMGT_SCAN_I, SCAN_TILE = SCAN_T * SCAN_I;  // 2048 items per CTA (4096 / 8192 measured equal)

__device__ __forceinline__ int64_t block_excl_scan(int64_t v, int64_t* sh_warp, int64_t* total) {
    int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int64_t x = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        int64_t y = __shfl_up_sync(0xffffffffu, x, d);
        if (lane >= d) x += y;
    }
    if (lane == 31) sh_warp[w] = x;
    __syncthreads();
    if (w == 0) {
        int64_t s = (lane < (int)(blockDim.x >> 5)) ? sh_warp[lane] : 0;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            int64_t y = __shfl_up_sync(0xffffffffu, s, d);
            if (lane >= d) s += y;
        }
        sh_warp[lane] = s;  // inclusive warp-sum prefix
    }
    __syncthreads();
    int64_t base = (w > 0) ? sh_warp[w - 1] : 0;
    if (total) *total = sh_warp[(blockDim.x >> 5) - 1];
    int64_t r = base + x - v;
    __syncthreads();
    return r;
}

// Single-pass exclusive scan (decoupled look-back): one launch.  Each CTA takes a ticket
// (logical tile order = scheduling order, so every predecessor is resident or done), publishes
// its tile aggregate, then warp 0 looks back over 32 predecessors at a time, summing
// aggregates until it meets a published inclusive prefix; the CTA publishes its own inclusive
// prefix and scans its tile.  st = [ticket | one status word per tile], zeroed by the host;
// status word = flag << 62 | value (flag 1 aggregate, 2 inclusive prefix; value < 2^62).
// Optionally also the maximum input (dmax, atomicMax).
constexpr unsigned long long ST_AGG = 1ull << 62, ST_INC = 2ull << 62, ST_VAL = (1ull << 62) - 1;
__device__ __forceinline__ void st_release(unsigned long long* p, unsigned long long v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_acquire(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__global__ void __launch_bounds__(SCAN_T) k_scan(const int64_t* __restrict__ in, int64_t n,
                                                 unsigned long long* __restrict__ st, int64_t* __restrict__ out,
                                                 unsigned long long* __restrict__ dmax) {
    __shared__ int64_t sh[32];
    __shared__ int64_t s_tile, s_excl;
    if (threadIdx.x == 0) s_tile = (int64_t)atomicAdd(st, 1ull);
    __syncthreads();
    const int64_t tile = s_tile;
    const int64_t base = tile * SCAN_TILE + (int64_t)threadIdx.x * SCAN_I;
    int64_t v[SCAN_I];
    int64_t s = 0, mx = 0;
#pragma unroll
    for (int i = 0; i < SCAN_I; ++i) {
        v[i] = (base + i < n) ? in[base + i] : 0;
        s += v[i];
        mx = max(mx, v[i]);
    }
    int64_t tot;
    const int64_t off = block_excl_scan(s, sh, &tot);
    unsigned long long* status = st + 1;
    if (threadIdx.x == 0) st_release(status + tile, (tile == 0 ? ST_INC : ST_AGG) | (unsigned long long)tot);
    if (threadIdx.x < 32) {
        const int lane = threadIdx.x;
        int64_t excl = 0;
        int64_t j = tile - 1;  // look back over status[j - lane], j decreasing by 32
        while (j >= 0) {
            const int64_t k = j - lane;
            unsigned long long w = k >= 0 ? ld_acquire(status + k) : ST_INC;  // before tile 0: prefix 0
            while (__any_sync(0xffffffffu, (w >> 62) == 0)) {
                if ((w >> 62) == 0) w = ld_acquire(status + k);
            }
            const unsigned inc = __ballot_sync(0xffffffffu, (w >> 62) == 2);
            const int stop = inc ? __ffs(inc) - 1 : 32;  // first lane (nearest tile) with a prefix
            int64_t val = (lane <= stop && k >= 0) ? (int64_t)(w & ST_VAL) : 0;
#pragma unroll
            for (int d = 16; d; d >>= 1) val += __shfl_xor_sync(0xffffffffu, val, d);
            excl += val;
            if (inc) break;
            j -= 32;
        }
        if (lane == 0) {
            s_excl = excl;
            if (tile > 0) st_release(status + tile, ST_INC | (unsigned long long)(excl + tot));
        }
    }
    __syncthreads();
    int64_t o = s_excl + off;
    if (tile == 0 && threadIdx.x == 0) out[0] = 0;
#pragma unroll
    for (int i = 0; i < SCAN_I; ++i) {
        o += v[i];
        if (base + i < n) out[base + i + 1] = o;
    }
    if (dmax) {
        for (int d = 16; d; d >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, d));
        if ((threadIdx.x & 31) == 0 && mx > 0) atomicMax(dmax, (unsigned long long)mx);
    }
}

amgt_status scan_exclusive(const int64_t* in, int64_t* out, int64_t n, Alloc& a, cudaStream_t s,
                           unsigned long long* dmax) {
    if (n <= 0) {
        AMGT_CUDA(cudaMemsetAsync(out, 0, sizeof(int64_t), s));
        return AMGT_OK;
    }
    const int64_t nb = ceil_div(n, SCAN_TILE);
    Scratch<unsigned long long> st;
    AMGT_TRY(st.init(a, nb + 1));
    AMGT_CUDA(cudaMemsetAsync(st.p, 0, (nb + 1) * sizeof(unsigned long long), s));
    k_scan<<<(unsigned)nb, SCAN_T, 0, s>>>(in, n, st.p, out, dmax);
    AMGT_LAUNCHED();
    return AMGT_OK;
}

// ------------------------------------------------------------------ instrumentation
static std::atomic<int64_t> g_launches{0};
static thread_local int g_pdl_depth = 0;
static bool pdl_allowed() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("AMGT_PDL");
        v = (e && e[0] == '0') ? 0 : 1;
    }
    return v == 1;
}
bool pdl_active() { return g_pdl_depth > 0 && pdl_allowed(); }
PdlScope::PdlScope() { ++g_pdl_depth; }
PdlScope::~PdlScope() { --g_pdl_depth; }

// AMGT_TRACE=1 (measurement only): named points; at each point the host time when the
// step's work was enqueued and, after a stream synchronisation, when the device finished it.
// (The synchronisations change the overlap; per-step device and host costs still separate.)
struct TracePt {
    const char* name;
    double enq_ms, done_ms;
};
static std::vector<TracePt> g_trace;
static bool trace_on() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("AMGT_TRACE");
        v = (e && e[0] == '1') ? 1 : 0;
    }
    return v == 1;
}
static double host_ms() {
    timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return ts.tv_sec * 1e3 + ts.tv_nsec * 1e-6;
}
static std::mutex g_trace_mu;  // loopback ranks trace from several threads
void trace_point(const char* name, cudaStream_t s) {
    if (!trace_on()) return;
    const double e = host_ms();
    cudaStreamSynchronize(s);
    std::lock_guard<std::mutex> lk(g_trace_mu);
    g_trace.push_back(TracePt{name, e, host_ms()});
}
void trace_dump() {
    if (!trace_on()) return;
    std::lock_guard<std::mutex> lk(g_trace_mu);
    if (g_trace.empty()) return;
    double prev = g_trace.front().done_ms;
    for (const TracePt& t : g_trace) {
        fprintf(stderr, "trace %-20s enqueue %8.3f ms  device-done %8.3f ms\n", t.name, t.enq_ms - prev,
                t.done_ms - t.enq_ms);
        prev = t.done_ms;
    }
    g_trace.clear();
}

// Small pinned host buffer (per thread, allocated once) for device values read back after a
// later synchronisation point instead of with a synchronisation of their own.
int64_t* pinned_slots() {
    static thread_local int64_t* p = nullptr;
    if (!p && cudaMallocHost(&p, PINNED_SLOTS * sizeof(int64_t)) != cudaSuccess) p = nullptr;
    return p;
}

void count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }
void count_launches(int64_t n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

struct TimerRec {
    int cls;
    double bytes;
    cudaEvent_t e0, e1;
};
static std::mutex g_tmu;
static unsigned g_timing = 0;  // bitmask of enabled timer classes
static std::vector<TimerRec> g_recs;
static std::vector<cudaEvent_t> g_pool;
static size_t g_used = 0;

static cudaEvent_t pool_event() {
    if (g_used < g_pool.size()) return g_pool[g_used++];
    cudaEvent_t e;
    cudaEventCreate(&e);
    g_pool.push_back(e);
    ++g_used;
    return e;
}

unsigned timing_mask() { return g_timing; }

static int g_sample_every = 1;  // time one scope in N of each class
static int64_t g_scope_count[AMGT_TIMER_CLASSES] = {};

TimerScope::TimerScope(int c, double b, cudaStream_t st) : cls(c), bytes(b), s(st), slot(-1) {
    if (!(g_timing & (1u << c))) return;
    std::lock_guard<std::mutex> lk(g_tmu);
    if (g_scope_count[c]++ % g_sample_every != 0) return;
    TimerRec r{c, b, pool_event(), pool_event()};
    cudaEventRecord(r.e0, s);
    g_recs.push_back(r);
    slot = (int)g_recs.size() - 1;
}

TimerScope::~TimerScope() {
    if (slot < 0) return;
    std::lock_guard<std::mutex> lk(g_tmu);
    g_recs[slot].bytes = bytes;
    cudaEventRecord(g_recs[slot].e1, s);
}

}  // namespace amgt

using namespace amgt;

extern "C" {

const char* amgt_last_error(void) { return amgt::g_err; }

const char* amgt_version(void) { return "amgt-b200 0.1 (sm_100a)"; }

amgt_status amgt_set_tc_threshold(int spgemm_threshold, int spmv_threshold) {
    if (spgemm_threshold < 0 || spgemm_threshold > 17 || spmv_threshold < 0 || spmv_threshold > 17)
        return fail(AMGT_ERR_ARG, "thresholds must be in [0, 17]");
    g_tc_thr_spgemm = spgemm_threshold;
    g_tc_thr_spmv = spmv_threshold;
    return AMGT_OK;
}

amgt_status amgt_timing_enable(int on) {
    std::lock_guard<std::mutex> lk(g_tmu);
    g_timing = on < 0 ? 0xFFu : (unsigned)on & 0xFFu;
    return AMGT_OK;
}

amgt_status amgt_timing_sample(int every) {
    if (every < 1) return fail(AMGT_ERR_ARG, "amgt_timing_sample: every must be >= 1");
    std::lock_guard<std::mutex> lk(g_tmu);
    g_sample_every = every;
    return AMGT_OK;
}

amgt_status amgt_timing_reset(void) {
    std::lock_guard<std::mutex> lk(g_tmu);
    for (int64_t& n : g_scope_count) n = 0;
    g_recs.clear();
    g_used = 0;
    g_launches.store(0);
    return AMGT_OK;
}

amgt_status amgt_timing_read(double* ms_total_host, int64_t* launches_host, double* bytes_host) {
    std::lock_guard<std::mutex> lk(g_tmu);
    for (int c = 0; c < AMGT_TIMER_CLASSES; ++c) {
        if (ms_total_host) ms_total_host[c] = 0;
        if (launches_host) launches_host[c] = 0;
        if (bytes_host) bytes_host[c] = 0;
    }
    for (auto& r : g_recs) {
        if (cudaEventSynchronize(r.e1) != cudaSuccess) return fail(AMGT_ERR_CUDA, "event sync failed");
        float ms = 0;
        cudaEventElapsedTime(&ms, r.e0, r.e1);
        if (ms_total_host) ms_total_host[r.cls] += ms;
        if (launches_host) launches_host[r.cls] += 1;
        if (bytes_host) bytes_host[r.cls] += r.bytes;
    }
    return AMGT_OK;
}

int64_t amgt_launch_count(void) { return g_launches.load(); }

}  // extern "C"
