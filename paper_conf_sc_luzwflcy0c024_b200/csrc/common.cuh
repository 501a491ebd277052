// common.cuh — internal helpers of libamgt (never installed; not part of the ABI).
#pragma once

#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <string>

#include "amgt.h"

namespace amgt {

// ------------------------------------------------------------------ errors
void set_error(const char* fmt, ...);
amgt_status fail(amgt_status st, const char* fmt, ...);

#define AMGT_CUDA(call)                                                                    \
    do {                                                                                   \
        cudaError_t e_ = (call);                                                           \
        if (e_ != cudaSuccess)                                                             \
            return ::amgt::fail(AMGT_ERR_CUDA, "%s:%d %s: %s", __FILE__, __LINE__, #call, \
                                cudaGetErrorString(e_));                                   \
    } while (0)

#define AMGT_LAUNCHED()                                                                          \
    do {                                                                                         \
        ::amgt::count_launch();                                                                  \
        cudaError_t e_ = cudaGetLastError();                                                     \
        if (e_ != cudaSuccess)                                                                   \
            return ::amgt::fail(AMGT_ERR_CUDA, "%s:%d launch: %s", __FILE__, __LINE__,           \
                                cudaGetErrorString(e_));                                         \
    } while (0)

// An error a previous CUDA call left pending in this host thread would be reported by the next
// launch check of a library call that did nothing wrong: name it at the entry point instead.
#define AMGT_NO_PENDING(fn)                                                                      \
    do {                                                                                         \
        cudaError_t e_ = cudaGetLastError();                                                     \
        if (e_ != cudaSuccess)                                                                   \
            return ::amgt::fail(AMGT_ERR_CUDA, "%s: CUDA error pending from an earlier call: %s", fn, \
                                cudaGetErrorString(e_));                                         \
    } while (0)

#define AMGT_TRY(expr)                       \
    do {                                     \
        amgt_status s_ = (expr);             \
        if (s_ != AMGT_OK) return s_;        \
    } while (0)

// ------------------------------------------------------------------ allocator
struct Alloc {
    const amgt_allocator* al;
    cudaStream_t s;
    void* get(size_t bytes);
    void put(void* p, size_t bytes);
};

// Library-internal temporaries: CUDA's stream-ordered pool (cudaMallocAsync on the call's
// stream; the pool keeps freed memory cached), never the caller's allocator — outputs the
// caller sees use the amgt_allocator, scratch does not need to cross the ABI.
void* scratch_get(size_t bytes, cudaStream_t s);
void scratch_put(void* p, cudaStream_t s);
// drops the SpGEMM numeric plan keyed by a C structure array being released (spgemm.cu)
void spgemm_plan_drop(const void* key, cudaStream_t s);

template <typename T>
struct Scratch {
    cudaStream_t s = nullptr;
    T* p = nullptr;
    size_t n = 0;
    Scratch() = default;
    Scratch(const Scratch&) = delete;
    Scratch& operator=(const Scratch&) = delete;
    amgt_status init(Alloc& al, size_t count) {
        s = al.s;
        n = count;
        if (count == 0) return AMGT_OK;
        p = static_cast<T*>(scratch_get(count * sizeof(T), s));
        if (!p) return fail(AMGT_ERR_ALLOC, "scratch allocation of %zu bytes failed", count * sizeof(T));
        return AMGT_OK;
    }
    bool try_init(Alloc& al, size_t count) {  // optional scratch: false (no error set) on failure
        s = al.s;
        n = count;
        if (count == 0) return true;
        p = static_cast<T*>(scratch_get(count * sizeof(T), s));
        return p != nullptr;
    }
    ~Scratch() {
        if (p) scratch_put(p, s);
    }
};

// ------------------------------------------------------------------ types
size_t prec_bytes(amgt_prec p);
inline bool prec_valid(int p) { return p == AMGT_FP64 || p == AMGT_FP32 || p == AMGT_FP16; }

template <typename T> struct AccOf { using type = float; };
template <> struct AccOf<double> { using type = double; };

__device__ __forceinline__ double to_f64(double v) { return v; }
__device__ __forceinline__ double to_f64(float v) { return (double)v; }
__device__ __forceinline__ double to_f64(__half v) { return (double)__half2float(v); }
__device__ __forceinline__ float to_f32(double v) { return (float)v; }
__device__ __forceinline__ float to_f32(float v) { return v; }
__device__ __forceinline__ float to_f32(__half v) { return __half2float(v); }

template <typename T> __device__ __forceinline__ T from_f64(double v);
template <> __device__ __forceinline__ double from_f64<double>(double v) { return v; }
template <> __device__ __forceinline__ float from_f64<float>(double v) { return __double2float_rn(v); }
template <> __device__ __forceinline__ __half from_f64<__half>(double v) { return __double2half(v); }  // RN, direct

template <typename T> __device__ __forceinline__ T from_acc(double v) { return from_f64<T>(v); }
template <typename T> __device__ __forceinline__ T from_acc(float v);
template <> __device__ __forceinline__ double from_acc<double>(float v) { return (double)v; }
template <> __device__ __forceinline__ float from_acc<float>(float v) { return v; }
template <> __device__ __forceinline__ __half from_acc<__half>(float v) { return __float2half_rn(v); }

template <typename A> __device__ __forceinline__ A acc_from(double v);
template <> __device__ __forceinline__ double acc_from<double>(double v) { return v; }
template <> __device__ __forceinline__ float acc_from<float>(double v) { return (float)v; }
template <typename A> __device__ __forceinline__ A acc_of(double v) { return (A)v; }
template <typename A> __device__ __forceinline__ A acc_of(float v) { return (A)v; }
template <typename A> __device__ __forceinline__ A acc_of(__half v) { return (A)__half2float(v); }

// ------------------------------------------------------------------ bitmaps
// BITMAPMULTIPLY (Alg. 3 line 7, Alg. 4 lines 8/22; reading R4): boolean 4x4 product.
// (mapA >> k) & 0x1111 marks rows r with A(r,k) != 0 at bit 4r; multiplying by B's
// row-k nibble places that nibble at 4r for each such r (no carries: nibbles disjoint).
__device__ __forceinline__ uint32_t bitmap_multiply(uint32_t a, uint32_t b) {
    return (((a >> 0) & 0x1111u) * ((b >> 0) & 0xFu)) | (((a >> 1) & 0x1111u) * ((b >> 4) & 0xFu)) |
           (((a >> 2) & 0x1111u) * ((b >> 8) & 0xFu)) | (((a >> 3) & 0x1111u) * ((b >> 12) & 0xFu));
}

// A 4-lane group (lanes gbase..gbase+3, mask gm) holds the four rows of an FP64 4x4 tile,
// lane r owning row r.  Store the 128-B tile with two instructions that each write 64
// contiguous bytes (full 32-B sectors: no partial-sector read-for-write in L2): lane q
// writes elements {2q, 2q+1} (row q>>1) and {8+2q, 9+2q} (row 2+(q>>1)).
__device__ __forceinline__ void group_store_tile_f64(double* tile, const double (&v)[4], int q, unsigned gm,
                                                     int gbase) {
    const int s1 = gbase + (q >> 1), s2 = gbase + 2 + (q >> 1);
    const double a0 = __shfl_sync(gm, v[0], s1), a1 = __shfl_sync(gm, v[1], s1);
    const double a2 = __shfl_sync(gm, v[2], s1), a3 = __shfl_sync(gm, v[3], s1);
    const double b0 = __shfl_sync(gm, v[0], s2), b1 = __shfl_sync(gm, v[1], s2);
    const double b2 = __shfl_sync(gm, v[2], s2), b3 = __shfl_sync(gm, v[3], s2);
    reinterpret_cast<double2*>(tile)[q] = (q & 1) ? make_double2(a2, a3) : make_double2(a0, a1);
    reinterpret_cast<double2*>(tile)[4 + q] = (q & 1) ? make_double2(b2, b3) : make_double2(b0, b1);
}

// ------------------------------------------------------------------ device flags
// Bits of the per-call device error word.
enum : uint32_t { FLAG_FORMAT = 1u, FLAG_RANGE = 2u };

// ------------------------------------------------------------------ scan
// out[0] = 0, out[i+1] = in[0] + ... + in[i]  (int64, n >= 0, inputs >= 0); one launch
// (decoupled look-back).  dmax (optional, device, pre-set by the caller): atomicMax of the inputs.
amgt_status scan_exclusive(const int64_t* in, int64_t* out, int64_t n, Alloc& a, cudaStream_t s,
                           unsigned long long* dmax = nullptr);

// ------------------------------------------------------------------ instrumentation
enum TimerClass : int {
    TC_SPMV_L1 = 0,
    TC_SPMV = 1,
    TC_SPGEMM_SYM = 2,
    TC_SPGEMM_NUM = 3,
    TC_CSR2MBSR = 4,
    TC_MBSR2CSR = 5,
    TC_CAST = 6,
    TC_VEC = 7
};
void count_launch();
void trace_point(const char* name, cudaStream_t s);  // AMGT_TRACE=1 only (measurement)
constexpr int PINNED_SLOTS = 16384;  // 128 KB
int64_t* pinned_slots();  // per-thread pinned host int64[PINNED_SLOTS], NULL if unavailable
// slot ranges (a pageable-memory cudaMemcpyAsync D2H stages through the driver and costs
// tens of microseconds; these small read-backs go to pinned memory instead)
constexpr int PIN_CREATE = 0;  // [0, 16): hierarchy creation, R_k row maxima (read at later syncs)
constexpr int PIN_SYM = 16;    // [16, 36): SpGEMM symbolic (16 stats, C tile count, longest row)
constexpr int PIN_CONV = 40;   // [40, 44): CSR -> mBSR (tile count, flags, longest row)
constexpr int PIN_NORMS = 64;  // [64, 1088): V-cycle / PCG residual norms
constexpr int PIN_COARSE = 2048;  // [2048, 16384): coarsest-level CSR on its way to the host factorisation
void trace_dump();
struct TimerScope {  // records start/end events on `s` when timing is enabled
    int cls;
    double bytes;
    cudaStream_t s;
    int slot;
    TimerScope(int cls, double bytes, cudaStream_t s);
    ~TimerScope();
};

// SpMV epilogue selection (AMGT_EPI_* in amgt.h) and its operands.
struct EpiArgs {
    int mode;
    const void* b;
    const void* dinv;
    const void* xs;
    double omega;
    int64_t I0, I1;  // block-row range [I0, I1); I1 < 0 = all rows
    void* r = nullptr;  // AMGT_EPI_JACOBI_RES: residual output (y's precision)
    void* x1 = nullptr;  // EPI_RES_X0: the zero-guess sweep's iterate (y's precision)
    double* nws = nullptr;  // EPI_JACOBI_NORM: one partial per warp
};
// Internal epilogue (not in the ABI): the residual of the first pre-smoothing sweep from a
// zero guess, r = b - A x1 with x1 = 0 + w dinv .* (b - 0) formed on the fly at every
// gathered column (the k_jacobi0 expression, bit-identical), and x1 of the row written too:
// Alg. 2 lines 2-3 on a coarse level in one pass.  FP32 vectors, FP32/FP16 operators.
constexpr int EPI_RES_X0 = 5;
// Internal epilogue: the Jacobi sweep (as AMGT_EPI_JACOBI) plus, per warp of the row kernel,
// the sum of (b_i - (A x)_i)^2 over its rows (xor-tree) into nws[warp] — the residual norm of
// the sweep's input without writing r (a deterministic fixed-order sum of the partials
// follows).  FP64 operator and vectors, no long rows (spmv_warp_norm_ok).
constexpr int EPI_JACOBI_NORM = 6;
bool spmv_warp_norm_ok(const amgt_mbsr* A);
int64_t spmv_warp_norm_count(const amgt_mbsr* A);  // partials written (warps of the row kernel)

// ------------------------------------------------------------------ programmatic dependent launch
// Inside a PdlScope (the V-cycle and PCG solve loops, including the CUDA-graph capture of the
// coarse sub-cycle) the solve kernels are launched with programmatic stream serialization:
// kernel N+1's CTAs may become resident while kernel N's last wave runs, and wait in
// pdl_wait() (griddepcontrol.wait: kernel N complete and its writes visible) before touching
// memory.  Every kernel launched through pdl_launch must call pdl_wait() before its first
// global memory access.  Outside a scope (or with AMGT_PDL=0) launches are ordinary.
bool pdl_active();
struct PdlScope {
    PdlScope();
    ~PdlScope();
};
__device__ __forceinline__ void pdl_wait() {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    asm volatile("griddepcontrol.wait;" ::: "memory");
}
template <typename... KArgs, typename... Args>
inline void pdl_launch(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args... args) {
    if (pdl_active()) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = grid;
        cfg.blockDim = block;
        cfg.dynamicSmemBytes = smem;
        cfg.stream = s;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[0].val.programmaticStreamSerializationAllowed = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        cudaLaunchKernelEx(&cfg, kern, static_cast<KArgs>(args)...);
    } else {
        kern<<<grid, block, smem, s>>>(static_cast<KArgs>(args)...);
    }
}

extern int g_tc_thr_spgemm;
extern int g_tc_thr_spmv;

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }
int num_sms();

// Opt a kernel into `bytes` of dynamic shared memory.  The attribute is process-wide while the
// loopback ranks launch from several host threads with different sizes, so it only ever rises
// (under a lock): a launch never finds it lowered below what its own call raised it to.
cudaError_t dyn_smem_optin(const void* kern, size_t bytes);
template <typename K>
inline cudaError_t dyn_smem(K* kern, size_t bytes) { return dyn_smem_optin((const void*)kern, bytes); }

}  // namespace amgt
