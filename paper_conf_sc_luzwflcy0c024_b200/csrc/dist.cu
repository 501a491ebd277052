// dist.cu — the row-partitioned multi-GPU path (the paper's 8-GPU runs go through
// HYPRE/MPI, L363-365 — this is the B200 re-design over NCCL / NVLink).
//
// Partition: rank r owns a contiguous range of rows of every distributed matrix (ranks in
// ascending order, every range but the last a whole number of 4-row block rows).  A rank holds
// its rows with GLOBAL column indices; the library derives everything else:
//   * halo plan  — the block-row range [eb, ee) its columns touch (contiguous: the row slabs of
//                  the paper's structured workloads), the pieces of it other ranks own (receive)
//                  and the pieces of its own rows other ranks need (send), from ONE host
//                  all-gather of (rows, min column, max column) per rank;
//   * SpMV       — x's halo exchanged (point-to-point, one group) on a communication stream
//                  while the interior block rows (rows that touch no halo column) run, then the
//                  boundary block rows (amgt_dist_spmv);
//   * RAP        — the rows of P (and, in general, of A·P) that a rank's columns reach are
//                  gathered from their owners as mBSR rows (row lengths, then tiles: one host
//                  sync), then A_l·P_ext and R_l·(AP) are local SpGEMMs (amgt_dist_rap);
//   * V-cycle    — Alg. 2 with distributed SpMVs on the fine levels and, from the first level
//                  with at most `agg_rows` global rows down, the levels agglomerated onto every
//                  rank: one all-gather of that level's right-hand side per cycle, then the
//                  single-GPU V-cycle machinery (CUDA graph, shared-memory tail, dense coarse
//                  solve) runs redundantly — instead of a halo exchange per coarse SpMV.
// Transports: NCCL (one process per GPU; libnccl.so.2 loaded at run time — the library torch
// already mapped — so libamgt has no link-time dependency), and a loopback transport that runs
// G virtual ranks as G host threads on ONE GPU: every transfer is a device-to-device copy
// ordered by CUDA events, collectives are deterministic rank-order sums.  The loopback lets the
// multi-rank code run (and be parity-tested) on a single B200.
#include <dlfcn.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cmath>
#include <condition_variable>
#include <cstring>
#include <deque>
#include <map>
#include <memory>
#include <mutex>
#include <vector>

#include "common.cuh"

namespace amgt {
amgt_status spmv_ex_impl(const amgt_mbsr* A, const void* x, amgt_prec xp, void* y, amgt_prec yp, const EpiArgs& ea,
                         cudaStream_t s, int timer_class);
amgt_status spmv_analyze_impl(amgt_mbsr* A, Alloc& a);
amgt_status mbsr_release(amgt_mbsr* M, Alloc& a);
amgt_status mbsr_alloc(amgt_mbsr* M, int64_t m, int64_t n, int64_t T, amgt_prec prec, Alloc& a, bool structure,
                       bool values, int64_t* existing_ptr);
amgt_status cast_impl(const amgt_mbsr* in, amgt_prec to, amgt_mbsr* out, Alloc& a, uint32_t* dflag);
amgt_status transpose_impl(const amgt_mbsr* in, amgt_mbsr* out, Alloc& a, unsigned long long* dmax);
amgt_status spgemm_symbolic_impl(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* C, amgt_spgemm_info* info,
                                 Alloc& a);
amgt_status spgemm_numeric_impl(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* C, Alloc& a);
amgt_status dinv_impl(const amgt_mbsr& A, int64_t off, void* dinv, amgt_prec vprec, cudaStream_t s, bool l1);
amgt_status hierarchy_create_tail(const amgt_mbsr* A, const amgt_mbsr* const* P, int nlev, const amgt_vcycle_opts* o,
                                  const amgt_allocator* al, cudaStream_t s, amgt_hierarchy** Hout);
void hierarchy_free(amgt_hierarchy* H);
amgt_prec hierarchy_vprec0(const amgt_hierarchy* H);
int64_t hierarchy_npad0(const amgt_hierarchy* H);
amgt_status hierarchy_apply(amgt_hierarchy* H, const void* b, void* x, cudaStream_t s, int64_t* calls);
}  // namespace amgt
using namespace amgt;

// ================================================================== NCCL (dlopen)
typedef struct {
    char internal[128];
} nccl_uid;
typedef void* nccl_comm;
typedef int nccl_result;
enum { NCCL_INT8 = 0, NCCL_FLOAT64 = 8 };
enum { NCCL_SUM = 0 };

struct NcclApi {
    void* h = nullptr;
    nccl_result (*GetUniqueId)(nccl_uid*) = nullptr;
    nccl_result (*CommInitRank)(nccl_comm*, int, nccl_uid, int) = nullptr;
    nccl_result (*CommDestroy)(nccl_comm) = nullptr;
    nccl_result (*Send)(const void*, size_t, int, int, nccl_comm, cudaStream_t) = nullptr;
    nccl_result (*Recv)(void*, size_t, int, int, nccl_comm, cudaStream_t) = nullptr;
    nccl_result (*GroupStart)() = nullptr;
    nccl_result (*GroupEnd)() = nullptr;
    nccl_result (*AllReduce)(const void*, void*, size_t, int, int, nccl_comm, cudaStream_t) = nullptr;
    nccl_result (*AllGather)(const void*, void*, size_t, int, nccl_comm, cudaStream_t) = nullptr;
    const char* (*GetErrorString)(nccl_result) = nullptr;
};
static NcclApi g_nccl;
static std::mutex g_nccl_mu;

static amgt_status load_nccl() {
    std::lock_guard<std::mutex> lk(g_nccl_mu);
    if (g_nccl.h) return AMGT_OK;
    const char* names[] = {"libnccl.so.2", "libnccl.so"};
    void* h = nullptr;
    for (const char* n : names)
        if ((h = dlopen(n, RTLD_NOW | RTLD_GLOBAL))) break;
    if (!h) return fail(AMGT_ERR_NCCL, "cannot dlopen libnccl.so.2: %s", dlerror());
    auto sym = [&](const char* s) { return dlsym(h, s); };
    g_nccl.GetUniqueId = (decltype(g_nccl.GetUniqueId))sym("ncclGetUniqueId");
    g_nccl.CommInitRank = (decltype(g_nccl.CommInitRank))sym("ncclCommInitRank");
    g_nccl.CommDestroy = (decltype(g_nccl.CommDestroy))sym("ncclCommDestroy");
    g_nccl.Send = (decltype(g_nccl.Send))sym("ncclSend");
    g_nccl.Recv = (decltype(g_nccl.Recv))sym("ncclRecv");
    g_nccl.GroupStart = (decltype(g_nccl.GroupStart))sym("ncclGroupStart");
    g_nccl.GroupEnd = (decltype(g_nccl.GroupEnd))sym("ncclGroupEnd");
    g_nccl.AllReduce = (decltype(g_nccl.AllReduce))sym("ncclAllReduce");
    g_nccl.AllGather = (decltype(g_nccl.AllGather))sym("ncclAllGather");
    g_nccl.GetErrorString = (decltype(g_nccl.GetErrorString))sym("ncclGetErrorString");
    if (!g_nccl.GetUniqueId || !g_nccl.CommInitRank || !g_nccl.Send || !g_nccl.Recv || !g_nccl.GroupStart ||
        !g_nccl.GroupEnd || !g_nccl.AllReduce || !g_nccl.AllGather || !g_nccl.CommDestroy)
        return fail(AMGT_ERR_NCCL, "libnccl.so.2 lacks a required symbol");
    g_nccl.h = h;
    return AMGT_OK;
}

#define AMGT_NCCL(call)                                                                                   \
    do {                                                                                                  \
        nccl_result r_ = (call);                                                                          \
        if (r_ != 0)                                                                                      \
            return fail(AMGT_ERR_NCCL, "%s:%d %s: %s", __FILE__, __LINE__, #call,                         \
                        g_nccl.GetErrorString ? g_nccl.GetErrorString(r_) : "nccl error");                \
    } while (0)

namespace {

// ================================================================== transports
struct Msg {
    int peer;
    void* buf;
    size_t bytes;
};

struct Transport {
    int rank = 0, size = 1;
    virtual ~Transport() = default;
    // grouped point-to-point: every send and receive of the call, stream-ordered on s; a send
    // buffer may be reused (in stream order) after the call
    virtual amgt_status exchange(const std::vector<Msg>& sends, const std::vector<Msg>& recvs, cudaStream_t s) = 0;
    // in-place sum over ranks (FP64); every rank gets the same bits
    virtual amgt_status allreduce_f64(double* buf, int64_t n, cudaStream_t s) = 0;
    // host buffers: out[q*bytes ...] = rank q's in (blocking)
    virtual amgt_status allgather_host(const void* in, void* out, size_t bytes) = 0;
};

struct NcclTransport final : Transport {
    nccl_comm comm = nullptr;
    cudaStream_t hs = nullptr;  // host-metadata collectives
    char* dbuf = nullptr;
    size_t dcap = 0;
    ~NcclTransport() override {
        if (hs) cudaStreamSynchronize(hs);
        if (dbuf) cudaFree(dbuf);
        if (comm && g_nccl.CommDestroy) g_nccl.CommDestroy(comm);
        if (hs) cudaStreamDestroy(hs);
    }
    amgt_status exchange(const std::vector<Msg>& sends, const std::vector<Msg>& recvs, cudaStream_t s) override {
        if (sends.empty() && recvs.empty()) return AMGT_OK;
        AMGT_NCCL(g_nccl.GroupStart());
        for (const Msg& m : sends)
            if (m.bytes) AMGT_NCCL(g_nccl.Send(m.buf, m.bytes, NCCL_INT8, m.peer, comm, s));
        for (const Msg& m : recvs)
            if (m.bytes) AMGT_NCCL(g_nccl.Recv(m.buf, m.bytes, NCCL_INT8, m.peer, comm, s));
        AMGT_NCCL(g_nccl.GroupEnd());
        return AMGT_OK;
    }
    amgt_status allreduce_f64(double* buf, int64_t n, cudaStream_t s) override {
        if (size > 1 && n > 0) AMGT_NCCL(g_nccl.AllReduce(buf, buf, (size_t)n, NCCL_FLOAT64, NCCL_SUM, comm, s));
        return AMGT_OK;
    }
    amgt_status allgather_host(const void* in, void* out, size_t bytes) override {
        if (size == 1) {
            memcpy(out, in, bytes);
            return AMGT_OK;
        }
        const size_t need = bytes * (size + 1);
        if (need > dcap) {
            if (dbuf) cudaFree(dbuf);
            dbuf = nullptr;
            AMGT_CUDA(cudaMalloc(&dbuf, need));
            dcap = need;
        }
        AMGT_CUDA(cudaMemcpyAsync(dbuf, in, bytes, cudaMemcpyHostToDevice, hs));
        AMGT_NCCL(g_nccl.AllGather(dbuf, dbuf + bytes, bytes, NCCL_INT8, comm, hs));
        AMGT_CUDA(cudaMemcpyAsync(out, dbuf + bytes, bytes * size, cudaMemcpyDeviceToHost, hs));
        AMGT_CUDA(cudaStreamSynchronize(hs));
        return AMGT_OK;
    }
};

constexpr int LOOP_MAX = 16;  // virtual ranks per loopback group
struct PtrList {
    const double* p[LOOP_MAX];
};
// deterministic rank-order sum of the ranks' buffers (loopback all-reduce)
__global__ void k_sum_ranks(int64_t n, PtrList in, int size, double* __restrict__ out) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        double a = in.p[0][i];
        for (int q = 1; q < size; ++q) a += in.p[q][i];
        out[i] = a;
    }
}

}  // namespace

// Shared state of one loopback group: per (source, destination) FIFO mailboxes for point-to-point
// messages and per-sequence-number slots for collectives (every virtual rank issues the same
// sequence of communication calls, as NCCL requires).
struct amgt_dist_group {
    int size = 1;
    std::atomic<bool> aborted{false};  // a member failed outside the library: wake the others
    std::mutex mu;
    std::condition_variable cv;
    struct Post {
        const void* src = nullptr;
        size_t bytes = 0;
        cudaEvent_t ready = nullptr, done = nullptr;
        bool consumed = false;
        bool bad = false;
    };
    std::map<std::pair<int, int>, std::deque<std::shared_ptr<Post>>> box;
    struct Coll {
        int arrived = 0, done = 0, left = 0;
        std::vector<const void*> ptr;
        std::vector<cudaEvent_t> ev, ev2;
        std::vector<char> host;
    };
    std::map<uint64_t, std::shared_ptr<Coll>> coll;
};

namespace {

constexpr double LOOP_TIMEOUT_S = 300.0;

struct LoopTransport final : Transport {
    amgt_dist_group* g = nullptr;
    uint64_t seq = 0;
    template <typename Pred>
    amgt_status wait(std::unique_lock<std::mutex>& lk, Pred pred, const char* what) {
        const bool ok = g->cv.wait_for(lk, std::chrono::duration<double>(LOOP_TIMEOUT_S),
                                       [&] { return g->aborted.load() || pred(); });
        if (g->aborted.load() && !pred())
            return fail(AMGT_ERR_NCCL, "loopback rank %d: group aborted while waiting for %s", rank, what);
        if (!ok)
            return fail(AMGT_ERR_NCCL, "loopback rank %d: timed out waiting for %s (mismatched communication calls?)",
                        rank, what);
        return AMGT_OK;
    }
    amgt_status exchange(const std::vector<Msg>& sends, const std::vector<Msg>& recvs, cudaStream_t s) override {
        using Post = amgt_dist_group::Post;
        std::vector<std::shared_ptr<Post>> mine;
        for (const Msg& m : sends) {
            if (!m.bytes) continue;
            auto p = std::make_shared<Post>();
            p->src = m.buf;
            p->bytes = m.bytes;
            AMGT_CUDA(cudaEventCreateWithFlags(&p->ready, cudaEventDisableTiming));
            AMGT_CUDA(cudaEventRecord(p->ready, s));
            {
                std::lock_guard<std::mutex> lk(g->mu);
                g->box[{rank, m.peer}].push_back(p);
            }
            mine.push_back(p);
        }
        g->cv.notify_all();
        amgt_status st = AMGT_OK;
        for (const Msg& m : recvs) {
            if (!m.bytes) continue;
            std::shared_ptr<Post> p;
            {
                std::unique_lock<std::mutex> lk(g->mu);
                auto& q = g->box[{m.peer, rank}];
                AMGT_TRY(wait(lk, [&] { return !q.empty(); }, "a message"));
                p = q.front();
                q.pop_front();
            }
            cudaEvent_t done = nullptr;
            if (p->bytes != m.bytes) {
                st = fail(AMGT_ERR_NCCL, "loopback: rank %d expected %zu bytes from %d, got %zu", rank, m.bytes, m.peer,
                          p->bytes);
            } else {
                AMGT_CUDA(cudaStreamWaitEvent(s, p->ready, 0));
                AMGT_CUDA(cudaMemcpyAsync(m.buf, p->src, m.bytes, cudaMemcpyDeviceToDevice, s));
                AMGT_CUDA(cudaEventCreateWithFlags(&done, cudaEventDisableTiming));
                AMGT_CUDA(cudaEventRecord(done, s));
            }
            {
                std::lock_guard<std::mutex> lk(g->mu);
                p->done = done;
                p->consumed = true;
                p->bad = done == nullptr;
            }
            g->cv.notify_all();
        }
        for (auto& p : mine) {
            {
                std::unique_lock<std::mutex> lk(g->mu);
                AMGT_TRY(wait(lk, [&] { return p->consumed; }, "a receiver"));
            }
            if (p->done) {
                AMGT_CUDA(cudaStreamWaitEvent(s, p->done, 0));  // the buffer is free once the copy ran
                cudaEventDestroy(p->done);
            }
            cudaEventDestroy(p->ready);
            if (p->bad && st == AMGT_OK) st = fail(AMGT_ERR_NCCL, "loopback: message size mismatch at the receiver");
        }
        return st;
    }
    std::shared_ptr<amgt_dist_group::Coll> slot(uint64_t key) {
        std::lock_guard<std::mutex> lk(g->mu);
        auto& e = g->coll[key];
        if (!e) {
            e = std::make_shared<amgt_dist_group::Coll>();
            e->ptr.assign(size, nullptr);
            e->ev.assign(size, nullptr);
            e->ev2.assign(size, nullptr);
        }
        return e;
    }
    void leave(uint64_t key, const std::shared_ptr<amgt_dist_group::Coll>& c) {
        std::lock_guard<std::mutex> lk(g->mu);
        if (++c->left == size) {
            for (auto e : c->ev) if (e) cudaEventDestroy(e);
            for (auto e : c->ev2) if (e) cudaEventDestroy(e);
            g->coll.erase(key);
        }
    }
    amgt_status allreduce_f64(double* buf, int64_t n, cudaStream_t s) override {
        if (size == 1 || n <= 0) return AMGT_OK;
        const uint64_t key = seq++;
        auto c = slot(key);
        cudaEvent_t e1, e2;
        AMGT_CUDA(cudaEventCreateWithFlags(&e1, cudaEventDisableTiming));
        AMGT_CUDA(cudaEventCreateWithFlags(&e2, cudaEventDisableTiming));
        AMGT_CUDA(cudaEventRecord(e1, s));
        {
            std::unique_lock<std::mutex> lk(g->mu);
            c->ptr[rank] = buf;
            c->ev[rank] = e1;
            c->ev2[rank] = e2;
            ++c->arrived;
            g->cv.notify_all();
            AMGT_TRY(wait(lk, [&] { return c->arrived == size; }, "an all-reduce"));
        }
        PtrList pl{};
        for (int q = 0; q < size; ++q) {
            pl.p[q] = (const double*)c->ptr[q];
            if (q != rank) AMGT_CUDA(cudaStreamWaitEvent(s, c->ev[q], 0));
        }
        Alloc a{nullptr, s};
        Scratch<double> tmp;
        AMGT_TRY(tmp.init(a, n));
        k_sum_ranks<<<(unsigned)std::min<int64_t>(ceil_div(n, 256), 1024), 256, 0, s>>>(n, pl, size, tmp.p);
        AMGT_LAUNCHED();
        AMGT_CUDA(cudaEventRecord(e2, s));
        {
            std::unique_lock<std::mutex> lk(g->mu);
            ++c->done;
            g->cv.notify_all();
            AMGT_TRY(wait(lk, [&] { return c->done == size; }, "an all-reduce"));
        }
        for (int q = 0; q < size; ++q)
            if (q != rank) AMGT_CUDA(cudaStreamWaitEvent(s, c->ev2[q], 0));  // every rank has read my buffer
        AMGT_CUDA(cudaMemcpyAsync(buf, tmp.p, n * sizeof(double), cudaMemcpyDeviceToDevice, s));
        leave(key, c);
        return AMGT_OK;
    }
    amgt_status allgather_host(const void* in, void* out, size_t bytes) override {
        if (size == 1) {
            memcpy(out, in, bytes);
            return AMGT_OK;
        }
        const uint64_t key = seq++;
        auto c = slot(key);
        {
            std::unique_lock<std::mutex> lk(g->mu);
            if (c->host.empty()) c->host.assign(bytes * size, 0);
            memcpy(c->host.data() + bytes * rank, in, bytes);
            ++c->arrived;
            g->cv.notify_all();
            AMGT_TRY(wait(lk, [&] { return c->arrived == size; }, "a metadata all-gather"));
            memcpy(out, c->host.data(), bytes * size);
        }
        leave(key, c);
        return AMGT_OK;
    }
};

}  // namespace

// ================================================================== plans
namespace {

struct Piece {
    int peer;
    int64_t g0, g1;  // global block rows [g0, g1)
};

// A rank's view of a row-partitioned operand M (rows of every rank, block-row offsets `off`) that
// its matrix's columns index: the extended block-row range [eb, ee) of those columns (containing
// the own rows [rb, re)), what it receives (the pieces of [eb, ee) other ranks own) and what it
// sends (the pieces of its own rows in other ranks' extended ranges).
struct Plan {
    int rank = 0, size = 1;
    std::vector<int64_t> off;  // size + 1 block-row offsets
    int64_t rb = 0, re = 0, eb = 0, ee = 0;
    std::vector<Piece> recv, send;
};

// Host-only: the plan from the all-gathered metadata (cmin > cmax: the rank's matrix has no tiles).
void plan_from_meta(int rank, int size, const std::vector<int64_t>& off, const int64_t* cmin, const int64_t* cmax,
                    Plan& P) {
    P.rank = rank;
    P.size = size;
    P.off = off;
    auto ext = [&](int q, int64_t& b, int64_t& e) {
        b = off[q];
        e = off[q + 1];
        if (cmin[q] <= cmax[q]) {
            b = std::min(b, cmin[q]);
            e = std::max(e, cmax[q] + 1);
        }
    };
    P.rb = off[rank];
    P.re = off[rank + 1];
    ext(rank, P.eb, P.ee);
    P.recv.clear();
    P.send.clear();
    for (int q = 0; q < size; ++q) {
        if (q == rank) continue;
        const int64_t qb = off[q], qe = off[q + 1];
        const int64_t mine[2][2] = {{P.eb, P.rb}, {P.re, P.ee}};  // my halo pieces owned by q
        for (auto& h : mine) {
            const int64_t lo = std::max(h[0], qb), hi = std::min(h[1], qe);
            if (lo < hi) P.recv.push_back({q, lo, hi});
        }
        int64_t qeb, qee;
        ext(q, qeb, qee);
        const int64_t theirs[2][2] = {{qeb, qb}, {qe, qee}};  // q's halo pieces that I own
        for (auto& h : theirs) {
            const int64_t lo = std::max(h[0], P.rb), hi = std::min(h[1], P.re);
            if (lo < hi) P.send.push_back({q, lo, hi});
        }
    }
}

// ---- kernels
__global__ void k_minmax_cols(int64_t BR, const int64_t* __restrict__ ptr, const int32_t* __restrict__ idx,
                              unsigned long long* __restrict__ out) {  // out = {min, max} (pre-set)
    unsigned long long mn = ~0ull, mx = 0;
    bool any = false;
    for (int64_t I = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; I < BR; I += (int64_t)gridDim.x * blockDim.x) {
        const int64_t a = ptr[I], b = ptr[I + 1];
        if (b > a) {
            any = true;
            mn = min(mn, (unsigned long long)idx[a]);
            mx = max(mx, (unsigned long long)idx[b - 1]);
        }
    }
    if (any) {
        atomicMin(out, mn);
        atomicMax(out + 1, mx + 1);  // stored +1 so that 0 = no tile
    }
}

// interior block rows of a square row-partitioned A: out[0] = 1 + last row with a column < lo,
// out[1] = first row with a column >= hi (pre-set to 0 and BR)
__global__ void k_interior(int64_t BR, const int64_t* __restrict__ ptr, const int32_t* __restrict__ idx, int64_t lo,
                           int64_t hi, unsigned long long* __restrict__ out) {
    for (int64_t I = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; I < BR; I += (int64_t)gridDim.x * blockDim.x) {
        const int64_t a = ptr[I], b = ptr[I + 1];
        if (b <= a) continue;
        if (idx[a] < lo) atomicMax(out, (unsigned long long)(I + 1));
        if (idx[b - 1] >= hi) atomicMin(out + 1, (unsigned long long)I);
    }
}

__global__ void k_row_len(int64_t BR, const int64_t* __restrict__ ptr, int64_t* __restrict__ len) {
    for (int64_t I = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; I < BR; I += (int64_t)gridDim.x * blockDim.x)
        len[I] = ptr[I + 1] - ptr[I];
}

__global__ void k_shift_copy(int64_t T, const int32_t* __restrict__ in, int32_t* __restrict__ out, int64_t delta) {
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < T; t += (int64_t)gridDim.x * blockDim.x)
        out[t] = (int32_t)(in[t] + delta);
}

constexpr int NB = 256;
__global__ void k_sq_partial(int64_t n, const double* __restrict__ r, double* __restrict__ part) {
    __shared__ double sh[32];
    double s = 0.0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        s = fma(r[i], r[i], s);
    for (int d = 16; d; d >>= 1) s += __shfl_xor_sync(0xffffffffu, s, d);
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        double a = 0.0;
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) a += sh[w];
        part[blockIdx.x] = a;
    }
}
__global__ void k_sq_final(const double* __restrict__ part, double* __restrict__ out) {
    if (threadIdx.x == 0) {
        double a = 0.0;
        for (int i = 0; i < NB; ++i) a += part[i];
        *out = a;
    }
}
// first pre-smoothing sweep of a coarse level from x = 0: x = 0 + w dinv .* (b - 0) (the SpMV of
// the zero vector and its halo exchange are skipped; the expression of the single-GPU k_jacobi0)
template <typename V>
__global__ void k_zero_sweep(int64_t n, const V* __restrict__ b, const V* __restrict__ dinv, V omega,
                             V* __restrict__ x) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const V zero = V(0), t = V(0);
    x[i] = zero + omega * dinv[i] * (b[i] - t);
}

unsigned grid1(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), 4096)); }
size_t vbytes(amgt_prec p) { return p == AMGT_FP64 ? 8 : 4; }
amgt_prec vec_prec(amgt_prec matrix) { return matrix == AMGT_FP64 ? AMGT_FP64 : AMGT_FP32; }  // R16

// pinned read-back slots of this module (per thread, see common.cuh)
constexpr int PIN_DIST = 1088;
constexpr int PIN_DIST_N = PIN_COARSE - PIN_DIST;

}  // namespace

// ================================================================== communicator
struct amgt_dist {
    std::unique_ptr<Transport> t;
    int rank = 0, size = 1;
    int64_t row_begin = 0, row_end = 0;
    cudaStream_t cs = nullptr;  // halo exchanges (overlap the interior rows)
    cudaEvent_t ready = nullptr, done = nullptr;
    struct SpmvPlanD;
    std::map<const void*, std::unique_ptr<SpmvPlanD>> plans;  // amgt_dist_spmv, keyed by the matrix arrays
    ~amgt_dist();
};

namespace {

// block-row partition of a distributed operand from every rank's own row count (one metadata
// all-gather together with the column range of the rank's matrix)
amgt_status gather_meta(amgt_dist* D, int64_t m_own, int64_t cmin, int64_t cmax, std::vector<int64_t>& off,
                        std::vector<int64_t>& mins, std::vector<int64_t>& maxs, std::vector<int64_t>* rows = nullptr) {
    const int G = D->size;
    int64_t mine[3] = {m_own, cmin, cmax};
    std::vector<int64_t> all(3 * G);
    AMGT_TRY(D->t->allgather_host(mine, all.data(), sizeof(mine)));
    off.assign(G + 1, 0);
    mins.resize(G);
    maxs.resize(G);
    if (rows) rows->assign(G + 1, 0);
    for (int q = 0; q < G; ++q) {
        const int64_t m = all[3 * q];
        if (q + 1 < G && m % 4)
            return fail(AMGT_ERR_UNSUPPORTED, "row partition: rank %d owns %lld rows (not a multiple of 4)", q,
                        (long long)m);
        off[q + 1] = off[q] + ceil_div(m, 4);
        if (rows) (*rows)[q + 1] = (*rows)[q] + m;
        mins[q] = all[3 * q + 1];
        maxs[q] = all[3 * q + 2];
    }
    return AMGT_OK;
}

// min/max tile column of a matrix (syncs); {1, 0} when it has no tile
amgt_status col_minmax(const amgt_mbsr* A, cudaStream_t s, int64_t& mn, int64_t& mx) {
    int64_t* pin = pinned_slots();
    Alloc a{nullptr, s};
    Scratch<unsigned long long> d;
    AMGT_TRY(d.init(a, 2));
    const unsigned long long init[2] = {~0ull, 0ull};
    AMGT_CUDA(cudaMemcpyAsync(d.p, init, sizeof(init), cudaMemcpyHostToDevice, s));
    if (A->blc_row > 0) {
        k_minmax_cols<<<grid1(A->blc_row), 256, 0, s>>>(A->blc_row, A->blc_ptr, A->blc_idx, d.p);
        AMGT_LAUNCHED();
    }
    unsigned long long h[2];
    if (pin) {
        AMGT_CUDA(cudaMemcpyAsync(pin + PIN_DIST, d.p, sizeof(h), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaStreamSynchronize(s));
        memcpy(h, pin + PIN_DIST, sizeof(h));
    } else {
        AMGT_CUDA(cudaMemcpyAsync(h, d.p, sizeof(h), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaStreamSynchronize(s));
    }
    if (h[1] == 0) {
        mn = 1;
        mx = 0;
    } else {
        mn = (int64_t)h[0];
        mx = (int64_t)h[1] - 1;
    }
    return AMGT_OK;
}

// the plan of matrix A (own rows, global columns) over an operand partitioned like m_part rows per
// rank (the operand's own rows on this rank: m_part)
amgt_status make_plan(amgt_dist* D, int64_t m_part, const amgt_mbsr* A, cudaStream_t s, Plan& P,
                      std::vector<int64_t>* rows = nullptr) {
    int64_t mn, mx;
    AMGT_TRY(col_minmax(A, s, mn, mx));
    std::vector<int64_t> off, mins, maxs;
    AMGT_TRY(gather_meta(D, m_part, mn, mx, off, mins, maxs, rows));
    if (mn <= mx && (mn < 0 || mx >= off[D->size]))
        return fail(AMGT_ERR_ARG, "distributed matrix: tile columns [%lld, %lld] outside the partition (%lld block rows)",
                    (long long)mn, (long long)mx, (long long)off[D->size]);
    plan_from_meta(D->rank, D->size, off, mins.data(), maxs.data(), P);
    return AMGT_OK;
}

// interior block-row range [i0, i1) of a square A under plan P (rows touching no halo); syncs
amgt_status interior_rows(const amgt_mbsr* A, const Plan& P, cudaStream_t s, int64_t& i0, int64_t& i1) {
    const int64_t BR = A->blc_row;
    Alloc a{nullptr, s};
    Scratch<unsigned long long> d;
    AMGT_TRY(d.init(a, 2));
    const unsigned long long init[2] = {0ull, (unsigned long long)BR};
    AMGT_CUDA(cudaMemcpyAsync(d.p, init, sizeof(init), cudaMemcpyHostToDevice, s));
    if (BR > 0) {
        k_interior<<<grid1(BR), 256, 0, s>>>(BR, A->blc_ptr, A->blc_idx, P.rb, P.re, d.p);
        AMGT_LAUNCHED();
    }
    unsigned long long h[2];
    AMGT_CUDA(cudaMemcpyAsync(h, d.p, sizeof(h), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaStreamSynchronize(s));
    i0 = (int64_t)h[0];
    i1 = (int64_t)h[1];
    if (i1 < i0) i0 = i1 = 0;
    return AMGT_OK;
}

// A view of `in` with its tile columns shifted by delta (out->n = n_new): a new column array, the
// row pointers, bitmaps and values borrowed from `in` (which must outlive the view).  Release
// with release_view.
amgt_status shifted_view(const amgt_mbsr* in, int64_t delta, int64_t n_new, amgt_mbsr* out, Alloc& a) {
    cudaStream_t s = a.s;
    amgt_mbsr M = *in;
    M.own = 0;
    M.aux = nullptr;
    const int64_t T = in->blc_num;
    M.blc_idx = (int32_t*)a.get(T * sizeof(int32_t));
    if (!M.blc_idx) return fail(AMGT_ERR_ALLOC, "distributed: column copy allocation failed");
    if (T > 0) {
        k_shift_copy<<<grid1(T), 256, 0, s>>>(T, in->blc_idx, M.blc_idx, delta);
        AMGT_LAUNCHED();
    }
    M.n = n_new;
    M.blc_col = ceil_div(n_new, 4);
    *out = M;
    return AMGT_OK;
}

void release_view(amgt_mbsr* V, Alloc& a) {
    if (!V->blc_idx && !V->aux) return;
    a.put(V->blc_idx, V->blc_num * sizeof(int32_t));
    V->blc_idx = nullptr;
    V->own = 0;
    mbsr_release(V, a);  // the SpMV plan (aux), nothing borrowed
}

// An owned copy of `in` in precision `prec` with shifted tile columns.
amgt_status copy_shifted(const amgt_mbsr* in, int64_t delta, int64_t n_new, amgt_prec prec, amgt_mbsr* out, Alloc& a) {
    cudaStream_t s = a.s;
    amgt_mbsr M{};
    AMGT_TRY(cast_impl(in, prec, &M, a, nullptr));  // values (own = 2), structure still in's
    const int64_t BR = in->blc_row, T = in->blc_num;
    int64_t* ptr = (int64_t*)a.get((BR + 1) * sizeof(int64_t));
    int32_t* idx = (int32_t*)a.get(T * sizeof(int32_t));
    uint16_t* map = (uint16_t*)a.get(((T + 1) & ~int64_t(1)) * sizeof(uint16_t));
    M.blc_ptr = ptr;
    M.blc_idx = idx;
    M.blc_map = map;
    M.own |= 1u;
    if (!ptr || !idx || !map) {
        mbsr_release(&M, a);
        return fail(AMGT_ERR_ALLOC, "distributed: structure copy allocation failed");
    }
    AMGT_CUDA(cudaMemcpyAsync(ptr, in->blc_ptr, (BR + 1) * sizeof(int64_t), cudaMemcpyDeviceToDevice, s));
    if (T > 0) {
        AMGT_CUDA(cudaMemcpyAsync(map, in->blc_map, T * sizeof(uint16_t), cudaMemcpyDeviceToDevice, s));
        k_shift_copy<<<grid1(T), 256, 0, s>>>(T, in->blc_idx, idx, delta);
        AMGT_LAUNCHED();
    }
    M.n = n_new;
    M.blc_col = ceil_div(n_new, 4);
    *out = M;
    return AMGT_OK;
}

// Rows [P.eb, P.ee) of the row-partitioned matrix whose own rows [P.rb, P.re) are M: own rows
// copied, the others received from their owners (row lengths first, then the tiles of the rows:
// one host sync for the sizes).  Columns and precision as M's; Mx->m = m_rows.
amgt_status gather_rows(amgt_dist* D, const Plan& P, const amgt_mbsr* M, int64_t m_rows, amgt_mbsr* Mx, Alloc& a) {
    cudaStream_t s = a.s;
    const int64_t BRo = P.re - P.rb, BRx = P.ee - P.eb;
    if (M->blc_row != BRo) return fail(AMGT_ERR_ARG, "row gather: %lld own block rows, plan has %lld",
                                       (long long)M->blc_row, (long long)BRo);
    Scratch<int64_t> own_len, xlen;
    AMGT_TRY(own_len.init(a, BRo + 1));
    AMGT_TRY(xlen.init(a, BRx + 1));
    if (BRo > 0) {
        k_row_len<<<grid1(BRo), 256, 0, s>>>(BRo, M->blc_ptr, own_len.p);
        AMGT_LAUNCHED();
        AMGT_CUDA(cudaMemcpyAsync(xlen.p + (P.rb - P.eb), own_len.p, BRo * sizeof(int64_t), cudaMemcpyDeviceToDevice, s));
    }
    std::vector<Msg> sends, recvs;
    for (const Piece& p : P.send) sends.push_back({p.peer, own_len.p + (p.g0 - P.rb), (size_t)(p.g1 - p.g0) * 8});
    for (const Piece& p : P.recv) recvs.push_back({p.peer, xlen.p + (p.g0 - P.eb), (size_t)(p.g1 - p.g0) * 8});
    AMGT_TRY(D->t->exchange(sends, recvs, s));
    amgt_mbsr X{};
    int64_t* xptr = (int64_t*)a.get((BRx + 1) * sizeof(int64_t));
    if (!xptr) return fail(AMGT_ERR_ALLOC, "row gather: pointer allocation failed");
    amgt_status st = scan_exclusive(xlen.p, xptr, BRx, a, s);
    if (st != AMGT_OK) { a.put(xptr, (BRx + 1) * sizeof(int64_t)); return st; }
    // sizes: total, the tile range of every received piece in X and of every sent piece in M
    const int nr = (int)P.recv.size(), ns = (int)P.send.size();
    const int need = 2 + 2 * nr + 2 * ns;
    std::vector<int64_t> h(need);
    int64_t* pin = pinned_slots();
    int64_t* dst = (pin && need <= PIN_DIST_N) ? pin + PIN_DIST : h.data();
    auto rd = [&](int slot, const int64_t* src) {
        return cudaMemcpyAsync(dst + slot, src, sizeof(int64_t), cudaMemcpyDeviceToHost, s);
    };
    AMGT_CUDA(rd(0, xptr + BRx));
    AMGT_CUDA(rd(1, xptr + (P.rb - P.eb)));
    for (int i = 0; i < nr; ++i) {
        AMGT_CUDA(rd(2 + 2 * i, xptr + (P.recv[i].g0 - P.eb)));
        AMGT_CUDA(rd(3 + 2 * i, xptr + (P.recv[i].g1 - P.eb)));
    }
    for (int i = 0; i < ns; ++i) {
        AMGT_CUDA(rd(2 + 2 * nr + 2 * i, M->blc_ptr + (P.send[i].g0 - P.rb)));
        AMGT_CUDA(rd(3 + 2 * nr + 2 * i, M->blc_ptr + (P.send[i].g1 - P.rb)));
    }
    AMGT_CUDA(cudaStreamSynchronize(s));
    if (dst != h.data()) memcpy(h.data(), dst, need * sizeof(int64_t));
    const int64_t T = h[0], own0 = h[1];
    st = mbsr_alloc(&X, m_rows, M->n, T, M->prec, a, true, true, xptr);
    if (st != AMGT_OK) { mbsr_release(&X, a); return st; }
    X.row_max = 0;
    const size_t vs = 16 * prec_bytes(M->prec);
    sends.clear();
    recvs.clear();
    for (int i = 0; i < ns; ++i) {
        const int64_t t0 = h[2 + 2 * nr + 2 * i], t1 = h[3 + 2 * nr + 2 * i];
        const int q = P.send[i].peer;
        sends.push_back({q, M->blc_idx + t0, (size_t)(t1 - t0) * 4});
        sends.push_back({q, M->blc_map + t0, (size_t)(t1 - t0) * 2});
        sends.push_back({q, (char*)M->blc_val + t0 * vs, (size_t)(t1 - t0) * vs});
    }
    for (int i = 0; i < nr; ++i) {
        const int64_t t0 = h[2 + 2 * i], t1 = h[3 + 2 * i];
        const int q = P.recv[i].peer;
        recvs.push_back({q, X.blc_idx + t0, (size_t)(t1 - t0) * 4});
        recvs.push_back({q, X.blc_map + t0, (size_t)(t1 - t0) * 2});
        recvs.push_back({q, (char*)X.blc_val + t0 * vs, (size_t)(t1 - t0) * vs});
    }
    if (M->blc_num > 0) {
        AMGT_CUDA(cudaMemcpyAsync(X.blc_idx + own0, M->blc_idx, M->blc_num * 4, cudaMemcpyDeviceToDevice, s));
        AMGT_CUDA(cudaMemcpyAsync(X.blc_map + own0, M->blc_map, M->blc_num * 2, cudaMemcpyDeviceToDevice, s));
        AMGT_CUDA(cudaMemcpyAsync((char*)X.blc_val + own0 * vs, M->blc_val, M->blc_num * vs, cudaMemcpyDeviceToDevice, s));
    }
    st = D->t->exchange(sends, recvs, s);
    if (st != AMGT_OK) { mbsr_release(&X, a); return st; }
    *Mx = X;
    return AMGT_OK;
}

// every rank's rows of a row-partitioned matrix (agglomeration): the plan whose extended range is
// everything
amgt_status allgather_rows(amgt_dist* D, const amgt_mbsr* M, amgt_mbsr* Mfull, Alloc& a, std::vector<int64_t>* rows) {
    std::vector<int64_t> off, mins, maxs;
    AMGT_TRY(gather_meta(D, M->m, 1, 0, off, mins, maxs, rows));
    Plan P;
    P.rank = D->rank;
    P.size = D->size;
    P.off = off;
    P.rb = off[D->rank];
    P.re = off[D->rank + 1];
    P.eb = 0;
    P.ee = off[D->size];
    for (int q = 0; q < D->size; ++q) {
        if (q == D->rank) continue;
        if (off[q + 1] > off[q]) P.recv.push_back({q, off[q], off[q + 1]});
        if (P.re > P.rb) P.send.push_back({q, P.rb, P.re});
    }
    const int64_t m_full = rows ? (*rows)[D->size] : 4 * off[D->size];
    return gather_rows(D, P, M, m_full, Mfull, a);
}

std::vector<Msg> msgs_of(const std::vector<Piece>& ps, const Plan& P, char* base, size_t elem, bool send) {
    std::vector<Msg> out;
    for (const Piece& p : ps) {
        (void)send;
        out.push_back({p.peer, base + (size_t)(4 * (p.g0 - P.eb)) * elem, (size_t)(4 * (p.g1 - p.g0)) * elem});
    }
    return out;
}

}  // namespace

// ---- amgt_dist_spmv plans (per matrix)
struct amgt_dist::SpmvPlanD {
    int64_t m = 0, T = 0;
    const void* val = nullptr;
    Plan P;
    int64_t int0 = 0, int1 = 0;
    amgt_mbsr As{};  // columns shifted to the extended range
    amgt_prec vp = AMGT_FP64;
    void* xe = nullptr;
    size_t xe_bytes = 0;
    std::vector<Msg> sends, recvs;
};

amgt_dist::~amgt_dist() {
    for (auto& kv : plans) {
        Alloc a{nullptr, cs};
        release_view(&kv.second->As, a);
        if (kv.second->xe) cudaFreeAsync(kv.second->xe, cs);
    }
    if (cs) cudaStreamSynchronize(cs);
    t.reset();
    if (ready) cudaEventDestroy(ready);
    if (done) cudaEventDestroy(done);
    if (cs) cudaStreamDestroy(cs);
}

namespace {

amgt_status dist_init(amgt_dist* D) {
    AMGT_CUDA(cudaStreamCreateWithFlags(&D->cs, cudaStreamNonBlocking));
    AMGT_CUDA(cudaEventCreateWithFlags(&D->ready, cudaEventDisableTiming));
    AMGT_CUDA(cudaEventCreateWithFlags(&D->done, cudaEventDisableTiming));
    return AMGT_OK;
}

// halo exchange on the communication stream, ordered after everything on s so far; the caller
// makes s wait for D->done before the boundary rows
amgt_status halo_begin(amgt_dist* D, const std::vector<Msg>& sends, const std::vector<Msg>& recvs, cudaStream_t s) {
    if (sends.empty() && recvs.empty()) return AMGT_OK;
    AMGT_CUDA(cudaEventRecord(D->ready, s));
    AMGT_CUDA(cudaStreamWaitEvent(D->cs, D->ready, 0));
    AMGT_TRY(D->t->exchange(sends, recvs, D->cs));
    AMGT_CUDA(cudaEventRecord(D->done, D->cs));
    return AMGT_OK;
}

// y = epi(A xe) over the own block rows: interior rows while the halo is in flight, then the rest
amgt_status halo_spmv(amgt_dist* D, const amgt_mbsr* A, int64_t int0, int64_t int1, const std::vector<Msg>& sends,
                      const std::vector<Msg>& recvs, const void* xe, amgt_prec vp, void* y, EpiArgs ea, cudaStream_t s,
                      int tcls) {
    const bool comm = !(sends.empty() && recvs.empty());
    AMGT_TRY(halo_begin(D, sends, recvs, s));
    const int64_t BR = A->blc_row;
    auto run = [&](int64_t i0, int64_t i1) -> amgt_status {
        if (i1 <= i0) return AMGT_OK;
        ea.I0 = i0;
        ea.I1 = i1;
        return spmv_ex_impl(A, xe, vp, y, vp, ea, s, tcls);
    };
    const bool has_int = comm && int1 > int0;
    if (has_int) AMGT_TRY(run(int0, int1));
    if (comm) AMGT_CUDA(cudaStreamWaitEvent(s, D->done, 0));
    if (has_int) {
        AMGT_TRY(run(0, int0));
        AMGT_TRY(run(int1, BR));
    } else {
        AMGT_TRY(run(0, BR));
    }
    return AMGT_OK;
}

}  // namespace

// ================================================================== distributed hierarchy
struct amgt_dist_level_ {
    amgt_mbsr Ag{};      // own rows, global columns, level precision (owned; level 1: the caller's A)
    amgt_mbsr A{};       // view of Ag with tile columns shifted to the extended range (eb -> 0)
    int64_t nglob = 0;   // global rows
    amgt_mbsr P{}, R{};  // own fine rows x own coarse rows (local indices), R = P^T; level precision
    Plan h;
    int64_t m = 0, int0 = 0, int1 = 0, off = 0;  // off: own segment in the extended vector (elements)
    amgt_prec vprec = AMGT_FP64;
    void* xe[2] = {nullptr, nullptr};
    void *b = nullptr, *r = nullptr, *dinv = nullptr;
    void* vblock = nullptr;
    size_t vblock_bytes = 0;
    std::vector<Msg> hs[2], hr[2];  // halo messages of xe[0] / xe[1]
};

struct amgt_dist_hierarchy {
    amgt_dist* D = nullptr;
    int nlev = 0, ka = 0;  // levels [0, ka) distributed, [ka, nlev) agglomerated (tail hierarchy)
    amgt_vcycle_opts o{};
    amgt_allocator al{};
    bool has_al = false;
    cudaStream_t s = nullptr;
    amgt_dist_level_ L[8];
    amgt_hierarchy* tail = nullptr;
    amgt_mbsr Atail{};               // the agglomerated level's operator (borrowed by tail)
    amgt_mbsr Ptail[8] = {};         // the gathered P_k of the agglomerated levels (tail shares their structure)
    std::vector<int64_t> tail_rows;  // row offsets of level ka per rank (size + 1)
    void *bfull = nullptr, *xfull = nullptr;
    size_t full_bytes = 0;
    amgt_prec tail_vprec = AMGT_FP64;
    std::vector<Msg> tail_sends, tail_recvs;  // in-place all-gather of b_ka
    double *norms = nullptr, *part = nullptr;
    int norms_cap = 0;
    int64_t calls = 0;
    Alloc alloc() { return Alloc{has_al ? &al : nullptr, s}; }
};

namespace {

void dh_destroy(amgt_dist_hierarchy* H) {
    if (!H) return;
    Alloc a = H->alloc();
    for (int k = 0; k < H->nlev; ++k) {
        auto& L = H->L[k];
        release_view(&L.A, a);
        mbsr_release(&L.Ag, a);
        mbsr_release(&L.P, a);
        mbsr_release(&L.R, a);
        a.put(L.vblock, L.vblock_bytes);
    }
    if (H->tail) hierarchy_free(H->tail);
    mbsr_release(&H->Atail, a);
    for (auto& P : H->Ptail) mbsr_release(&P, a);
    a.put(H->bfull, H->full_bytes);
    a.put(H->xfull, H->full_bytes);
    a.put(H->norms, (size_t)H->norms_cap * sizeof(double));
    a.put(H->part, NB * sizeof(double));
    cudaStreamSynchronize(H->s);
    delete H;
}

// coarse partition of P_k (own fine rows, global coarse columns): the own coarse rows are the
// contiguous tile-column range its columns cover; the ranges must tile the coarse level in rank
// order (aggregates never straddle ranks — true for the z-slab partition of the configs)
amgt_status coarse_range(amgt_dist* D, const amgt_mbsr* P, cudaStream_t s, int64_t& cb, int64_t& ce, bool& ok) {
    int64_t mn, mx;
    AMGT_TRY(col_minmax(P, s, mn, mx));
    int64_t mine[2] = {mn, mx};
    std::vector<int64_t> all(2 * D->size);
    AMGT_TRY(D->t->allgather_host(mine, all.data(), sizeof(mine)));
    int64_t pos = 0;
    ok = true;
    for (int q = 0; q < D->size && ok; ++q) {
        const int64_t a = all[2 * q], b = all[2 * q + 1];
        if (a > b) continue;  // no coarse rows
        if (a != pos) ok = false;
        pos = b + 1;
    }
    if (pos != P->blc_col) ok = false;
    cb = mn <= mx ? mn : 0;
    ce = mn <= mx ? mx + 1 : 0;
    return AMGT_OK;
}

amgt_status level_vectors(amgt_dist_level_& L, Alloc& a, cudaStream_t s) {
    const size_t e = vbytes(L.vprec);
    const int64_t next = 4 * (L.h.ee - L.h.eb), nown = 4 * L.A.blc_row;
    const size_t xb = ((size_t)next * e + 255) & ~size_t(255), ob = ((size_t)nown * e + 255) & ~size_t(255);
    L.vblock_bytes = 2 * xb + 3 * ob;
    L.vblock = a.get(L.vblock_bytes);
    if (!L.vblock) return fail(AMGT_ERR_ALLOC, "distributed level vectors: allocation failed");
    AMGT_CUDA(cudaMemsetAsync(L.vblock, 0, L.vblock_bytes, s));
    char* p = (char*)L.vblock;
    L.xe[0] = p;
    L.xe[1] = p + xb;
    L.b = p + 2 * xb;
    L.r = p + 2 * xb + ob;
    L.dinv = p + 2 * xb + 2 * ob;
    L.off = 4 * (L.h.rb - L.h.eb);
    for (int i = 0; i < 2; ++i) {
        L.hs[i] = msgs_of(L.h.send, L.h, (char*)L.xe[i], e, true);
        L.hr[i] = msgs_of(L.h.recv, L.h, (char*)L.xe[i], e, false);
    }
    return AMGT_OK;
}

// distributed level k from its own rows Ag (global columns, level precision): plan, shifted copy,
// SpMV analysis, vectors, D^-1
amgt_status setup_level(amgt_dist_hierarchy* H, int k, const amgt_mbsr* Ag) {
    cudaStream_t s = H->s;
    Alloc a = H->alloc();
    auto& L = H->L[k];
    L.m = Ag->m;
    L.nglob = Ag->n;
    AMGT_TRY(make_plan(H->D, Ag->m, Ag, s, L.h));
    trace_point("dist plan", s);
    AMGT_TRY(interior_rows(Ag, L.h, s, L.int0, L.int1));
    trace_point("dist interior", s);
    const int64_t n_ext = std::min<int64_t>(4 * L.h.ee, Ag->n) - 4 * L.h.eb;
    AMGT_TRY(shifted_view(Ag, -L.h.eb, n_ext, &L.A, a));
    AMGT_TRY(spmv_analyze_impl(&L.A, a));
    L.vprec = k == 0 ? AMGT_FP64 : vec_prec(H->o.level_prec[k]);
    AMGT_TRY(level_vectors(L, a, s));
    AMGT_TRY(dinv_impl(L.A, L.h.rb - L.h.eb, L.dinv, L.vprec, s, H->o.smoother == AMGT_SMOOTH_L1_JACOBI));
    trace_point("dist level vectors", s);
    return AMGT_OK;
}

// Galerkin product of distributed level k (Alg. 1 line 5) in level k's precision: P rows of the
// halo gathered, AP = A_k P_ext, A_{k+1} own rows = R_loc (AP) with R_loc = P_loc^T (aggregates are
// rank-local, so R's columns are the own fine rows).  Ac: own coarse rows, global coarse columns.
amgt_status setup_rap(amgt_dist_hierarchy* H, int k, const amgt_mbsr* Pin, int64_t cb, int64_t ce, amgt_mbsr* Ac) {
    Alloc a = H->alloc();
    auto& L = H->L[k];
    const amgt_prec pk = H->o.level_prec[k];
    if (Pin->m != L.m) return fail(AMGT_ERR_ARG, "P[%d] has %lld rows, the rank's level has %lld", k, (long long)Pin->m,
                                   (long long)L.m);
    amgt_mbsr Pext{}, Pext_k{}, AP{}, C{};
    const int64_t m_ext = std::min<int64_t>(4 * L.h.ee, L.nglob) - 4 * L.h.eb;
    AMGT_TRY(gather_rows(H->D, L.h, Pin, m_ext, &Pext, a));
    trace_point("dist P gather", H->s);
    amgt_status st = cast_impl(&Pext, pk, &Pext_k, a, nullptr);
    if (st == AMGT_OK) {
        // the cast shares Pext's structure: hand the structure to Pext_k
        Pext_k.own |= 1u;
        Pext.own &= ~1u;
        mbsr_release(&Pext, a);
        Pext_k.row_max = 0;
        st = spgemm_symbolic_impl(&L.A, &Pext_k, &AP, nullptr, a);
    } else {
        mbsr_release(&Pext, a);
    }
    if (st == AMGT_OK) st = spgemm_numeric_impl(&L.A, &Pext_k, &AP, a);
    trace_point("dist A P", H->s);
    mbsr_release(&Pext_k, a);
    if (st == AMGT_OK) st = copy_shifted(Pin, -cb, std::min<int64_t>(4 * ce, Pin->n) - 4 * cb, pk, &L.P, a);
    if (st == AMGT_OK) st = transpose_impl(&L.P, &L.R, a, nullptr);
    if (st == AMGT_OK) st = spgemm_symbolic_impl(&L.R, &AP, &C, nullptr, a);
    if (st == AMGT_OK) st = spgemm_numeric_impl(&L.R, &AP, &C, a);
    trace_point("dist R AP", H->s);
    mbsr_release(&AP, a);
    if (st == AMGT_OK) st = spmv_analyze_impl(&L.P, a);
    if (st == AMGT_OK) st = spmv_analyze_impl(&L.R, a);
    if (st != AMGT_OK) {
        mbsr_release(&C, a);
        return st;
    }
    *Ac = C;
    return AMGT_OK;
}

amgt_status dh_create(amgt_dist_hierarchy* H, const amgt_mbsr* A, const amgt_mbsr* const* P, int64_t agg_rows) {
    amgt_dist* D = H->D;
    cudaStream_t s = H->s;
    Alloc a = H->alloc();
    const int nlev = H->nlev;
    // first agglomerated level: the first (below level 1) with at most agg_rows global rows, the
    // coarsest at the latest; one rank = everything replicated (the single-GPU hierarchy)
    int ka = nlev - 1;
    if (D->size == 1) ka = 0;
    else
        for (int k = 1; k < nlev; ++k)
            if (P[k - 1]->n <= agg_rows) { ka = k; break; }
    H->ka = ka;
    amgt_mbsr cur{};  // own rows of the next level, global columns (owned until handed to a level)
    amgt_status st = AMGT_OK;
    for (int k = 0; k < ka && st == AMGT_OK; ++k) {
        if (k > 0) {
            H->L[k].Ag = cur;  // the level owns its operator; its shifted view borrows from it
            cur = amgt_mbsr{};
        }
        // a level whose aggregates straddle ranks (its coarse rows do not form contiguous ranges in
        // rank order — e.g. one grid plane per rank) is the first agglomerated one
        const amgt_mbsr* Ak = k == 0 ? A : &H->L[k].Ag;
        if (P[k]->m != Ak->m) {
            st = fail(AMGT_ERR_ARG, "P[%d] has %lld rows, the rank's level has %lld", k, (long long)P[k]->m,
                      (long long)Ak->m);
            break;
        }
        int64_t cb = 0, ce = 0;
        bool tiles = true;
        st = coarse_range(D, P[k], s, cb, ce, tiles);
        trace_point("dist coarse range", s);
        if (st != AMGT_OK) break;
        if (!tiles) {
            ka = H->ka = k;
            if (k > 0) {  // back to `cur`: the agglomeration below gathers it
                cur = H->L[k].Ag;
                H->L[k].Ag = amgt_mbsr{};
            }
            break;
        }
        st = setup_level(H, k, Ak);
        amgt_mbsr Ac{};
        if (st == AMGT_OK) st = setup_rap(H, k, P[k], cb, ce, &Ac);
        if (st != AMGT_OK) break;
        const amgt_prec pn = H->o.level_prec[k + 1];
        if (pn != Ac.prec) {
            amgt_mbsr Cn{};
            st = cast_impl(&Ac, pn, &Cn, a, nullptr);
            if (st == AMGT_OK) {
                Ac.own &= ~1u;
                mbsr_release(&Ac, a);
                Cn.own |= 1u;
                cur = Cn;
            } else {
                mbsr_release(&Ac, a);
            }
        } else {
            cur = Ac;
        }
    }
    if (st != AMGT_OK) {
        mbsr_release(&cur, a);
        return st;
    }
    // agglomerated levels ka..nlev-1: every rank's rows of A_ka and of P_ka..P_{M-1}
    const amgt_mbsr* Aka = ka == 0 ? A : &cur;
    if (D->size == 1) {  // nothing to gather: borrow (level 1: the caller's A)
        if (ka == 0) {
            H->Atail = *A;
            H->Atail.own = 0;
            H->Atail.aux = nullptr;
        } else {
            H->Atail = cur;
            cur = amgt_mbsr{};
        }
        H->tail_rows = {0, Aka == A ? A->m : H->Atail.m};
    } else {
        st = allgather_rows(D, Aka, &H->Atail, a, &H->tail_rows);
        mbsr_release(&cur, a);
        AMGT_TRY(st);
    }
    if (H->Atail.prec != H->o.level_prec[ka]) {
        amgt_mbsr Cn{};
        AMGT_TRY(cast_impl(&H->Atail, H->o.level_prec[ka], &Cn, a, nullptr));
        H->Atail.own &= ~1u;
        mbsr_release(&H->Atail, a);
        Cn.own |= 1u;
        H->Atail = Cn;
    }
    amgt_mbsr* Pf = H->Ptail;  // kept for the tail's lifetime: its P_k (a cast) shares their structure
    std::vector<const amgt_mbsr*> Pp(nlev, nullptr);
    trace_point("dist gather A_tail", s);
    for (int k = ka; k + 1 < nlev && st == AMGT_OK; ++k) {
        if (D->size == 1) {
            Pp[k - ka] = P[k];
            continue;
        }
        st = allgather_rows(D, P[k], &Pf[k], a, nullptr);
        Pp[k - ka] = &Pf[k];
    }
    if (st == AMGT_OK) {
        amgt_vcycle_opts ot = H->o;
        for (int k = 0; k < 8; ++k) ot.level_prec[k] = k + ka < 8 ? H->o.level_prec[k + ka] : AMGT_FP16;
        ot.max_levels = nlev - ka;
        if (ka == 0) {  // replicated whole problem: exactly the single-GPU hierarchy
            amgt_hierarchy* T = nullptr;
            st = amgt_hierarchy_create(&H->Atail, Pp.data(), nlev, &ot, H->has_al ? &H->al : nullptr, s, &T);
            H->tail = T;
        } else {
            st = hierarchy_create_tail(&H->Atail, Pp.data(), nlev - ka, &ot, H->has_al ? &H->al : nullptr, s, &H->tail);
        }
    }
    AMGT_TRY(st);
    trace_point("dist tail hierarchy", s);
    if (ka > 0) {
        H->tail_vprec = hierarchy_vprec0(H->tail);
        const size_t e = vbytes(H->tail_vprec);
        H->full_bytes = (size_t)hierarchy_npad0(H->tail) * e;
        H->bfull = a.get(H->full_bytes);
        H->xfull = a.get(H->full_bytes);
        if (!H->bfull || !H->xfull) return fail(AMGT_ERR_ALLOC, "agglomerated level vectors: allocation failed");
        AMGT_CUDA(cudaMemsetAsync(H->bfull, 0, H->full_bytes, s));
        AMGT_CUDA(cudaMemsetAsync(H->xfull, 0, H->full_bytes, s));
        const auto& off = H->tail_rows;
        const int me = D->rank;
        for (int q = 0; q < D->size; ++q) {
            if (q == me) continue;
            const size_t my_n = (size_t)(off[me + 1] - off[me]), q_n = (size_t)(off[q + 1] - off[q]);
            if (my_n) H->tail_sends.push_back({q, (char*)H->bfull + off[me] * e, my_n * e});
            if (q_n) H->tail_recvs.push_back({q, (char*)H->bfull + off[q] * e, q_n * e});
        }
    }
    H->part = (double*)a.get(NB * sizeof(double));
    if (!H->part) return fail(AMGT_ERR_ALLOC, "norm partial allocation failed");
    AMGT_CUDA(cudaStreamSynchronize(s));
    trace_dump();
    return AMGT_OK;
}

// ---- solve
void* own_seg(const amgt_dist_level_& L, int i) { return (char*)L.xe[i] + L.off * vbytes(L.vprec); }

// levels below this many own block rows skip the interior / boundary split (one launch after the
// halo instead of three: launch latency dominates there)
static int64_t split_min_br() {
    static int64_t v = -1;
    if (v < 0) {
        const char* e = getenv("AMGT_DIST_SPLIT_MIN_BR");
        v = e ? atoll(e) : 16384;
    }
    return v;
}

amgt_status dspmv(amgt_dist_hierarchy* H, int k, int src, void* y, int mode, const void* b, const void* xs,
                  void* r = nullptr) {
    auto& L = H->L[k];
    H->calls += mode == AMGT_EPI_JACOBI_RES ? 2 : 1;  // the fused sweep stands for two of Alg. 2's SpMVs
    EpiArgs ea{mode, b, L.dinv, xs, H->o.omega, 0, -1};
    ea.r = r;
    const bool split = L.A.blc_row >= split_min_br();
    return halo_spmv(H->D, &L.A, split ? L.int0 : 0, split ? L.int1 : 0, L.hs[src], L.hr[src], L.xe[src], L.vprec, y,
                     ea, H->s, k == 0 ? TC_SPMV_L1 : TC_SPMV);
}

amgt_status local_spmv(amgt_dist_hierarchy* H, const amgt_mbsr* M, const void* x, amgt_prec xp, void* y, amgt_prec yp,
                       int mode) {
    ++H->calls;
    return spmv_ex_impl(M, x, xp, y, yp, EpiArgs{mode, nullptr, nullptr, nullptr, H->o.omega, 0, -1}, H->s, TC_SPMV);
}

amgt_status dh_vcycle(amgt_dist_hierarchy* H, const double* b, double* x, int ncycles, double* res_host,
                      int64_t* calls_host) {
    cudaStream_t s = H->s;
    amgt_dist* D = H->D;
    H->calls = 0;
    if (H->ka == 0) {  // everything replicated: the single-GPU V-cycle
        AMGT_TRY(amgt_vcycle(H->tail, b, x, ncycles, res_host, calls_host, s));
        return AMGT_OK;
    }
    PdlScope pdl;  // solve kernels with programmatic dependent launch (as amgt_vcycle)
    Alloc a = H->alloc();
    if (ncycles + 1 > H->norms_cap) {
        a.put(H->norms, (size_t)H->norms_cap * sizeof(double));
        H->norms_cap = ncycles + 1;
        H->norms = (double*)a.get((size_t)H->norms_cap * sizeof(double));
        if (!H->norms) return fail(AMGT_ERR_ALLOC, "norm buffer allocation failed");
    }
    const int ka = H->ka;
    constexpr int JAC = AMGT_EPI_JACOBI, RES = AMGT_EPI_RESIDUAL, ACC = AMGT_EPI_ACCUM;
    int cur[8] = {0};
    auto& L0 = H->L[0];
    const size_t tail_e = vbytes(H->tail_vprec);
    char* b_tail_own = (char*)H->bfull + H->tail_rows[D->rank] * tail_e;
    char* x_tail_own = (char*)H->xfull + H->tail_rows[D->rank] * tail_e;
    AMGT_CUDA(cudaMemcpyAsync(own_seg(L0, 0), x, L0.m * sizeof(double), cudaMemcpyDeviceToDevice, s));
    auto norm_of_r = [&](int slot) -> amgt_status {  // ||r_1||^2 over all ranks into norms[slot]
        k_sq_partial<<<NB, 256, 0, s>>>(4 * L0.A.blc_row, (const double*)L0.r, H->part);
        AMGT_LAUNCHED();
        k_sq_final<<<1, 32, 0, s>>>(H->part, H->norms + slot);
        AMGT_LAUNCHED();
        return D->t->allreduce_f64(H->norms + slot, 1, s);
    };
    auto resnorm = [&](int slot) -> amgt_status {
        AMGT_TRY(dspmv(H, 0, cur[0], L0.r, RES, b, nullptr));
        return norm_of_r(slot);
    };
    // the residual after cycle c (L308) comes from cycle c+1's first level-1 pre-smoothing sweep
    // (AMGT_EPI_JACOBI_RES, same x and arithmetic); only the last cycle needs its own pass
    const bool fused = H->o.nu1 >= 1;
    auto smooth = [&](int k, const void* bk, int sweeps, int norm_slot) -> amgt_status {
        auto& L = H->L[k];
        for (int i = 0; i < sweeps; ++i) {
            const int src = cur[k], dst = 1 - src;
            if (i == 0 && norm_slot >= 0) {
                AMGT_TRY(dspmv(H, k, src, own_seg(L, dst), AMGT_EPI_JACOBI_RES, bk, own_seg(L, src), L.r));
                AMGT_TRY(norm_of_r(norm_slot));
            } else {
                AMGT_TRY(dspmv(H, k, src, own_seg(L, dst), JAC, bk, own_seg(L, src)));
            }
            cur[k] = dst;
        }
        return AMGT_OK;
    };
    if (!fused || ncycles == 0) AMGT_TRY(resnorm(0));
    for (int cyc = 1; cyc <= ncycles; ++cyc) {
        for (int k = 0; k < ka; ++k) {  // Alg. 2 lines 1-5 on the distributed levels
            auto& L = H->L[k];
            const void* bk = k == 0 ? (const void*)b : L.b;
            int sweeps = H->o.nu1;
            if (k > 0) {
                const int64_t nk = 4 * L.A.blc_row;
                if (H->o.nu1 >= 1) {  // zero initial guess: the first sweep is w D^-1 b (no SpMV, no halo)
                    if (L.vprec == AMGT_FP64)
                        k_zero_sweep<double><<<(unsigned)ceil_div(nk, 256), 256, 0, s>>>(
                            nk, (const double*)bk, (const double*)L.dinv, H->o.omega, (double*)own_seg(L, 1));
                    else
                        k_zero_sweep<float><<<(unsigned)ceil_div(nk, 256), 256, 0, s>>>(
                            nk, (const float*)bk, (const float*)L.dinv, (float)H->o.omega, (float*)own_seg(L, 1));
                    AMGT_LAUNCHED();
                    ++H->calls;  // Alg. 2's sweep (its SpMV is A 0 = 0)
                    cur[k] = 1;
                    sweeps = H->o.nu1 - 1;
                } else {
                    cur[k] = 0;
                    AMGT_CUDA(cudaMemsetAsync(own_seg(L, 0), 0, nk * vbytes(L.vprec), s));
                }
            }
            AMGT_TRY(smooth(k, bk, sweeps, (k == 0 && fused) ? cyc - 1 : -1));
            AMGT_TRY(dspmv(H, k, cur[k], L.r, RES, bk, nullptr));
            if (k + 1 < ka) {
                auto& N = H->L[k + 1];
                AMGT_TRY(local_spmv(H, &L.R, L.r, L.vprec, N.b, N.vprec, AMGT_EPI_Y));
            } else {  // line 4 into the own segment of the agglomerated right-hand side
                AMGT_TRY(local_spmv(H, &L.R, L.r, L.vprec, b_tail_own, H->tail_vprec, AMGT_EPI_Y));
            }
        }
        // levels ka..M on every rank: all-gather b_ka (in place), one V-cycle of the tail
        AMGT_TRY(D->t->exchange(H->tail_sends, H->tail_recvs, s));
        AMGT_TRY(hierarchy_apply(H->tail, H->bfull, H->xfull, s, &H->calls));
        for (int k = ka - 1; k >= 0; --k) {  // lines 7-11
            auto& L = H->L[k];
            const void* bk = k == 0 ? (const void*)b : L.b;
            const void* xn = k + 1 < ka ? own_seg(H->L[k + 1], cur[k + 1]) : (const void*)x_tail_own;
            const amgt_prec np = k + 1 < ka ? H->L[k + 1].vprec : H->tail_vprec;
            AMGT_TRY(local_spmv(H, &L.P, xn, np, own_seg(L, cur[k]), L.vprec, ACC));
            AMGT_TRY(smooth(k, bk, H->o.nu2, -1));
        }
        if (!fused || cyc == ncycles) AMGT_TRY(resnorm(cyc));
    }
    AMGT_CUDA(cudaMemcpyAsync(x, own_seg(L0, cur[0]), L0.m * sizeof(double), cudaMemcpyDeviceToDevice, s));
    std::vector<double> hn(ncycles + 1);
    AMGT_CUDA(cudaMemcpyAsync(hn.data(), H->norms, (ncycles + 1) * sizeof(double), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaStreamSynchronize(s));
    if (res_host)
        for (int i = 0; i <= ncycles; ++i) res_host[i] = std::sqrt(hn[i]);
    if (calls_host) *calls_host = H->calls;
    return AMGT_OK;
}

}  // namespace

// ================================================================== C ABI
extern "C" {

amgt_status amgt_nccl_unique_id(void* id128_host) {
    if (!id128_host) return fail(AMGT_ERR_ARG, "amgt_nccl_unique_id: NULL");
    AMGT_TRY(load_nccl());
    nccl_uid u;
    AMGT_NCCL(g_nccl.GetUniqueId(&u));
    std::copy(u.internal, u.internal + 128, (char*)id128_host);
    return AMGT_OK;
}

amgt_status amgt_dist_create(const void* id128_host, int rank, int size, int64_t row_begin, int64_t row_end,
                             amgt_dist** Dout) {
    if (!id128_host || !Dout || size < 1 || rank < 0 || rank >= size || row_begin < 0 || row_end < row_begin)
        return fail(AMGT_ERR_ARG, "amgt_dist_create: bad argument");
    AMGT_TRY(load_nccl());
    nccl_uid u;
    std::copy((const char*)id128_host, (const char*)id128_host + 128, u.internal);
    auto T = std::make_unique<NcclTransport>();
    T->rank = rank;
    T->size = size;
    nccl_result r = g_nccl.CommInitRank(&T->comm, size, u, rank);
    if (r != 0) return fail(AMGT_ERR_NCCL, "ncclCommInitRank: %s", g_nccl.GetErrorString ? g_nccl.GetErrorString(r) : "?");
    AMGT_CUDA(cudaStreamCreateWithFlags(&T->hs, cudaStreamNonBlocking));
    amgt_dist* D = new amgt_dist();
    D->t = std::move(T);
    D->rank = rank;
    D->size = size;
    D->row_begin = row_begin;
    D->row_end = row_end;
    const amgt_status st = dist_init(D);
    if (st != AMGT_OK) {
        delete D;
        return st;
    }
    *Dout = D;
    return AMGT_OK;
}

amgt_status amgt_dist_group_create(int size, amgt_dist_group** G) {
    if (!G || size < 1 || size > LOOP_MAX) return fail(AMGT_ERR_ARG, "amgt_dist_group_create: size must be 1..%d", LOOP_MAX);
    *G = new amgt_dist_group();
    (*G)->size = size;
    return AMGT_OK;
}

amgt_status amgt_dist_group_abort(amgt_dist_group* G) {
    if (!G) return fail(AMGT_ERR_ARG, "amgt_dist_group_abort: NULL");
    {
        std::lock_guard<std::mutex> lk(G->mu);
        G->aborted = true;
    }
    G->cv.notify_all();
    return AMGT_OK;
}

amgt_status amgt_dist_group_destroy(amgt_dist_group* G) {
    delete G;
    return AMGT_OK;
}

amgt_status amgt_dist_create_loopback(amgt_dist_group* G, int rank, int64_t row_begin, int64_t row_end,
                                      amgt_dist** Dout) {
    if (!G || !Dout || rank < 0 || rank >= G->size || row_begin < 0 || row_end < row_begin)
        return fail(AMGT_ERR_ARG, "amgt_dist_create_loopback: bad argument");
    auto T = std::make_unique<LoopTransport>();
    T->rank = rank;
    T->size = G->size;
    T->g = G;
    amgt_dist* D = new amgt_dist();
    D->t = std::move(T);
    D->rank = rank;
    D->size = G->size;
    D->row_begin = row_begin;
    D->row_end = row_end;
    const amgt_status st = dist_init(D);
    if (st != AMGT_OK) {
        delete D;
        return st;
    }
    *Dout = D;
    return AMGT_OK;
}

amgt_status amgt_dist_destroy(amgt_dist* D) {
    delete D;
    return AMGT_OK;
}

amgt_status amgt_dist_allreduce_sum(amgt_dist* D, double* buf, int64_t count, void* stream) {
    if (!D || (!buf && count) || count < 0) return fail(AMGT_ERR_ARG, "amgt_dist_allreduce_sum: bad argument");
    return D->t->allreduce_f64(buf, count, (cudaStream_t)stream);
}

amgt_status amgt_dist_plan_host(int rank, int size, const int64_t* rows, const int64_t* colmin, const int64_t* colmax,
                                int64_t* ext_host, amgt_dist_piece* recv, int* nrecv, amgt_dist_piece* send, int* nsend,
                                int cap) {
    if (size < 1 || rank < 0 || rank >= size || !rows || !colmin || !colmax || !ext_host || !nrecv || !nsend ||
        cap < 0 || (cap > 0 && (!recv || !send)))
        return fail(AMGT_ERR_ARG, "amgt_dist_plan_host: bad argument");
    std::vector<int64_t> off(size + 1, 0);
    for (int q = 0; q < size; ++q) {
        if (rows[q] < 0 || (q + 1 < size && rows[q] % 4))
            return fail(AMGT_ERR_UNSUPPORTED, "amgt_dist_plan_host: rank %d owns %lld rows", q, (long long)rows[q]);
        off[q + 1] = off[q] + ceil_div(rows[q], 4);
    }
    Plan P;
    plan_from_meta(rank, size, off, colmin, colmax, P);
    ext_host[0] = P.eb;
    ext_host[1] = P.ee;
    *nrecv = (int)P.recv.size();
    *nsend = (int)P.send.size();
    if ((int)P.recv.size() > cap || (int)P.send.size() > cap)
        return fail(AMGT_ERR_ARG, "amgt_dist_plan_host: %zu/%zu pieces exceed cap %d", P.recv.size(), P.send.size(), cap);
    for (size_t i = 0; i < P.recv.size(); ++i) recv[i] = {P.recv[i].peer, P.recv[i].g0, P.recv[i].g1};
    for (size_t i = 0; i < P.send.size(); ++i) send[i] = {P.send[i].peer, P.send[i].g0, P.send[i].g1};
    return AMGT_OK;
}

amgt_status amgt_dist_spmv(amgt_dist* D, const amgt_mbsr* A, const void* x_local, void* y_local, void* stream) {
    if (!D || !A || (A->blc_row > 0 && (!x_local || !y_local))) return fail(AMGT_ERR_ARG, "amgt_dist_spmv: bad argument");
    if (!prec_valid(A->prec)) return fail(AMGT_ERR_ARG, "amgt_dist_spmv: bad precision");
    cudaStream_t s = (cudaStream_t)stream;
    Alloc a{nullptr, s};
    auto& slot = D->plans[(const void*)A->blc_idx];
    if (!slot || slot->m != A->m || slot->T != A->blc_num || slot->val != A->blc_val) {
        if (slot) {
            release_view(&slot->As, a);
            if (slot->xe) cudaFreeAsync(slot->xe, s);
        }
        slot = std::make_unique<amgt_dist::SpmvPlanD>();
        auto& Q = *slot;
        Q.m = A->m;
        Q.T = A->blc_num;
        Q.val = A->blc_val;
        AMGT_TRY(make_plan(D, A->m, A, s, Q.P));
        if (4 * Q.P.off[D->size] != 4 * ceil_div(A->n, 4))
            return fail(AMGT_ERR_ARG, "amgt_dist_spmv: A has %lld columns, the ranks own %lld rows", (long long)A->n,
                        (long long)(4 * Q.P.off[D->size]));
        AMGT_TRY(interior_rows(A, Q.P, s, Q.int0, Q.int1));
        const int64_t n_ext = std::min<int64_t>(4 * Q.P.ee, A->n) - 4 * Q.P.eb;
        AMGT_TRY(shifted_view(A, -Q.P.eb, n_ext, &Q.As, a));
        AMGT_TRY(spmv_analyze_impl(&Q.As, a));
        Q.vp = vec_prec(A->prec);
        Q.xe_bytes = (size_t)4 * (Q.P.ee - Q.P.eb) * vbytes(Q.vp) + 16;
        AMGT_CUDA(cudaMallocAsync(&Q.xe, Q.xe_bytes, s));
        AMGT_CUDA(cudaMemsetAsync(Q.xe, 0, Q.xe_bytes, s));
        Q.sends = msgs_of(Q.P.send, Q.P, (char*)Q.xe, vbytes(Q.vp), true);
        Q.recvs = msgs_of(Q.P.recv, Q.P, (char*)Q.xe, vbytes(Q.vp), false);
    }
    auto& Q = *slot;
    const size_t e = vbytes(Q.vp);
    if (A->m > 0)
        AMGT_CUDA(cudaMemcpyAsync((char*)Q.xe + 4 * (Q.P.rb - Q.P.eb) * e, x_local, A->m * e, cudaMemcpyDeviceToDevice, s));
    return halo_spmv(D, &Q.As, Q.int0, Q.int1, Q.sends, Q.recvs, Q.xe, Q.vp, y_local,
                     EpiArgs{AMGT_EPI_Y, nullptr, nullptr, nullptr, 0.0, 0, -1}, s, TC_SPMV);
}

amgt_status amgt_dist_rap(amgt_dist* D, const amgt_mbsr* R_l, const amgt_mbsr* A_l, const amgt_mbsr* P_l, amgt_mbsr* Ac_l,
                          const amgt_allocator* al, void* stream) {
    if (!D || !R_l || !A_l || !P_l || !Ac_l) return fail(AMGT_ERR_ARG, "amgt_dist_rap: NULL argument");
    if (A_l->prec != P_l->prec || A_l->prec != R_l->prec) return fail(AMGT_ERR_ARG, "amgt_dist_rap: precisions differ");
    if (P_l->m != A_l->m) return fail(AMGT_ERR_ARG, "amgt_dist_rap: P_l has %lld rows, A_l %lld", (long long)P_l->m,
                                      (long long)A_l->m);
    cudaStream_t s = (cudaStream_t)stream;
    Alloc a{al, s};
    Plan hA, hR;
    std::vector<int64_t> rows;
    AMGT_TRY(make_plan(D, A_l->m, A_l, s, hA, &rows));
    const int64_t n_fine = rows[D->size];
    amgt_mbsr Pext{}, As{}, AP{}, APext{}, Rs{}, C{};
    auto cleanup = [&] {
        mbsr_release(&Pext, a);
        release_view(&As, a);
        mbsr_release(&AP, a);
        mbsr_release(&APext, a);
        release_view(&Rs, a);
    };
    amgt_status st = gather_rows(D, hA, P_l, std::min<int64_t>(4 * hA.ee, n_fine) - 4 * hA.eb, &Pext, a);
    if (st == AMGT_OK)
        st = shifted_view(A_l, -hA.eb, std::min<int64_t>(4 * hA.ee, A_l->n) - 4 * hA.eb, &As, a);
    if (st == AMGT_OK) st = spgemm_symbolic_impl(&As, &Pext, &AP, nullptr, a);
    if (st == AMGT_OK) st = spgemm_numeric_impl(&As, &Pext, &AP, a);
    // R_l's columns index the fine rows, i.e. AP's row partition (= A's)
    if (st == AMGT_OK) st = make_plan(D, A_l->m, R_l, s, hR);
    if (st == AMGT_OK) st = gather_rows(D, hR, &AP, std::min<int64_t>(4 * hR.ee, n_fine) - 4 * hR.eb, &APext, a);
    if (st == AMGT_OK)
        st = shifted_view(R_l, -hR.eb, std::min<int64_t>(4 * hR.ee, R_l->n) - 4 * hR.eb, &Rs, a);
    if (st == AMGT_OK) st = spgemm_symbolic_impl(&Rs, &APext, &C, nullptr, a);
    if (st == AMGT_OK) st = spgemm_numeric_impl(&Rs, &APext, &C, a);
    cleanup();
    if (st != AMGT_OK) {
        mbsr_release(&C, a);
        return st;
    }
    *Ac_l = C;
    return AMGT_OK;
}

amgt_status amgt_dist_allgather_mbsr(amgt_dist* D, const amgt_mbsr* M_l, amgt_mbsr* M_full, const amgt_allocator* al,
                                     void* stream) {
    if (!D || !M_l || !M_full) return fail(AMGT_ERR_ARG, "amgt_dist_allgather_mbsr: NULL argument");
    Alloc a{al, (cudaStream_t)stream};
    std::vector<int64_t> rows;
    return allgather_rows(D, M_l, M_full, a, &rows);
}

amgt_status amgt_dist_hierarchy_create(amgt_dist* D, const amgt_mbsr* A_l, const amgt_mbsr* const* P_l, int nlev,
                                       const amgt_vcycle_opts* o, int64_t agg_rows, const amgt_allocator* al,
                                       void* stream, amgt_dist_hierarchy** Hout) {
    if (!D || !A_l || !o || !Hout || nlev < 1 || nlev > 8 || (nlev > 1 && !P_l) || agg_rows < 0)
        return fail(AMGT_ERR_ARG, "amgt_dist_hierarchy_create: bad argument");
    if (A_l->prec != AMGT_FP64) return fail(AMGT_ERR_ARG, "amgt_dist_hierarchy_create: A_l must be FP64");
    if (A_l->m != D->row_end - D->row_begin)
        return fail(AMGT_ERR_ARG, "amgt_dist_hierarchy_create: A_l has %lld rows, the communicator's range has %lld",
                    (long long)A_l->m, (long long)(D->row_end - D->row_begin));
    for (int k = 0; k < nlev; ++k)
        if (!prec_valid(o->level_prec[k])) return fail(AMGT_ERR_ARG, "bad level precision %d", k);
    if (o->level_prec[0] != AMGT_FP64) return fail(AMGT_ERR_ARG, "amgt_dist_hierarchy_create: level 1 must be FP64");
    for (int k = 0; k + 1 < nlev; ++k)
        if (!P_l[k] || P_l[k]->prec != AMGT_FP64) return fail(AMGT_ERR_ARG, "P_l[%d] missing or not FP64", k);
    if (o->nu1 < 0 || o->nu2 < 0 || o->interp != AMGT_INTERP_GIVEN)
        return fail(AMGT_ERR_UNSUPPORTED, "amgt_dist_hierarchy_create: sweep counts >= 0 and given interpolation only");
    // the communicator's level-1 ranges must tile the rows in rank order
    {
        int64_t mine[2] = {D->row_begin, D->row_end};
        std::vector<int64_t> all(2 * D->size);
        AMGT_TRY(D->t->allgather_host(mine, all.data(), sizeof(mine)));
        int64_t pos = 0;
        for (int q = 0; q < D->size; ++q) {
            if (all[2 * q] != pos) return fail(AMGT_ERR_ARG, "rank %d's rows start at %lld, expected %lld", q,
                                               (long long)all[2 * q], (long long)pos);
            pos = all[2 * q + 1];
        }
        if (pos != A_l->n) return fail(AMGT_ERR_ARG, "the ranks own %lld rows, A has %lld columns", (long long)pos,
                                       (long long)A_l->n);
    }
    amgt_dist_hierarchy* H = new amgt_dist_hierarchy();
    H->D = D;
    H->nlev = nlev;
    H->o = *o;
    H->s = (cudaStream_t)stream;
    if (al) { H->al = *al; H->has_al = true; }
    const amgt_status st = dh_create(H, A_l, P_l, agg_rows);
    if (st != AMGT_OK) {
        dh_destroy(H);
        return st;
    }
    *Hout = H;
    return AMGT_OK;
}

amgt_status amgt_dist_vcycle(amgt_dist_hierarchy* H, const double* b_local, double* x_local, int ncycles,
                             double* res_norms_host, int64_t* spmv_calls_host, void* stream) {
    if (!H || ncycles < 0 || (H->L[0].m > 0 && (!b_local || !x_local)))
        return fail(AMGT_ERR_ARG, "amgt_dist_vcycle: bad argument");
    H->s = (cudaStream_t)stream;
    return dh_vcycle(H, b_local, x_local, ncycles, res_norms_host, spmv_calls_host);
}

amgt_status amgt_dist_hierarchy_info(const amgt_dist_hierarchy* H, amgt_dist_hier_info* out) {
    if (!H || !out) return fail(AMGT_ERR_ARG, "amgt_dist_hierarchy_info: NULL argument");
    *out = amgt_dist_hier_info{};
    out->nlev = H->nlev;
    out->agg_level = H->ka;
    for (int k = 0; k < H->ka; ++k) {
        const auto& L = H->L[k];
        out->rows[k] = L.m;
        out->row_begin[k] = 4 * L.h.rb;
        out->ext_begin[k] = 4 * L.h.eb;
        out->ext_end[k] = std::min<int64_t>(4 * L.h.ee, 4 * L.h.off[L.h.size]);
        out->halo_recv[k] = (int)L.h.recv.size();
        out->halo_send[k] = (int)L.h.send.size();
        out->interior[k][0] = L.int0;
        out->interior[k][1] = L.int1;
        out->tiles[k] = L.A.blc_num;
    }
    if (H->tail) {
        for (int k = H->ka; k < H->nlev; ++k) {
            const amgt_mbsr* Ak = nullptr;
            amgt_hierarchy_level(H->tail, k - H->ka, &Ak, nullptr, nullptr);
            if (Ak) {
                out->rows[k] = Ak->m;
                out->tiles[k] = Ak->blc_num;
            }
        }
    }
    return AMGT_OK;
}

amgt_status amgt_dist_hierarchy_destroy(amgt_dist_hierarchy* H) {
    dh_destroy(H);
    return AMGT_OK;
}

}  // extern "C"
