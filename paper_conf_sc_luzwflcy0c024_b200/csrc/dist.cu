// dist.cu — native distributed V-cycle over row slabs (the paper's 8-GPU runs
// go through HYPRE/MPI, L363-365).  NCCL is loaded at run time (dlopen of libnccl.so.2 — the
// same library torch.distributed already mapped), so libamgt has no link-time dependency.
//
// Per A_k SpMV: the own segment of the extended buffer is sent to the ranks whose halo it
// is and the halo is received (ncclSend/ncclRecv in one group on a communication stream,
// NVLink P2P on an NVSwitch box) while the interior block rows run on the compute stream;
// the boundary block rows follow once the halo has landed (event dependency, no host sync).
// R_k and P_k SpMVs are rank-local (aggregates never straddle slabs).  Norm: local
// deterministic reduction + ncclAllReduce on the device.  Coarsest level: the right-hand
// side is all-gathered (P2P, variable counts) and every rank applies the dense inverse.
// The plans (peers, offsets, counts, interior ranges) come from the host-side setup
// (paper_conf_sc_luzwflcy0c024_b200/dist.py).
#include <dlfcn.h>

#include <algorithm>
#include <cmath>
#include <vector>

#include "common.cuh"

namespace amgt {
amgt_status spmv_ex_impl(const amgt_mbsr* A, const void* x, amgt_prec xp, void* y, amgt_prec yp, const EpiArgs& ea,
                         cudaStream_t s, int timer_class);
}
using namespace amgt;

// ---- minimal NCCL ABI (nccl.h 2.x), resolved with dlsym
typedef struct {
    char internal[128];
} nccl_uid;
typedef void* nccl_comm;
typedef int nccl_result;
enum { NCCL_INT8 = 0, NCCL_FLOAT32 = 7, NCCL_FLOAT64 = 8 };
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
    const char* (*GetErrorString)(nccl_result) = nullptr;
};

static NcclApi g_nccl;

static amgt_status load_nccl() {
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
    g_nccl.GetErrorString = (decltype(g_nccl.GetErrorString))sym("ncclGetErrorString");
    if (!g_nccl.GetUniqueId || !g_nccl.CommInitRank || !g_nccl.Send || !g_nccl.Recv || !g_nccl.GroupStart ||
        !g_nccl.GroupEnd || !g_nccl.AllReduce || !g_nccl.CommDestroy)
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

struct amgt_dist {
    nccl_comm comm = nullptr;
    int rank = 0, size = 1;
    cudaStream_t cs = nullptr;  // communication stream
    cudaEvent_t ready = nullptr, done = nullptr;
};

namespace {

size_t vb(amgt_prec p) { return p == AMGT_FP64 ? 8 : 4; }
int nccl_type(amgt_prec p) { return p == AMGT_FP64 ? NCCL_FLOAT64 : NCCL_FLOAT32; }

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
// first pre-smoothing sweep of a coarse level from x = 0: x = 0 + w dinv .* (b - 0) on the own
// rows (the SpMV of the zero vector and its halo exchange are skipped; same expression as the
// single-GPU k_jacobi0)
template <typename V>
__global__ void k_zero_sweep(int64_t n, const V* __restrict__ b, const V* __restrict__ dinv, V omega,
                             V* __restrict__ x) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const V zero = V(0), t = V(0);
    x[i] = zero + omega * dinv[i] * (b[i] - t);
}

template <typename V>
__global__ void k_dense_apply(int64_t n, const double* __restrict__ Ainv, const V* __restrict__ b, V* __restrict__ x) {
    const int64_t row = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (row >= n) return;
    double s = 0.0;
    for (int64_t j = lane; j < n; j += 32) s = fma(Ainv[row * n + j], (double)b[j], s);
    for (int d = 16; d; d >>= 1) s += __shfl_xor_sync(0xffffffffu, s, d);
    if (lane == 0) x[row] = (V)s;
}

struct Ctx {
    amgt_dist* D;
    cudaStream_t s;
    double omega;
    int64_t calls = 0;
};

// halo exchange of extended buffer xe of level L (async on the comm stream)
amgt_status halo_begin(Ctx& c, const amgt_dist_level& L, void* xe) {
    if (L.nsend + L.nrecv == 0) return AMGT_OK;
    AMGT_CUDA(cudaEventRecord(c.D->ready, c.s));
    AMGT_CUDA(cudaStreamWaitEvent(c.D->cs, c.D->ready, 0));
    const size_t e = vb(L.vprec);
    AMGT_NCCL(g_nccl.GroupStart());
    for (int i = 0; i < L.nsend; ++i)
        AMGT_NCCL(g_nccl.Send((char*)xe + L.send_off[i] * e, (size_t)L.send_cnt[i], nccl_type(L.vprec), L.send_peer[i],
                              c.D->comm, c.D->cs));
    for (int i = 0; i < L.nrecv; ++i)
        AMGT_NCCL(g_nccl.Recv((char*)xe + L.recv_off[i] * e, (size_t)L.recv_cnt[i], nccl_type(L.vprec), L.recv_peer[i],
                              c.D->comm, c.D->cs));
    AMGT_NCCL(g_nccl.GroupEnd());
    AMGT_CUDA(cudaEventRecord(c.D->done, c.D->cs));
    return AMGT_OK;
}

// distributed A_k SpMV with epilogue: y = epi(A xe)
// r (AMGT_EPI_JACOBI_RES only): the residual of the sweep's input, written in the same pass
amgt_status dspmv(Ctx& c, const amgt_dist_level& L, int k, void* xe, void* y, int mode, const void* b, const void* xs,
                  void* r = nullptr) {
    c.calls += mode == AMGT_EPI_JACOBI_RES ? 2 : 1;  // the fused sweep stands for two of Alg. 2's SpMVs
    AMGT_TRY(halo_begin(c, L, xe));
    const int tcls = k == 0 ? TC_SPMV_L1 : TC_SPMV;
    const int64_t BR = L.A->blc_row;
    auto run = [&](int64_t i0, int64_t i1) -> amgt_status {
        if (i1 <= i0) return AMGT_OK;
        EpiArgs ea{mode, b, L.dinv, xs, c.omega, i0, i1};
        ea.r = r;
        return spmv_ex_impl(L.A, xe, L.vprec, y, L.vprec, ea, c.s, tcls);
    };
    const bool has_int = L.int1 > L.int0 && (L.nsend + L.nrecv) > 0;  // no halo: one launch
    if (has_int) AMGT_TRY(run(L.int0, L.int1));
    if (L.nsend + L.nrecv) AMGT_CUDA(cudaStreamWaitEvent(c.s, c.D->done, 0));
    if (has_int) {
        AMGT_TRY(run(0, L.int0));
        AMGT_TRY(run(L.int1, BR));
    } else {
        AMGT_TRY(run(0, BR));
    }
    return AMGT_OK;
}

amgt_status local_spmv(Ctx& c, const amgt_mbsr* M, const void* x, amgt_prec xp, void* y, amgt_prec yp, int mode) {
    ++c.calls;
    return spmv_ex_impl(M, x, xp, y, yp, EpiArgs{mode, nullptr, nullptr, nullptr, c.omega, 0, -1}, c.s, TC_SPMV);
}

void* own(const amgt_dist_level& L, int i) { return (char*)L.xe[i] + L.off * vb(L.vprec); }

}  // namespace

extern "C" {

amgt_status amgt_dist_unique_id(void* id128_host) {
    if (!id128_host) return fail(AMGT_ERR_ARG, "amgt_dist_unique_id: NULL");
    AMGT_TRY(load_nccl());
    nccl_uid u;
    AMGT_NCCL(g_nccl.GetUniqueId(&u));
    std::copy(u.internal, u.internal + 128, (char*)id128_host);
    return AMGT_OK;
}

amgt_status amgt_dist_create(const void* id128_host, int rank, int size, amgt_dist** Dout) {
    if (!id128_host || !Dout || size < 1 || rank < 0 || rank >= size) return fail(AMGT_ERR_ARG, "amgt_dist_create: bad argument");
    AMGT_TRY(load_nccl());
    nccl_uid u;
    std::copy((const char*)id128_host, (const char*)id128_host + 128, u.internal);
    amgt_dist* D = new amgt_dist();
    D->rank = rank;
    D->size = size;
    nccl_result r = g_nccl.CommInitRank(&D->comm, size, u, rank);
    if (r != 0) {
        delete D;
        return fail(AMGT_ERR_NCCL, "ncclCommInitRank: %s", g_nccl.GetErrorString ? g_nccl.GetErrorString(r) : "?");
    }
    AMGT_CUDA(cudaStreamCreateWithFlags(&D->cs, cudaStreamNonBlocking));
    AMGT_CUDA(cudaEventCreateWithFlags(&D->ready, cudaEventDisableTiming));
    AMGT_CUDA(cudaEventCreateWithFlags(&D->done, cudaEventDisableTiming));
    *Dout = D;
    return AMGT_OK;
}

amgt_status amgt_dist_destroy(amgt_dist* D) {
    if (!D) return AMGT_OK;
    if (D->cs) cudaStreamSynchronize(D->cs);
    if (D->comm && g_nccl.CommDestroy) g_nccl.CommDestroy(D->comm);
    if (D->ready) cudaEventDestroy(D->ready);
    if (D->done) cudaEventDestroy(D->done);
    if (D->cs) cudaStreamDestroy(D->cs);
    delete D;
    return AMGT_OK;
}

amgt_status amgt_dist_allreduce_sum(amgt_dist* D, double* buf, int64_t count, void* stream) {
    if (!D || (!buf && count)) return fail(AMGT_ERR_ARG, "amgt_dist_allreduce_sum: bad argument");
    AMGT_NCCL(g_nccl.AllReduce(buf, buf, (size_t)count, NCCL_FLOAT64, NCCL_SUM, D->comm, (cudaStream_t)stream));
    return AMGT_OK;
}

amgt_status amgt_dist_vcycle(amgt_dist* D, int nlev, const amgt_dist_level* Ls, const amgt_dist_coarse* C, double omega,
                             int nu1, int nu2, const double* b, double* x, int ncycles, double* res_host,
                             int64_t* calls_host, void* stream) {
    if (!D || nlev < 1 || !Ls || !C || !b || !x || ncycles < 0) return fail(AMGT_ERR_ARG, "amgt_dist_vcycle: bad argument");
    for (int k = 0; k < nlev; ++k)
        if (!Ls[k].A || !Ls[k].xe[0] || !Ls[k].xe[1] || !Ls[k].r || (k + 1 < nlev && (!Ls[k].P || !Ls[k].R)))
            return fail(AMGT_ERR_ARG, "amgt_dist_vcycle: incomplete level %d", k);
    cudaStream_t s = (cudaStream_t)stream;
    // SpMV kernels with programmatic dependent launch, as in amgt_vcycle: a launch that follows
    // an event wait (the halo) or a non-PDL kernel gets an ordinary full dependency
    PdlScope pdl;
    Ctx c{D, s, omega};
    const int M = nlev - 1;
    constexpr int JAC = 1, RES = 2, ACC = 3;
    Alloc a{nullptr, s};
    Scratch<double> norms, part;
    AMGT_TRY(norms.init(a, ncycles + 1));
    AMGT_TRY(part.init(a, NB));
    std::vector<int> cur(nlev, 0);
    const amgt_dist_level& L0 = Ls[0];
    AMGT_CUDA(cudaMemcpyAsync(own(L0, 0), x, L0.m * sizeof(double), cudaMemcpyDeviceToDevice, s));
    auto norm_of_r = [&](int slot) -> amgt_status {  // ||r_1||^2 into norms[slot] (all ranks)
        k_sq_partial<<<NB, 256, 0, s>>>(4 * L0.A->blc_row, (const double*)L0.r, part.p);
        AMGT_LAUNCHED();
        k_sq_final<<<1, 32, 0, s>>>(part.p, norms.p + slot);
        AMGT_LAUNCHED();
        if (D->size > 1)
            AMGT_NCCL(g_nccl.AllReduce(norms.p + slot, norms.p + slot, 1, NCCL_FLOAT64, NCCL_SUM, D->comm, s));
        return AMGT_OK;
    };
    auto resnorm = [&](int slot) -> amgt_status {
        AMGT_TRY(dspmv(c, L0, 0, L0.xe[cur[0]], L0.r, RES, b, nullptr));
        return norm_of_r(slot);
    };
    // The residual after cycle c (L308) is what cycle c+1's first level-1 pre-smoothing sweep
    // computes anyway (same x, same arithmetic): that sweep also writes r (AMGT_EPI_JACOBI_RES)
    // and the norm is taken from it, as in the single-GPU amgt_vcycle; only the last cycle's
    // residual needs its own pass over A_1.
    const bool fused = nu1 >= 1 && M > 0;
    auto smooth = [&](int k, const void* bk, int sweeps, int norm_slot = -1) -> amgt_status {
        const amgt_dist_level& L = Ls[k];
        for (int i = 0; i < sweeps; ++i) {
            const int src = cur[k], dst = 1 - src;
            if (i == 0 && norm_slot >= 0) {
                AMGT_TRY(dspmv(c, L, k, L.xe[src], own(L, dst), AMGT_EPI_JACOBI_RES, bk, own(L, src), L.r));
                AMGT_TRY(norm_of_r(norm_slot));
            } else {
                AMGT_TRY(dspmv(c, L, k, L.xe[src], own(L, dst), JAC, bk, own(L, src)));
            }
            cur[k] = dst;
        }
        return AMGT_OK;
    };
    if (!fused || ncycles == 0) AMGT_TRY(resnorm(0));
    for (int cyc = 1; cyc <= ncycles; ++cyc) {
        for (int k = 0; k < M; ++k) {  // Alg. 2 lines 1-5
            const amgt_dist_level& L = Ls[k];
            const void* bk = k == 0 ? (const void*)b : L.b;
            int sweeps = nu1;
            if (k > 0) {
                const int64_t nk = 4 * L.A->blc_row;
                if (nu1 >= 1) {  // zero initial guess: the first sweep is w D^-1 b (no SpMV, no halo)
                    const unsigned g = (unsigned)ceil_div(nk, 256);
                    if (L.vprec == AMGT_FP64)
                        k_zero_sweep<double><<<g, 256, 0, s>>>(nk, (const double*)bk, (const double*)L.dinv, omega,
                                                                (double*)own(L, 1));
                    else
                        k_zero_sweep<float><<<g, 256, 0, s>>>(nk, (const float*)bk, (const float*)L.dinv, (float)omega,
                                                               (float*)own(L, 1));
                    AMGT_LAUNCHED();
                    ++c.calls;  // Alg. 2's sweep (its SpMV is A 0 = 0)
                    cur[k] = 1;
                    sweeps = nu1 - 1;
                } else {
                    cur[k] = 0;
                    AMGT_CUDA(cudaMemsetAsync(own(L, 0), 0, nk * vb(L.vprec), s));
                }
            }
            AMGT_TRY(smooth(k, bk, sweeps, (k == 0 && fused) ? cyc - 1 : -1));
            AMGT_TRY(dspmv(c, L, k, L.xe[cur[k]], L.r, RES, bk, nullptr));
            AMGT_TRY(local_spmv(c, L.R, L.r, L.vprec, Ls[k + 1].b, Ls[k + 1].vprec, 0));
        }
        {  // line 6: all-gather b_M (variable counts, P2P), dense solve on every rank
            const amgt_dist_level& L = Ls[M];
            const size_t e = vb(L.vprec);
            AMGT_CUDA(cudaMemcpyAsync((char*)C->bfull + C->displs[D->rank] * e, L.b, L.m * e, cudaMemcpyDeviceToDevice, s));
            if (D->size > 1) {
                AMGT_NCCL(g_nccl.GroupStart());
                for (int q = 0; q < D->size; ++q) {
                    if (q == D->rank) continue;
                    AMGT_NCCL(g_nccl.Send(L.b, (size_t)L.m, nccl_type(L.vprec), q, D->comm, s));
                    AMGT_NCCL(g_nccl.Recv((char*)C->bfull + C->displs[q] * e, (size_t)C->counts[q], nccl_type(L.vprec), q,
                                          D->comm, s));
                }
                AMGT_NCCL(g_nccl.GroupEnd());
            }
            if (L.vprec == AMGT_FP64)
                k_dense_apply<double><<<(unsigned)ceil_div(C->n * 32, 256), 256, 0, s>>>(C->n, C->Ainv, (const double*)C->bfull,
                                                                                        (double*)C->xfull);
            else
                k_dense_apply<float><<<(unsigned)ceil_div(C->n * 32, 256), 256, 0, s>>>(C->n, C->Ainv, (const float*)C->bfull,
                                                                                       (float*)C->xfull);
            AMGT_LAUNCHED();
            cur[M] = 0;
            AMGT_CUDA(cudaMemsetAsync(own(L, 0), 0, 4 * L.A->blc_row * e, s));
            AMGT_CUDA(cudaMemcpyAsync(own(L, 0), (char*)C->xfull + C->displs[D->rank] * e, L.m * e, cudaMemcpyDeviceToDevice, s));
        }
        for (int k = M - 1; k >= 0; --k) {  // lines 7-11
            const amgt_dist_level& L = Ls[k];
            const amgt_dist_level& N = Ls[k + 1];
            const void* bk = k == 0 ? (const void*)b : L.b;
            AMGT_TRY(local_spmv(c, L.P, own(N, cur[k + 1]), N.vprec, own(L, cur[k]), L.vprec, ACC));
            AMGT_TRY(smooth(k, bk, nu2));
        }
        if (!fused || cyc == ncycles) AMGT_TRY(resnorm(cyc));
    }
    AMGT_CUDA(cudaMemcpyAsync(x, own(L0, cur[0]), L0.m * sizeof(double), cudaMemcpyDeviceToDevice, s));
    std::vector<double> hn(ncycles + 1);
    AMGT_CUDA(cudaMemcpyAsync(hn.data(), norms.p, (ncycles + 1) * sizeof(double), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaStreamSynchronize(s));
    if (res_host)
        for (int i = 0; i <= ncycles; ++i) res_host[i] = std::sqrt(hn[i]);
    if (calls_host) *calls_host = c.calls;
    return AMGT_OK;
}

}  // extern "C"
