// convert.cu — CSR <-> mBSR conversion, per-level precision cast, tile transpose.
//
// CSR2MBSR (L234, L262; Fig. 6 step 4) on B200: a 4-lane group owns one block row and
// lane r owns CSR row 4I+r.  The group walks the four sorted column lists in lockstep
// (a 4-way merge on tile column col>>2, two shuffles per step); each lane writes its own
// tile row (one 16 B / 32 B vector store) and the group ORs its four nibbles into the
// 16-bit bitmap (bit 4r+c, R1).  Eight block rows per warp, all reads of a lane
// sequential in its row.  Two passes (count, fill) around a device prefix sum; one
// host sync to size the tile arrays.
#include <climits>
#include <cstdlib>

#include "common.cuh"

namespace amgt {

static __device__ __forceinline__ void store_row(double* p, const double (&v)[4]) {
    reinterpret_cast<double2*>(p)[0] = make_double2(v[0], v[1]);
    reinterpret_cast<double2*>(p)[1] = make_double2(v[2], v[3]);
}
static __device__ __forceinline__ void store_row(float* p, const double (&v)[4]) {
    *reinterpret_cast<float4*>(p) =
        make_float4(__double2float_rn(v[0]), __double2float_rn(v[1]), __double2float_rn(v[2]), __double2float_rn(v[3]));
}
static __device__ __forceinline__ void store_row(__half* p, const double (&v)[4]) {
    __half2 a = __halves2half2(__double2half(v[0]), __double2half(v[1]));
    __half2 b = __halves2half2(__double2half(v[2]), __double2half(v[3]));
    uint2 u;
    u.x = *reinterpret_cast<uint32_t*>(&a);
    u.y = *reinterpret_cast<uint32_t*>(&b);
    *reinterpret_cast<uint2*>(p) = u;
}

template <typename T> __device__ __forceinline__ bool overflows(double v) { return false; }
template <> __device__ __forceinline__ bool overflows<__half>(double v) {
    return fabs(v) > 65504.0 && fabs(v) < INFINITY && __hisinf(__double2half(v));
}

// Block rows with more than LONG_CONV CSR entries (power-law rows) are handled by one CTA
// each (k_csr2mbsr_long): the 4-lane lockstep merge would serialise them.
constexpr int64_t LONG_CONV = 4096;

// One CTA per long block row: the row's tile columns are marked in a bitmap over the tile
// columns (shared memory when it fits, else a per-CTA global slice); popcounts give the
// count, an exclusive scan of word popcounts gives every tile's position (ascending J by
// construction).  Entries are placed in parallel (distinct value slots); bitmap bits are
// ORed with 32-bit atomics on the 16-bit map array.  Validation as in the group kernel.
template <bool FILL, typename T>
__global__ void __launch_bounds__(512) k_csr2mbsr_long(int64_t m, int64_t n, int64_t coff, const int64_t* __restrict__ rp,
                                                       const int32_t* __restrict__ ci, const double* __restrict__ v,
                                                       const int32_t* __restrict__ longl,
                                                       const unsigned long long* __restrict__ nlong, int64_t W,
                                                       uint32_t* __restrict__ gws, int64_t* __restrict__ cnt,
                                                       const int64_t* __restrict__ bptr, int32_t* __restrict__ bidx,
                                                       uint16_t* __restrict__ bmap, T* __restrict__ bval,
                                                       uint32_t* __restrict__ flag) {
    extern __shared__ __align__(16) uint32_t smw[];
    __shared__ long long sh_sum[17];
    uint32_t* bm = gws ? gws + (int64_t)blockIdx.x * 2 * W : smw;
    uint32_t* pre = bm + W;
    const int tid = threadIdx.x, nt = blockDim.x, lane = tid & 31, w = tid >> 5, nw = nt >> 5;
    const int64_t nl = (int64_t)*nlong;
    uint32_t bad = 0, range = 0;
    for (int64_t li = blockIdx.x; li < nl; li += gridDim.x) {
        const int64_t I = longl[li];
        for (int64_t i = tid; i < W; i += nt) bm[i] = 0;
        __syncthreads();
        for (int r = 0; r < 4 && 4 * I + r < m; ++r) {
            const int64_t a = rp[4 * I + r], b = rp[4 * I + r + 1];
            for (int64_t p = a + tid; p < b; p += nt) {
                const int64_t col = ci[p] - coff;
                if (!FILL && (col < 0 || col >= n || (p > a && ci[p] <= ci[p - 1]))) bad = 1;
                if (col >= 0 && col < n) atomicOr(bm + (col >> 7), 1u << ((col >> 2) & 31));
            }
        }
        __syncthreads();
        const int64_t per = (W + nt - 1) / nt;
        const int64_t w0 = min(W, per * (int64_t)tid), w1 = min(W, w0 + per);
        long long sloc = 0;
        for (int64_t i = w0; i < w1; ++i) sloc += __popc(bm[i]);
        long long incl = sloc;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const long long y = __shfl_up_sync(0xffffffffu, incl, d);
            if (lane >= d) incl += y;
        }
        if (lane == 31) sh_sum[w] = incl;
        __syncthreads();
        if (tid == 0) {
            long long acc = 0;
            for (int k = 0; k < nw; ++k) { const long long x = sh_sum[k]; sh_sum[k] = acc; acc += x; }
            sh_sum[nw] = acc;
        }
        __syncthreads();
        if (!FILL) {
            if (tid == 0) cnt[I] = sh_sum[nw];
            __syncthreads();
            continue;
        }
        const int64_t t0 = bptr[I];
        long long run = sh_sum[w] + incl - sloc;
        for (int64_t i = w0; i < w1; ++i) {  // tile columns in ascending order
            pre[i] = (uint32_t)run;
            uint32_t bits = bm[i];
            while (bits) {
                const int b = __ffs(bits) - 1;
                bits &= bits - 1;
                bidx[t0 + run] = (int32_t)(32 * i + b);
                ++run;
            }
        }
        const int64_t ntile = sh_sum[nw];
        for (int64_t e2 = tid; e2 < 16 * ntile; e2 += nt) bval[16 * t0 + e2] = from_f64<T>(0.0);
        for (int64_t tt = tid; tt < ntile; tt += nt) bmap[t0 + tt] = 0;
        __syncthreads();
        for (int r = 0; r < 4 && 4 * I + r < m; ++r) {
            const int64_t a = rp[4 * I + r], b = rp[4 * I + r + 1];
            for (int64_t p = a + tid; p < b; p += nt) {
                const int64_t col = ci[p] - coff;
                const int64_t J = col >> 2;
                const int64_t q = t0 + pre[J >> 5] + __popc(bm[J >> 5] & ((1u << (J & 31)) - 1u));
                const int bit = 4 * r + (int)(col & 3);
                const double x = v[p];
                bval[16 * q + bit] = from_f64<T>(x);
                if (overflows<T>(x)) range = 1;
                atomicOr(reinterpret_cast<unsigned int*>(bmap) + (q >> 1), (1u << bit) << (16 * (q & 1)));
            }
        }
        __syncthreads();
    }
    if (bad) atomicOr(flag, FLAG_FORMAT);
    if (range) atomicOr(flag, FLAG_RANGE);
}

// FILL = false: count tiles per block row into cnt[I] and validate the CSR.
// FILL = true : write blc_idx / blc_map / blc_val at offsets bptr[I].
// Fill pass: the warp's 32 CSR rows are one contiguous range of the column / value arrays; when it
// holds at most CONV_STAGE entries the warp first copies it to shared memory with coalesced loads,
// so the lanes' per-row merges read shared memory instead of issuing dependent scattered global
// loads (config-3 A_1 fill: 8.3 -> 7.2 ms of cold kernel time).  The count pass reads only the
// columns and keeps the unstaged loads and the higher occupancy.
// AMGT_CONV_STAGE=0: the fill pass without the shared-memory staging (measurement knob)
static bool conv_stage() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("AMGT_CONV_STAGE");
        v = (e && e[0] == '0') ? 0 : 1;
    }
    return v == 1;
}
constexpr int CONV_WARPS = 4;     // 128-thread CTAs
constexpr int CONV_STAGE = 896;  // entries per warp (27-point: 32 rows x 27 = 864; 5 CTAs per SM)
template <bool FILL>
constexpr int conv_smem_bytes() { return FILL ? CONV_WARPS * CONV_STAGE * 12 : 0; }

template <bool FILL, typename T>
__global__ void __launch_bounds__(128) k_csr2mbsr(int64_t m, int64_t n, int64_t nnz, int64_t BR, int64_t coff,
                                                  const int64_t* __restrict__ rp, const int32_t* __restrict__ ci,
                                                  const double* __restrict__ v, int64_t* __restrict__ cnt,
                                                  const int64_t* __restrict__ bptr, int32_t* __restrict__ bidx,
                                                  uint16_t* __restrict__ bmap, T* __restrict__ bval,
                                                  uint32_t* __restrict__ flag, int32_t* __restrict__ longl,
                                                  unsigned long long* __restrict__ nlong, bool stage_ok) {
    extern __shared__ __align__(16) unsigned char conv_sm[];
    const int lane = threadIdx.x & 31, g = lane >> 2, r = lane & 3, wib = threadIdx.x >> 5;
    const int64_t W = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t I = W * 8 + g;
    if (W * 8 >= BR) return;  // whole warp idle
    const bool active = I < BR;
    const int64_t row = 4 * I + r;
    int64_t p = 0, e = 0;
    uint32_t bad = 0, range = 0;
    if (active && row < m) {
        p = rp[row];
        e = rp[row + 1];
        if (!FILL) {
            if (p > e || p < 0 || e > nnz) { bad = 1; e = p; }
            if (row == 0 && p != 0) bad = 1;
            if (row == m - 1 && e != nnz) bad = 1;
        }
    }
    {  // block rows with many entries go to the CTA-per-row kernel (k_csr2mbsr_long)
        int64_t bn = e - p;
        bn += __shfl_xor_sync(0xffffffffu, bn, 1);
        bn += __shfl_xor_sync(0xffffffffu, bn, 2);
        if (bn > LONG_CONV) {
            if (!FILL && r == 0) longl[atomicAdd(nlong, 1ull)] = (int32_t)I;
            e = p;
        }
    }
    // stage the warp's entries [wb, we) (rows 32 W .. 32 W + 31); every lane's [p, e) must lie
    // inside (true for a valid CSR; a malformed one is read from global memory and flagged)
    double* sv = reinterpret_cast<double*>(conv_sm) + (int64_t)wib * CONV_STAGE;
    int32_t* sci = reinterpret_cast<int32_t*>(conv_sm + (size_t)CONV_WARPS * CONV_STAGE * 8) + (int64_t)wib * CONV_STAGE;
    int64_t wb = 0, we = 0;
    if (FILL && lane == 0) {
        wb = rp[min(32 * W, m)];
        we = rp[min(32 * W + 32, m)];
    }
    wb = __shfl_sync(0xffffffffu, wb, 0);
    we = __shfl_sync(0xffffffffu, we, 0);
    const bool staged = FILL && stage_ok && __all_sync(0xffffffffu, we - wb >= 0 && we - wb <= CONV_STAGE && wb >= 0 && we <= nnz &&
                                                             (p >= e || (p >= wb && e <= we)));
    if (staged) {
        const int64_t ne = we - wb;
        for (int64_t q = lane; q < ne; q += 32) sci[q] = __ldg(ci + wb + q);
        for (int64_t q = lane; q < ne; q += 32) sv[q] = __ldg(v + wb + q);
        __syncwarp();
    }
    auto ld_ci = [&](int64_t q) { return staged ? sci[q - wb] : __ldg(ci + q); };
    auto ld_v = [&](int64_t q) { return staged ? sv[q - wb] : __ldg(v + q); };
    int64_t t = (FILL && active) ? bptr[I] : 0;
    int64_t c = 0;
    int32_t prev = -1;
    // the lane's next entry's column, loaded one entry ahead (the merge chain then waits for
    // one shared-memory / global load per entry, not two)
    int32_t col = (p < e) ? (int32_t)(ld_ci(p) - coff) : 0;
    for (;;) {
        const int32_t J = (p < e) ? (col >> 2) : INT_MAX;
        int32_t Jm = min(J, __shfl_xor_sync(0xffffffffu, J, 1));
        Jm = min(Jm, __shfl_xor_sync(0xffffffffu, Jm, 2));
        if (!__any_sync(0xffffffffu, Jm != INT_MAX)) break;
        double rv[4] = {0.0, 0.0, 0.0, 0.0};
        uint32_t nib = 0;
        if (Jm != INT_MAX) {
            while (p < e && (col >> 2) == Jm) {
                const int64_t pc = p++;
                const int32_t ncol = (p < e) ? (int32_t)(ld_ci(p) - coff) : 0;
                if (!FILL) {
                    if (col <= prev || col >= n || col < 0) bad = 1;
                    prev = col;
                } else {
                    const int cc = col & 3;
                    const double x = ld_v(pc);
                    rv[0] = cc == 0 ? x : rv[0];
                    rv[1] = cc == 1 ? x : rv[1];
                    rv[2] = cc == 2 ? x : rv[2];
                    rv[3] = cc == 3 ? x : rv[3];
                    if (overflows<T>(x)) range = 1;
                }
                nib |= 1u << (col & 3);
                col = ncol;
            }
        }
        uint32_t mp = nib << (4 * r);
        mp |= __shfl_xor_sync(0xffffffffu, mp, 1);
        mp |= __shfl_xor_sync(0xffffffffu, mp, 2);
        if (Jm != INT_MAX) {
            if (FILL) {
                if constexpr (sizeof(T) == 8)
                    group_store_tile_f64((double*)(bval + 16 * t), rv, r, 0xFu << (lane & ~3), lane & ~3);
                else
                    store_row(bval + 16 * t + 4 * r, rv);
                if (r == 0) {
                    bidx[t] = Jm;
                    bmap[t] = (uint16_t)mp;
                }
            }
            ++c;
            ++t;
        }
    }
    if (!FILL && active && r == 0) cnt[I] = c;  // long rows: overwritten by k_csr2mbsr_long
    if (bad) atomicOr(flag, FLAG_FORMAT);
    if (range) atomicOr(flag, FLAG_RANGE);
}

// Row nnz from bitmaps: lane r counts the set bits of nibble r over the block row.
__global__ void __launch_bounds__(256) k_mbsr2csr_count(int64_t m, int64_t BR, const int64_t* __restrict__ bptr,
                                                        const uint16_t* __restrict__ bmap, int64_t* __restrict__ rn) {
    const int64_t gt = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t I = gt >> 2;
    const int r = (int)(gt & 3);
    if (I >= BR) return;
    const int64_t row = 4 * I + r;
    if (row >= m) return;
    int64_t c = 0;
    for (int64_t t = bptr[I]; t < bptr[I + 1]; ++t) c += __popc((bmap[t] >> (4 * r)) & 0xFu);
    rn[row] = c;
}

template <typename T>
__global__ void __launch_bounds__(256) k_mbsr2csr_fill(int64_t m, int64_t BR, const int64_t* __restrict__ bptr,
                                                       const int32_t* __restrict__ bidx,
                                                       const uint16_t* __restrict__ bmap, const T* __restrict__ bval,
                                                       const int64_t* __restrict__ rp, int32_t* __restrict__ ci,
                                                       double* __restrict__ v) {
    const int64_t gt = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t I = gt >> 2;
    const int r = (int)(gt & 3);
    if (I >= BR) return;
    const int64_t row = 4 * I + r;
    if (row >= m) return;
    int64_t d = rp[row];
    for (int64_t t = bptr[I]; t < bptr[I + 1]; ++t) {
        const uint32_t nib = (bmap[t] >> (4 * r)) & 0xFu;
        if (!nib) continue;
        const int32_t J = bidx[t];
#pragma unroll
        for (int c = 0; c < 4; ++c)
            if (nib & (1u << c)) {
                ci[d] = 4 * J + c;
                v[d] = to_f64(bval[16 * t + 4 * r + c]);
                ++d;
            }
    }
}

__global__ void k_popc_sum(int64_t T, const uint16_t* __restrict__ bmap, unsigned long long* __restrict__ out) {
    int64_t s = 0;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < T; t += (int64_t)gridDim.x * blockDim.x)
        s += __popc(bmap[t]);
    for (int d = 16; d; d >>= 1) s += __shfl_xor_sync(0xffffffffu, s, d);
    if ((threadIdx.x & 31) == 0 && s) atomicAdd(out, (unsigned long long)s);
}

template <typename Ti, typename To>
__global__ void k_cast(int64_t n, const Ti* __restrict__ in, To* __restrict__ out, uint32_t* __restrict__ flag) {
    uint32_t bad = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const double x = to_f64(in[i]);
        To y;
        if constexpr (sizeof(Ti) == 4 && sizeof(To) == 2) {
            y = __float2half_rn((float)x);  // FP32 -> FP16 (single rounding from FP32)
        } else {
            y = from_f64<To>(x);  // direct from FP64 (R18)
        }
        if (overflows<To>(x)) bad = 1;
        out[i] = y;
    }
    if (bad) atomicOr(flag, FLAG_RANGE);
}

// ---- transpose: (1) count per destination row, (2) scan, (3) scatter (idx, perm),
// (4) per-row sort by column, (5) gather transposed tiles.
__global__ void k_tr_count(int64_t T, const int32_t* __restrict__ bidx, unsigned long long* __restrict__ cnt) {
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < T; t += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(cnt + bidx[t], 1ull);
}

__global__ void k_tr_scatter(int64_t BR, const int64_t* __restrict__ bptr, const int32_t* __restrict__ bidx,
                             const int64_t* __restrict__ optr, unsigned long long* __restrict__ fill,
                             int32_t* __restrict__ oidx, int64_t* __restrict__ perm) {
    for (int64_t I = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; I < BR; I += (int64_t)gridDim.x * blockDim.x)
        for (int64_t t = bptr[I]; t < bptr[I + 1]; ++t) {
            const int32_t J = bidx[t];
            const int64_t d = optr[J] + (int64_t)atomicAdd(fill + J, 1ull);
            oidx[d] = (int32_t)I;
            perm[d] = t;
        }
}

__global__ void k_tr_sort(int64_t BRo, const int64_t* __restrict__ optr, int32_t* __restrict__ oidx,
                          int64_t* __restrict__ perm) {
    for (int64_t J = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; J < BRo; J += (int64_t)gridDim.x * blockDim.x) {
        const int64_t a = optr[J], b = optr[J + 1];
        for (int64_t i = a + 1; i < b; ++i) {  // insertion sort (rows of P^T are short)
            const int32_t k = oidx[i];
            const int64_t pv = perm[i];
            int64_t j = i - 1;
            while (j >= a && oidx[j] > k) {
                oidx[j + 1] = oidx[j];
                perm[j + 1] = perm[j];
                --j;
            }
            oidx[j + 1] = k;
            perm[j + 1] = pv;
        }
    }
}

// Output tile d = (input tile perm[d])^T.  One 4-lane group per tile: lane q gathers column q
// of the input tile (its four rows' q-th entries: each load instruction of the group reads
// the 32-B row r) and writes it as row q of the output tile (the group's stores cover the
// output tile contiguously); the bitmap is transposed by lane 0.
template <typename T>
__global__ void k_tr_gather(int64_t T_, const int64_t* __restrict__ perm, const uint16_t* __restrict__ bmap,
                            const T* __restrict__ bval, uint16_t* __restrict__ omap, T* __restrict__ oval) {
    const int q = threadIdx.x & 3;
    for (int64_t d = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 2; d < T_;
         d += ((int64_t)gridDim.x * blockDim.x) >> 2) {
        const int64_t s = perm[d];
        T v[4];
#pragma unroll
        for (int r = 0; r < 4; ++r) v[r] = bval[16 * s + 4 * r + q];
#pragma unroll
        for (int r = 0; r < 4; ++r) oval[16 * d + 4 * q + r] = v[r];
        if (q == 0) {
            const uint32_t mp = bmap[s];
            uint32_t tm = 0;
#pragma unroll
            for (int r = 0; r < 4; ++r)
#pragma unroll
                for (int c = 0; c < 4; ++c)
                    if (mp & (1u << (4 * r + c))) tm |= 1u << (4 * c + r);
            omap[d] = (uint16_t)tm;
        }
    }
}

static unsigned grid_for(int64_t work, int threads) {
    int64_t b = ceil_div(work, threads);
    int64_t cap = (int64_t)num_sms() * 16;
    if (b > cap) b = cap;
    if (b < 1) b = 1;
    return (unsigned)b;
}

amgt_status mbsr_alloc(amgt_mbsr* M, int64_t m, int64_t n, int64_t T, amgt_prec prec, Alloc& a, bool structure,
                       bool values, int64_t* existing_ptr) {
    M->m = m;
    M->n = n;
    M->blc_row = ceil_div(m, 4);
    M->blc_col = ceil_div(n, 4);
    M->blc_num = T;
    M->prec = prec;
    M->aux = nullptr;
    M->own = 0;
    M->row_max = 0;
    if (structure) {
        M->blc_ptr = existing_ptr ? existing_ptr : (int64_t*)a.get((M->blc_row + 1) * sizeof(int64_t));
        M->blc_idx = (int32_t*)a.get(T * sizeof(int32_t));
        M->blc_map = (uint16_t*)a.get(((T + 1) & ~int64_t(1)) * sizeof(uint16_t));  // even count: u32 atomics
        M->own |= 1u;
        if (!M->blc_ptr || !M->blc_idx || !M->blc_map) return fail(AMGT_ERR_ALLOC, "mBSR structure allocation failed");
    }
    if (values) {
        M->blc_val = a.get(16 * T * prec_bytes(prec));
        M->own |= 2u;
        if (!M->blc_val) return fail(AMGT_ERR_ALLOC, "mBSR value allocation failed (%lld tiles)", (long long)T);
    }
    return AMGT_OK;
}

void spmv_plan_free(void* aux, Alloc& a);

amgt_status mbsr_release(amgt_mbsr* M, Alloc& a) {
    if (!M) return AMGT_OK;
    if (M->aux) spmv_plan_free(M->aux, a);
    if (M->own & 1u) {
        spgemm_plan_drop(M->blc_idx, a.s);
        a.put(M->blc_ptr, (M->blc_row + 1) * sizeof(int64_t));
        a.put(M->blc_idx, M->blc_num * sizeof(int32_t));
        a.put(M->blc_map, ((M->blc_num + 1) & ~int64_t(1)) * sizeof(uint16_t));
    }
    if (M->own & 2u) a.put(M->blc_val, 16 * M->blc_num * prec_bytes(M->prec));
    *M = amgt_mbsr{};
    return AMGT_OK;
}

static amgt_status read_flag(uint32_t* dflag, cudaStream_t s, uint32_t* out) {
    AMGT_CUDA(cudaMemcpyAsync(out, dflag, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaStreamSynchronize(s));
    return AMGT_OK;
}

amgt_status csr_to_mbsr_impl(int64_t m, int64_t n, int64_t nnz, const int64_t* rp, const int32_t* ci,
                             const double* v, amgt_prec prec, amgt_mbsr* out, Alloc& a, int64_t coff) {
    cudaStream_t s = a.s;
    const int64_t BR = ceil_div(m, 4);
    Scratch<int64_t> cnt;
    Scratch<uint32_t> flag;
    Scratch<int32_t> longl;
    Scratch<unsigned long long> nlong;
    AMGT_TRY(cnt.init(a, BR + 1));
    AMGT_TRY(flag.init(a, 1));
    AMGT_TRY(longl.init(a, BR + 1));
    AMGT_TRY(nlong.init(a, 1));
    AMGT_CUDA(cudaMemsetAsync(flag.p, 0, sizeof(uint32_t), s));
    AMGT_CUDA(cudaMemsetAsync(nlong.p, 0, sizeof(unsigned long long), s));
    // long-row kernel resources: bitmap + word prefix over the tile columns
    const int64_t W = ceil_div(ceil_div(n, 4), 32);
    const size_t lsm = (size_t)W * 2 * sizeof(uint32_t);
    const bool lsmem = lsm <= 160 * 1024;
    const unsigned LG = lsmem ? (unsigned)num_sms() : 16u;
    Scratch<uint32_t> lws;
    if (!lsmem) AMGT_TRY(lws.init(a, (size_t)LG * 2 * W));
    auto launch_long = [&](auto kern, int64_t* cntp, const int64_t* bp, int32_t* bi, uint16_t* bmp, auto* bv) -> amgt_status {
        if (lsmem) AMGT_CUDA(dyn_smem(kern, lsm));
        kern<<<LG, 512, lsmem ? lsm : 0, s>>>(m, n, coff, rp, ci, v, longl.p, nlong.p, W, lsmem ? nullptr : lws.p, cntp,
                                               bp, bi, bmp, bv, flag.p);
        AMGT_LAUNCHED();
        return AMGT_OK;
    };
    amgt_mbsr M{};
    const double bytes_in = nnz * 12.0 + (m + 1) * 8.0;
    const unsigned blocks = (unsigned)ceil_div(ceil_div(BR, 8) * 32, 32 * CONV_WARPS);
    // > 48 KB of dynamic shared memory for the staged fill
    AMGT_CUDA(dyn_smem(k_csr2mbsr<true, double>, conv_smem_bytes<true>()));
    AMGT_CUDA(dyn_smem(k_csr2mbsr<true, float>, conv_smem_bytes<true>()));
    AMGT_CUDA(dyn_smem(k_csr2mbsr<true, __half>, conv_smem_bytes<true>()));
    {
        TimerScope ts(TC_CSR2MBSR, bytes_in, s);
        if (BR > 0) {
            k_csr2mbsr<false, double><<<blocks, 32 * CONV_WARPS, conv_smem_bytes<false>(), s>>>(m, n, nnz, BR, coff, rp, ci, v, cnt.p, nullptr, nullptr,
                                                             nullptr, nullptr, flag.p, longl.p, nlong.p, false);
            AMGT_LAUNCHED();
            AMGT_TRY(launch_long(k_csr2mbsr_long<false, double>, cnt.p, nullptr, nullptr, nullptr, (double*)nullptr));
        }
    }
    // blc_ptr lives in the output; scan the counts into it.
    M.blc_ptr = (int64_t*)a.get((BR + 1) * sizeof(int64_t));
    if (!M.blc_ptr) return fail(AMGT_ERR_ALLOC, "blc_ptr allocation failed");
    Scratch<unsigned long long> rmax;  // longest block row (lets the SpMV analysis skip its sync)
    AMGT_TRY(rmax.init(a, 1));
    AMGT_CUDA(cudaMemsetAsync(rmax.p, 0, sizeof(unsigned long long), s));
    AMGT_TRY(scan_exclusive(cnt.p, M.blc_ptr, BR, a, s, rmax.p));
    int64_t hT[1] = {0};
    uint32_t hflag = 0;
    unsigned long long hmax = 0;
    if (int64_t* pin = pinned_slots()) {  // pinned read-back (pageable D2H copies stage through the driver)
        int64_t* pc = pin + PIN_CONV;
        pc[1] = 0;
        AMGT_CUDA(cudaMemcpyAsync(pc, M.blc_ptr + BR, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaMemcpyAsync(pc + 1, flag.p, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaMemcpyAsync(pc + 2, rmax.p, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaStreamSynchronize(s));
        hT[0] = pc[0];
        hflag = (uint32_t)pc[1];
        hmax = (unsigned long long)pc[2];
    } else {
        AMGT_CUDA(cudaMemcpyAsync(hT, M.blc_ptr + BR, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaMemcpyAsync(&hflag, flag.p, sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaMemcpyAsync(&hmax, rmax.p, sizeof(hmax), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaStreamSynchronize(s));
    }
    if (hflag & FLAG_FORMAT) {
        a.put(M.blc_ptr, (BR + 1) * sizeof(int64_t));
        return fail(AMGT_ERR_FORMAT, "CSR input: row_ptr not monotone from 0 to nnz, or columns unsorted/duplicate/out of range");
    }
    const int64_t T = hT[0];
    amgt_status st = mbsr_alloc(&M, m, n, T, prec, a, true, true, M.blc_ptr);
    if (st != AMGT_OK) { mbsr_release(&M, a); return st; }
    M.row_max = (int64_t)hmax;
    {
        const double bytes = bytes_in + T * (16.0 * prec_bytes(prec) + 6.0) + (BR + 1) * 8.0;
        TimerScope ts(TC_CSR2MBSR, bytes, s);
        if (BR > 0) {
            switch (prec) {
                case AMGT_FP64:
                    k_csr2mbsr<true, double><<<blocks, 32 * CONV_WARPS, conv_smem_bytes<true>(), s>>>(m, n, nnz, BR, coff, rp, ci, v, nullptr, M.blc_ptr,
                                                                    M.blc_idx, M.blc_map, (double*)M.blc_val, flag.p,
                                                                    longl.p, nlong.p, conv_stage());
                    AMGT_LAUNCHED();
                    AMGT_TRY(launch_long(k_csr2mbsr_long<true, double>, nullptr, M.blc_ptr, M.blc_idx, M.blc_map,
                                         (double*)M.blc_val));
                    break;
                case AMGT_FP32:
                    k_csr2mbsr<true, float><<<blocks, 32 * CONV_WARPS, conv_smem_bytes<true>(), s>>>(m, n, nnz, BR, coff, rp, ci, v, nullptr, M.blc_ptr,
                                                                   M.blc_idx, M.blc_map, (float*)M.blc_val, flag.p,
                                                                   longl.p, nlong.p, conv_stage());
                    AMGT_LAUNCHED();
                    AMGT_TRY(launch_long(k_csr2mbsr_long<true, float>, nullptr, M.blc_ptr, M.blc_idx, M.blc_map,
                                         (float*)M.blc_val));
                    break;
                default:
                    k_csr2mbsr<true, __half><<<blocks, 32 * CONV_WARPS, conv_smem_bytes<true>(), s>>>(m, n, nnz, BR, coff, rp, ci, v, nullptr, M.blc_ptr,
                                                                    M.blc_idx, M.blc_map, (__half*)M.blc_val, flag.p,
                                                                    longl.p, nlong.p, conv_stage());
                    AMGT_LAUNCHED();
                    AMGT_TRY(launch_long(k_csr2mbsr_long<true, __half>, nullptr, M.blc_ptr, M.blc_idx, M.blc_map,
                                         (__half*)M.blc_val));
            }
        }
    }
    if (prec == AMGT_FP16) {
        AMGT_TRY(read_flag(flag.p, s, &hflag));
        if (hflag & FLAG_RANGE) {
            mbsr_release(&M, a);
            return fail(AMGT_ERR_RANGE, "value exceeds the FP16 range (65504)");
        }
    }
    *out = M;
    return AMGT_OK;
}

template <typename T>
static void launch_m2c_fill(const amgt_mbsr* A, const int64_t* rp, int32_t* ci, double* v, cudaStream_t s) {
    const unsigned blocks = (unsigned)ceil_div(A->blc_row * 4, 256);
    k_mbsr2csr_fill<T><<<blocks, 256, 0, s>>>(A->m, A->blc_row, A->blc_ptr, A->blc_idx, A->blc_map,
                                              (const T*)A->blc_val, rp, ci, v);
}

amgt_status mbsr_to_csr_impl(const amgt_mbsr* A, int64_t* rp, int32_t* ci, double* v, Alloc& a) {
    cudaStream_t s = a.s;
    Scratch<int64_t> rn;
    AMGT_TRY(rn.init(a, A->m + 1));
    const int64_t nnz_est = A->blc_num * 16;
    TimerScope ts(TC_MBSR2CSR, A->blc_num * (16.0 * prec_bytes(A->prec) + 6.0) + (A->m + 1) * 8.0, s);
    if (A->blc_row > 0) {
        k_mbsr2csr_count<<<(unsigned)ceil_div(A->blc_row * 4, 256), 256, 0, s>>>(A->m, A->blc_row, A->blc_ptr,
                                                                                  A->blc_map, rn.p);
        AMGT_LAUNCHED();
    }
    AMGT_TRY(scan_exclusive(rn.p, rp, A->m, a, s));
    (void)nnz_est;
    if (A->blc_row > 0) {
        switch (A->prec) {
            case AMGT_FP64: launch_m2c_fill<double>(A, rp, ci, v, s); break;
            case AMGT_FP32: launch_m2c_fill<float>(A, rp, ci, v, s); break;
            default: launch_m2c_fill<__half>(A, rp, ci, v, s);
        }
        AMGT_LAUNCHED();
    }
    return AMGT_OK;
}

// dflag (optional, device): the FP16 range flag is OR-ed there and NOT read back (no sync);
// the caller checks it after a later synchronisation (amgt_hierarchy_create)
amgt_status cast_impl(const amgt_mbsr* in, amgt_prec to, amgt_mbsr* out, Alloc& a, uint32_t* dflag) {
    cudaStream_t s = a.s;
    if (prec_bytes(to) > prec_bytes(in->prec)) return fail(AMGT_ERR_ARG, "cast must not widen (from %d to %d)", in->prec, to);
    amgt_mbsr M = *in;
    M.own = 0;
    M.aux = nullptr;
    M.prec = to;
    const int64_t n = 16 * in->blc_num;
    M.blc_val = a.get(n * prec_bytes(to));
    if (!M.blc_val) return fail(AMGT_ERR_ALLOC, "cast value allocation failed");
    M.own = 2u;
    Scratch<uint32_t> own_flag;
    uint32_t* fl = dflag;
    if (!fl) {
        AMGT_TRY(own_flag.init(a, 1));
        AMGT_CUDA(cudaMemsetAsync(own_flag.p, 0, sizeof(uint32_t), s));
        fl = own_flag.p;
    }
    {
        TimerScope ts(TC_CAST, (double)n * (prec_bytes(in->prec) + prec_bytes(to)), s);
        if (n > 0) {
            const unsigned g = grid_for(n, 256);
            if (in->prec == to) {
                AMGT_CUDA(cudaMemcpyAsync(M.blc_val, in->blc_val, n * prec_bytes(to), cudaMemcpyDeviceToDevice, s));
            } else if (in->prec == AMGT_FP64 && to == AMGT_FP32) {
                k_cast<double, float><<<g, 256, 0, s>>>(n, (const double*)in->blc_val, (float*)M.blc_val, fl);
                AMGT_LAUNCHED();
            } else if (in->prec == AMGT_FP64 && to == AMGT_FP16) {
                k_cast<double, __half><<<g, 256, 0, s>>>(n, (const double*)in->blc_val, (__half*)M.blc_val, fl);
                AMGT_LAUNCHED();
            } else {
                k_cast<float, __half><<<g, 256, 0, s>>>(n, (const float*)in->blc_val, (__half*)M.blc_val, fl);
                AMGT_LAUNCHED();
            }
        }
    }
    if (to == AMGT_FP16 && in->prec != AMGT_FP16 && !dflag) {
        uint32_t hflag = 0;
        AMGT_TRY(read_flag(fl, s, &hflag));
        if (hflag & FLAG_RANGE) {
            a.put(M.blc_val, n * prec_bytes(to));
            return fail(AMGT_ERR_RANGE, "value exceeds the FP16 range (65504)");
        }
    }
    *out = M;
    return AMGT_OK;
}

template <typename T>
static void launch_tr_gather(const amgt_mbsr* in, const int64_t* perm, amgt_mbsr* o, cudaStream_t s) {
    k_tr_gather<T><<<grid_for(4 * in->blc_num, 256), 256, 0, s>>>(in->blc_num, perm, in->blc_map, (const T*)in->blc_val,
                                                             o->blc_map, (T*)o->blc_val);
}

// dmax (optional, device): atomicMax of the longest block row of the transpose, for callers
// that read it after a later synchronisation (amgt_hierarchy_create)
amgt_status transpose_impl(const amgt_mbsr* in, amgt_mbsr* out, Alloc& a, unsigned long long* dmax) {
    cudaStream_t s = a.s;
    amgt_mbsr M{};
    AMGT_TRY(mbsr_alloc(&M, in->n, in->m, in->blc_num, in->prec, a, true, true, nullptr));
    const int64_t BRo = M.blc_row, T = in->blc_num;
    Scratch<unsigned long long> cnt;
    Scratch<int64_t> perm;
    amgt_status st = cnt.init(a, BRo + 1);
    if (st == AMGT_OK) st = perm.init(a, T);
    if (st != AMGT_OK) { mbsr_release(&M, a); return st; }
    AMGT_CUDA(cudaMemsetAsync(cnt.p, 0, (BRo + 1) * sizeof(unsigned long long), s));
    if (T > 0) {
        k_tr_count<<<grid_for(T, 256), 256, 0, s>>>(T, in->blc_idx, cnt.p);
        AMGT_LAUNCHED();
    }
    AMGT_TRY(scan_exclusive((const int64_t*)cnt.p, M.blc_ptr, BRo, a, s, dmax));
    AMGT_CUDA(cudaMemsetAsync(cnt.p, 0, (BRo + 1) * sizeof(unsigned long long), s));
    if (T > 0) {
        k_tr_scatter<<<grid_for(in->blc_row, 128), 128, 0, s>>>(in->blc_row, in->blc_ptr, in->blc_idx, M.blc_ptr, cnt.p,
                                                                M.blc_idx, perm.p);
        AMGT_LAUNCHED();
        k_tr_sort<<<grid_for(BRo, 128), 128, 0, s>>>(BRo, M.blc_ptr, M.blc_idx, perm.p);
        AMGT_LAUNCHED();
        switch (in->prec) {
            case AMGT_FP64: launch_tr_gather<double>(in, perm.p, &M, s); break;
            case AMGT_FP32: launch_tr_gather<float>(in, perm.p, &M, s); break;
            default: launch_tr_gather<__half>(in, perm.p, &M, s);
        }
        AMGT_LAUNCHED();
    }
    *out = M;
    return AMGT_OK;
}

// ---- distributed-path helpers: tile-column shift and column-range statistics
__global__ void k_shift_cols(int64_t T, int32_t* __restrict__ idx, int64_t delta) {
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < T; t += (int64_t)gridDim.x * blockDim.x)
        idx[t] = (int32_t)(idx[t] + delta);
}

// out[0] = min column, out[1] = max column, out[2] = max |col - (row + row_offset)|;
// TILES: over mBSR tiles (tile units), else over CSR entries (scalar units).
template <bool TILES>
__global__ void k_col_range(int64_t rows, const int64_t* __restrict__ ptr, const int32_t* __restrict__ idx,
                            int64_t row_offset, unsigned long long* __restrict__ out) {
    long long mn = LLONG_MAX, mx = LLONG_MIN, bw = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < rows; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t a = ptr[i], b = ptr[i + 1];
        if (a == b) continue;
        const long long lo = idx[a], hi = idx[b - 1], g = i + row_offset;
        mn = min(mn, lo);
        mx = max(mx, hi);
        bw = max(bw, max(g - lo, hi - g));
    }
    for (int d = 16; d; d >>= 1) {
        mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, d));
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, d));
        bw = max(bw, __shfl_xor_sync(0xffffffffu, bw, d));
    }
    if ((threadIdx.x & 31) == 0) {
        atomicMin(reinterpret_cast<long long*>(out), mn);
        atomicMax(reinterpret_cast<long long*>(out) + 1, mx);
        atomicMax(reinterpret_cast<long long*>(out) + 2, bw);
    }
}

static amgt_status col_range(bool tiles, int64_t rows, const int64_t* ptr, const int32_t* idx, int64_t row_offset,
                             int64_t* out_host, cudaStream_t s) {
    Alloc a{nullptr, s};
    Scratch<unsigned long long> d;
    AMGT_TRY(d.init(a, 3));
    const long long init[3] = {LLONG_MAX, LLONG_MIN, 0};
    AMGT_CUDA(cudaMemcpyAsync(d.p, init, sizeof(init), cudaMemcpyHostToDevice, s));
    if (rows > 0) {
        if (tiles) k_col_range<true><<<grid_for(rows, 256), 256, 0, s>>>(rows, ptr, idx, row_offset, d.p);
        else k_col_range<false><<<grid_for(rows, 256), 256, 0, s>>>(rows, ptr, idx, row_offset, d.p);
        AMGT_LAUNCHED();
    }
    long long h[3];
    AMGT_CUDA(cudaMemcpyAsync(h, d.p, sizeof(h), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaStreamSynchronize(s));
    for (int k = 0; k < 3; ++k) out_host[k] = h[k];
    return AMGT_OK;
}

}  // namespace amgt

using namespace amgt;

extern "C" {

amgt_status amgt_csr_to_mbsr(int64_t m, int64_t n, int64_t nnz, const int64_t* row_ptr, const int32_t* col_idx,
                             const double* val, amgt_prec prec, amgt_mbsr* out, const amgt_allocator* al,
                             void* stream) {
    if (!out || m < 0 || n < 0 || nnz < 0 || !prec_valid(prec)) return fail(AMGT_ERR_ARG, "amgt_csr_to_mbsr: bad argument");
    if (m > 0 && !row_ptr) return fail(AMGT_ERR_ARG, "amgt_csr_to_mbsr: row_ptr is NULL");
    if (nnz > 0 && (!col_idx || !val)) return fail(AMGT_ERR_ARG, "amgt_csr_to_mbsr: col/val NULL");
    if (ceil_div(n, 4) > INT32_MAX) return fail(AMGT_ERR_ARG, "amgt_csr_to_mbsr: too many columns for int32 tile indices");
    AMGT_NO_PENDING("amgt_csr_to_mbsr");
    Alloc a{al, (cudaStream_t)stream};
    return csr_to_mbsr_impl(m, n, nnz, row_ptr, col_idx, val, prec, out, a, 0);
}

amgt_status amgt_csr_to_mbsr_ex(int64_t m, int64_t n, int64_t nnz, const int64_t* row_ptr, const int32_t* col_idx,
                                const double* val, int64_t col_offset, amgt_prec prec, amgt_mbsr* out,
                                const amgt_allocator* al, void* stream) {
    if (!out || m < 0 || n < 0 || nnz < 0 || !prec_valid(prec) || col_offset < 0)
        return fail(AMGT_ERR_ARG, "amgt_csr_to_mbsr_ex: bad argument");
    if (m > 0 && !row_ptr) return fail(AMGT_ERR_ARG, "amgt_csr_to_mbsr_ex: row_ptr is NULL");
    if (nnz > 0 && (!col_idx || !val)) return fail(AMGT_ERR_ARG, "amgt_csr_to_mbsr_ex: col/val NULL");
    Alloc a{al, (cudaStream_t)stream};
    return csr_to_mbsr_impl(m, n, nnz, row_ptr, col_idx, val, prec, out, a, col_offset);
}

amgt_status amgt_mbsr_nnz(const amgt_mbsr* A, int64_t* nnz_host, void* stream) {
    if (!A || !nnz_host) return fail(AMGT_ERR_ARG, "amgt_mbsr_nnz: NULL argument");
    cudaStream_t s = (cudaStream_t)stream;
    Alloc a{nullptr, s};
    Scratch<unsigned long long> d;
    AMGT_TRY(d.init(a, 1));
    AMGT_CUDA(cudaMemsetAsync(d.p, 0, sizeof(unsigned long long), s));
    if (A->blc_num > 0) {
        k_popc_sum<<<grid_for(A->blc_num, 256), 256, 0, s>>>(A->blc_num, A->blc_map, d.p);
        AMGT_LAUNCHED();
    }
    unsigned long long h = 0;
    AMGT_CUDA(cudaMemcpyAsync(&h, d.p, sizeof(h), cudaMemcpyDeviceToHost, s));
    AMGT_CUDA(cudaStreamSynchronize(s));
    *nnz_host = (int64_t)h;
    return AMGT_OK;
}

amgt_status amgt_mbsr_to_csr(const amgt_mbsr* A, int64_t* row_ptr, int32_t* col_idx, double* val, void* stream) {
    if (!A || !row_ptr) return fail(AMGT_ERR_ARG, "amgt_mbsr_to_csr: NULL argument");
    Alloc a{nullptr, (cudaStream_t)stream};
    return mbsr_to_csr_impl(A, row_ptr, col_idx, val, a);
}

amgt_status amgt_mbsr_cast(const amgt_mbsr* in, amgt_prec to, amgt_mbsr* out, const amgt_allocator* al, void* stream) {
    if (!in || !out || !prec_valid(to)) return fail(AMGT_ERR_ARG, "amgt_mbsr_cast: bad argument");
    Alloc a{al, (cudaStream_t)stream};
    return cast_impl(in, to, out, a, nullptr);
}

amgt_status amgt_mbsr_free(amgt_mbsr* A, const amgt_allocator* al, void* stream) {
    Alloc a{al, (cudaStream_t)stream};
    return mbsr_release(A, a);
}

amgt_status amgt_mbsr_transpose(const amgt_mbsr* in, amgt_mbsr* out, const amgt_allocator* al, void* stream) {
    if (!in || !out) return fail(AMGT_ERR_ARG, "amgt_mbsr_transpose: NULL argument");
    Alloc a{al, (cudaStream_t)stream};
    return transpose_impl(in, out, a, nullptr);
}

amgt_status amgt_mbsr_shift_cols(amgt_mbsr* A, int64_t delta_tiles, int64_t new_n, void* stream) {
    if (!A || new_n < 0) return fail(AMGT_ERR_ARG, "amgt_mbsr_shift_cols: bad argument");
    cudaStream_t s = (cudaStream_t)stream;
    if (A->blc_num > 0 && delta_tiles != 0) {
        k_shift_cols<<<grid_for(A->blc_num, 256), 256, 0, s>>>(A->blc_num, A->blc_idx, delta_tiles);
        AMGT_LAUNCHED();
    }
    A->n = new_n;
    A->blc_col = ceil_div(new_n, 4);
    return AMGT_OK;
}

amgt_status amgt_csr_col_range(int64_t m, const int64_t* row_ptr, const int32_t* col_idx, int64_t row_offset,
                               int64_t* out3_host, void* stream) {
    if (!out3_host || m < 0) return fail(AMGT_ERR_ARG, "amgt_csr_col_range: bad argument");
    return col_range(false, m, row_ptr, col_idx, row_offset, out3_host, (cudaStream_t)stream);
}

amgt_status amgt_mbsr_col_range(const amgt_mbsr* A, int64_t blk_row_offset, int64_t* out3_host, void* stream) {
    if (!A || !out3_host) return fail(AMGT_ERR_ARG, "amgt_mbsr_col_range: bad argument");
    return col_range(true, A->blc_row, A->blc_ptr, A->blc_idx, blk_row_offset, out3_host, (cudaStream_t)stream);
}

amgt_status amgt_mbsr_wrap(int64_t m, int64_t n, int64_t blc_num, int64_t* blc_ptr, int32_t* blc_idx,
                           uint16_t* blc_map, void* blc_val, amgt_prec prec, amgt_mbsr* out) {
    if (!out || m < 0 || n < 0 || blc_num < 0 || !prec_valid(prec)) return fail(AMGT_ERR_ARG, "amgt_mbsr_wrap: bad argument");
    *out = amgt_mbsr{};
    out->m = m;
    out->n = n;
    out->blc_row = ceil_div(m, 4);
    out->blc_col = ceil_div(n, 4);
    out->blc_num = blc_num;
    out->blc_ptr = blc_ptr;
    out->blc_idx = blc_idx;
    out->blc_map = blc_map;
    out->blc_val = blc_val;
    out->prec = prec;
    return AMGT_OK;
}

}  // extern "C"
