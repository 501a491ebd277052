// spgemm.cu — C = A*B over mBSR (§IV.C; Alg. 3; Alg. 4).
//
// Pipeline (all on the device; one host sync when every row has <= 32 candidates, else two):
//   step 1        k_sym_flat<1> over every block row: Cub(I) = sum_{K in A(I,:)}
//                 #tiles(B(K,:)) and bin(I) (L149-151; 8 bins, edges 128*2^b, reading R7)
//                 and, for the rows with Cub <= 32 (category 8), the distinct tile columns J
//                 with BITMAPMULTIPLY(mapA, mapB) != 0 (Alg. 3 lines 1-13) -> nnzC_row;
//                 prefix sum -> blc_ptrC; host reads the bins and the C tile count (L153).
//   long rows     (only when some row has Cub > 32) row lists per bin (k_bin_scatter), the
//                 per-bin hash kernels of step 1, prefix sum again, second host sync.
//   step 2        insert again, OR the bitmaps (R15), compress, sort ascending (Alg. 3 lines
//                 13-14) -> blc_idxC, blc_mapC: k_sym_flat<2> + the per-bin kernels.
//   numeric       rows by C-row length (<= 8 C tiles: staged 4-lane-group kernel; 9-32: warp
//                 per row; longer rows: one streaming pass over the records step 2 left —
//                 the numeric plan, DESIGN R34 — or, without records, 33-512 warp / > 512
//                 two-pass kernels).  A tiles with POPCOUNT >= threshold go to the tensor-core
//                 route (DMMA m8n8k4: fragA = [A;A], fragB = [Bj|Bj'], keep the two diagonal
//                 quadrants, L157-171); the others to CUDA cores (L173).  Deterministic for rows
//                 with <= 32 C tiles (all rows with AMGT_SPGEMM_DET=1).
//
// Hash tables (R8): power-of-two, >= 2x the bin's Cub upper bound, multiplicative hash,
// linear probing.  Bins 0-1: one warp per row, table per warp; bins 2-4: one block per row,
// table per block, block radix sort; from the bin whose lower edge reaches W/8 words (W = B's
// column words): dense bitmaps over B's tile columns — per row in global memory, the row spread
// over (row, 256-tile) work items (k_gdense_*; or k_sym_dense, one CTA per row) — sorted by
// construction.
#include <algorithm>
#include <cmath>
#include <climits>
#include <cstring>
#include <mutex>
#include <type_traits>
#include <vector>

#include "common.cuh"

#include <cub/block/block_radix_sort.cuh>

namespace amgt {

amgt_status mbsr_alloc(amgt_mbsr* M, int64_t m, int64_t n, int64_t T, amgt_prec prec, Alloc& a, bool structure,
                       bool values, int64_t* existing_ptr);
amgt_status mbsr_release(amgt_mbsr* M, Alloc& a);

constexpr int NBINS = 8;
// Internal row categories: the paper's 8 bins (L151) plus category 8 = the rows of bin 0
// with Cub <= 32, which the 4-lane-group symbolic kernel takes.  stats[] layout:
// [0..7] bins (category 8 counted separately), [8] cub_total, [9] pairs_nonzero,
// [10] pairs_tc, [11] scalar products, [12] category-8 rows.
constexpr int NCAT = 9;
constexpr int SMALL_CUB = 32;
__host__ __device__ inline int cat_stat(int c) { return c < NBINS ? c : 12; }
constexpr int EMPTY_KEY = -1;

struct SymCtx {  // device pointers shared by the symbolic kernels
    const int64_t* aptr;
    const int32_t* aidx;
    const uint16_t* amap;
    const int64_t* bptr;
    const int32_t* bidx;
    const uint16_t* bmap;
};

// ---------------------------------------------------------------- analysis + binning
// (Cub and the bins are computed by k_sym_flat<1> below, L149-151.)

// Pair statistics for amgt_spgemm_info (info only): one thread per A tile over its B row.
__global__ void k_pair_stats(int64_t TA, SymCtx c, unsigned long long* __restrict__ stats, int tc_thr) {
    unsigned long long pnz = 0, ptc = 0, sp = 0;
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < TA; t += (int64_t)gridDim.x * blockDim.x) {
        const int32_t K = c.aidx[t];
        const uint32_t ma = c.amap[t];
        const bool tc = __popc(ma) >= tc_thr;
        for (int64_t j = c.bptr[K]; j < c.bptr[K + 1]; ++j) {
            const uint32_t mb = c.bmap[j];
            if (bitmap_multiply(ma, mb)) {
                ++pnz;
                ptc += tc;
#pragma unroll
                for (int k = 0; k < 4; ++k) sp += __popc((ma >> k) & 0x1111u) * __popc((mb >> (4 * k)) & 0xFu);
            }
        }
    }
    for (int d = 16; d; d >>= 1) {
        pnz += __shfl_xor_sync(0xffffffffu, pnz, d);
        ptc += __shfl_xor_sync(0xffffffffu, ptc, d);
        sp += __shfl_xor_sync(0xffffffffu, sp, d);
    }
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(stats + 9, pnz);
        atomicAdd(stats + 10, ptc);
        atomicAdd(stats + 11, sp);
    }
}

__global__ void k_bin_scatter(int64_t BR, const int64_t* __restrict__ bin_of, const unsigned long long* __restrict__ stats,
                              unsigned long long* __restrict__ cursor, int32_t* __restrict__ rows) {
    __shared__ unsigned long long off[NCAT];
    if (threadIdx.x == 0) {
        unsigned long long s = 0;
        for (int b = 0; b < NCAT; ++b) { off[b] = s; s += stats[cat_stat(b)]; }
    }
    __syncthreads();
    const int lane = threadIdx.x & 31;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < BR; base += (int64_t)gridDim.x * blockDim.x) {
        const int64_t I = base + threadIdx.x;
        const int b = I < BR ? (int)bin_of[I] : -1;
        const uint32_t peers = __match_any_sync(0xffffffffu, b);  // warp-aggregated atomics
        const int leader = __ffs(peers) - 1;
        unsigned long long pos = 0;
        if (lane == leader && b >= 0) pos = atomicAdd(&cursor[b], (unsigned long long)__popc(peers));
        pos = __shfl_sync(0xffffffffu, pos, leader);
        if (b >= 0) rows[off[b] + pos + __popc(peers & ((1u << lane) - 1u))] = (int32_t)I;
    }
}

// ---------------------------------------------------------------- hashing
__device__ __forceinline__ uint32_t hash_slot(int32_t J, int logS) {
    return ((uint32_t)J * 0x9E3779B1u) >> (32 - logS);
}

// Returns true when J was newly inserted.
__device__ __forceinline__ bool hash_insert(int* keys, uint32_t* maps, int logS, int32_t J, uint32_t mapC, bool or_map) {
    const uint32_t mask = (1u << logS) - 1u;
    uint32_t h = hash_slot(J, logS);
    for (;;) {
        const int k = ((volatile int*)keys)[h];
        if (k == J) {
            if (or_map) atomicOr(maps + h, mapC);
            return false;
        }
        if (k == EMPTY_KEY) {
            const int old = atomicCAS(keys + h, EMPTY_KEY, J);
            if (old == EMPTY_KEY || old == J) {
                if (or_map) atomicOr(maps + h, mapC);
                return old == EMPTY_KEY;
            }
        }
        h = (h + 1) & mask;
    }
}

// hash_insert that also returns the slot holding J (the plan's records refer to it until the
// sort has fixed the columns' ranks)
__device__ __forceinline__ int hash_insert_at(int* keys, uint32_t* maps, int logS, int32_t J, uint32_t mapC) {
    const uint32_t mask = (1u << logS) - 1u;
    uint32_t h = hash_slot(J, logS);
    for (;;) {
        const int k = ((volatile int*)keys)[h];
        if (k == J) {
            atomicOr(maps + h, mapC);
            return (int)h;
        }
        if (k == EMPTY_KEY) {
            const int old = atomicCAS(keys + h, EMPTY_KEY, J);
            if (old == EMPTY_KEY || old == J) {
                atomicOr(maps + h, mapC);
                return (int)h;
            }
        }
        h = (h + 1) & mask;
    }
}

// Warp-cooperative enumeration of the (A tile, B tile) pairs of block row I: lanes take
// up to 32 A tiles, warp-scan their B-row lengths, then spread the pairs over lanes.
// fn(J, mapC) is called for every pair with mapC != 0 — or fn(J, mapC, t, j, pos) with the
// pair's A tile t, B tile j and its ordinal among the row's pairs (A-tile order, then B order).
template <typename F>
__device__ __forceinline__ void warp_pairs(const SymCtx& c, int64_t I, int lane, F&& fn) {
    const int64_t a0 = c.aptr[I], a1 = c.aptr[I + 1];
    int64_t rbase = 0;  // pairs of the previous 32-tile chunks
    for (int64_t base = a0; base < a1; base += 32) {
        const int64_t t = base + lane;
        const bool v = t < a1;
        const int32_t K = v ? c.aidx[t] : 0;
        const uint32_t ma = v ? c.amap[t] : 0u;
        const int64_t b0 = v ? c.bptr[K] : 0;
        const int64_t len = v ? c.bptr[K + 1] - b0 : 0;
        int64_t incl = len;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const int64_t y = __shfl_up_sync(0xffffffffu, incl, d);
            if (lane >= d) incl += y;
        }
        const int64_t excl = incl - len;
        const int64_t total = __shfl_sync(0xffffffffu, incl, 31);
        for (int64_t p0 = 0; p0 < total; p0 += 32) {
            const int64_t p = p0 + lane;
            int lo = 0;
#pragma unroll
            for (int step = 16; step; step >>= 1) {
                const int cand = lo + step;
                const int64_t e = __shfl_sync(0xffffffffu, excl, cand & 31);
                if (cand < 32 && e <= p) lo = cand;
            }
            const int64_t ob0 = __shfl_sync(0xffffffffu, b0, lo);
            const int64_t oex = __shfl_sync(0xffffffffu, excl, lo);
            const uint32_t oma = __shfl_sync(0xffffffffu, ma, lo);
            if (p < total) {
                const int64_t j = ob0 + (p - oex);
                const uint32_t mc = bitmap_multiply(oma, c.bmap[j]);
                if constexpr (std::is_invocable_v<F, int32_t, uint32_t, int64_t, int64_t, int64_t>) {
                    if (mc) fn(c.bidx[j], mc, base + lo, j, rbase + p);
                } else {
                    if (mc) fn(c.bidx[j], mc);
                }
            }
        }
        rbase += total;
    }
}

// Block-cooperative version: chunks of blockDim A tiles, owner search in shared memory.
constexpr int PAIR_U = 4;
template <typename F>
__device__ __forceinline__ void block_pairs_range(const SymCtx& c, int64_t a0, int64_t a1, int64_t* sh_excl,
                                                  int64_t* sh_b0, uint32_t* sh_ma, int64_t* sh_tot, F&& fn) {
    const int nt = blockDim.x, tid = threadIdx.x;
    const int lane = tid & 31, w = tid >> 5, nw = nt >> 5;
    for (int64_t base = a0; base < a1; base += nt) {
        const int64_t t = base + tid;
        const bool v = t < a1;
        const int32_t K = v ? c.aidx[t] : 0;
        const uint32_t ma = v ? c.amap[t] : 0u;
        const int64_t b0 = v ? c.bptr[K] : 0;
        const int64_t len = v ? c.bptr[K + 1] - b0 : 0;
        // block exclusive scan of len (warp scans + warp totals in sh_tot)
        int64_t incl = len;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const int64_t y = __shfl_up_sync(0xffffffffu, incl, d);
            if (lane >= d) incl += y;
        }
        if (lane == 31) sh_tot[w] = incl;
        __syncthreads();
        if (tid == 0) {
            int64_t s = 0;
            for (int k = 0; k < nw; ++k) { const int64_t x = sh_tot[k]; sh_tot[k] = s; s += x; }
            sh_tot[nw] = s;
        }
        __syncthreads();
        const int64_t excl = sh_tot[w] + incl - len;
        sh_excl[tid] = excl;
        sh_b0[tid] = b0;
        sh_ma[tid] = ma;
        const int64_t total = sh_tot[nw];
        __syncthreads();
        const int nvalid = (int)min((int64_t)nt, a1 - base);
        // PAIR_U pairs per thread per round: their B-tile loads are all in flight together
        for (int64_t p0 = tid; p0 < total; p0 += (int64_t)nt * PAIR_U) {
            int lo_[PAIR_U];
            int64_t j_[PAIR_U];
            uint32_t mb_[PAIR_U];
            int32_t J_[PAIR_U];
#pragma unroll
            for (int u = 0; u < PAIR_U; ++u) {
                const int64_t p = p0 + (int64_t)u * nt;
                int lo = 0, hi = nvalid - 1;  // largest o with excl[o] <= p
                while (lo < hi) {
                    const int mid = (lo + hi + 1) >> 1;
                    if (sh_excl[mid] <= p) lo = mid; else hi = mid - 1;
                }
                lo_[u] = lo;
                j_[u] = p < total ? sh_b0[lo] + (p - sh_excl[lo]) : -1;
            }
#pragma unroll
            for (int u = 0; u < PAIR_U; ++u) {
                mb_[u] = j_[u] >= 0 ? c.bmap[j_[u]] : 0u;
                J_[u] = j_[u] >= 0 ? c.bidx[j_[u]] : 0;
            }
#pragma unroll
            for (int u = 0; u < PAIR_U; ++u) {
                const uint32_t mc = j_[u] >= 0 ? bitmap_multiply(sh_ma[lo_[u]], mb_[u]) : 0u;
                if (mc) fn(J_[u], mc);
            }
        }
        __syncthreads();
    }
}
// block_pairs_range that also hands fn the pair's A tile t, B tile j and aux(t) + (j - first
// tile of B row K): aux(t, K, pos0) is evaluated once per A tile (pos0: the ordinal of the
// tile's first pair in the range; the plan's record position base).
template <typename G, typename F>
__device__ __forceinline__ void block_pairs_aux(const SymCtx& c, int64_t a0, int64_t a1, int64_t* sh_excl,
                                                int64_t* sh_b0, uint32_t* sh_ma, int64_t* sh_tot, int64_t* sh_aux,
                                                G&& aux, F&& fn) {
    const int nt = blockDim.x, tid = threadIdx.x;
    const int lane = tid & 31, w = tid >> 5, nw = nt >> 5;
    int64_t rbase = 0;  // pairs of the previous chunks of the range
    for (int64_t base = a0; base < a1; base += nt) {
        const int64_t t = base + tid;
        const bool v = t < a1;
        const int32_t K = v ? c.aidx[t] : 0;
        const uint32_t ma = v ? c.amap[t] : 0u;
        const int64_t b0 = v ? c.bptr[K] : 0;
        const int64_t len = v ? c.bptr[K + 1] - b0 : 0;
        int64_t incl = len;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const int64_t y = __shfl_up_sync(0xffffffffu, incl, d);
            if (lane >= d) incl += y;
        }
        if (lane == 31) sh_tot[w] = incl;
        __syncthreads();
        if (tid == 0) {
            int64_t s = 0;
            for (int k = 0; k < nw; ++k) { const int64_t x = sh_tot[k]; sh_tot[k] = s; s += x; }
            sh_tot[nw] = s;
        }
        __syncthreads();
        const int64_t excl = sh_tot[w] + incl - len;
        sh_excl[tid] = excl;
        sh_b0[tid] = b0;
        sh_ma[tid] = ma;
        sh_aux[tid] = v ? aux(t, K, rbase + excl) : 0;
        const int64_t total = sh_tot[nw];
        __syncthreads();
        const int nvalid = (int)min((int64_t)nt, a1 - base);
        for (int64_t p0 = tid; p0 < total; p0 += (int64_t)nt * PAIR_U) {
            int lo_[PAIR_U];
            int64_t j_[PAIR_U], off_[PAIR_U];
            uint32_t mb_[PAIR_U];
            int32_t J_[PAIR_U];
#pragma unroll
            for (int u = 0; u < PAIR_U; ++u) {
                const int64_t p = p0 + (int64_t)u * nt;
                int lo = 0, hi = nvalid - 1;
                while (lo < hi) {
                    const int mid = (lo + hi + 1) >> 1;
                    if (sh_excl[mid] <= p) lo = mid; else hi = mid - 1;
                }
                lo_[u] = lo;
                off_[u] = p - sh_excl[lo];
                j_[u] = p < total ? sh_b0[lo] + off_[u] : -1;
            }
#pragma unroll
            for (int u = 0; u < PAIR_U; ++u) {
                mb_[u] = j_[u] >= 0 ? c.bmap[j_[u]] : 0u;
                J_[u] = j_[u] >= 0 ? c.bidx[j_[u]] : 0;
            }
#pragma unroll
            for (int u = 0; u < PAIR_U; ++u) {
                const uint32_t mc = j_[u] >= 0 ? bitmap_multiply(sh_ma[lo_[u]], mb_[u]) : 0u;
                if (mc) fn(J_[u], mc, base + lo_[u], j_[u], sh_aux[lo_[u]] + off_[u]);
            }
        }
        rbase += total;
        __syncthreads();
    }
}
template <typename F>
__device__ __forceinline__ void block_pairs(const SymCtx& c, int64_t I, int64_t* sh_excl, int64_t* sh_b0,
                                            uint32_t* sh_ma, int64_t* sh_tot, F&& fn) {
    block_pairs_range(c, c.aptr[I], c.aptr[I + 1], sh_excl, sh_b0, sh_ma, sh_tot, fn);
}

// Numeric plan records of the hash-bin rows with more than CAP C tiles (written by symbolic
// step 2 after the sort): rec[hoff[I] + pos] for the row's pos-th pair (A-tile order, then B
// order), products per C tile counted in cnt, rowf[I] = 1.
struct HRec {
    const int64_t* hoff;  // [BR+1] record offsets per row (0-length: no records)
    int4* rec;
    uint32_t* cnt;
    uint8_t* rowf;
};

// ---------------------------------------------------------------- step kernels: warp bins
// LOGS = log2(table slots per warp).  STEP 1: count -> nnz_row[I].  STEP 2: write sorted
// idx/map at ptrC[I].
template <int LOGS, int STEP>
__global__ void __launch_bounds__(256, 8) k_sym_warp(int64_t nrows, const int32_t* __restrict__ rows, SymCtx c,
                                                  int64_t* __restrict__ nnz_row, const int64_t* __restrict__ cptr,
                                                  int32_t* __restrict__ cidx, uint16_t* __restrict__ cmap, HRec hr) {
    constexpr int S = 1 << LOGS;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int* keys = reinterpret_cast<int*>(smem_raw) + w * (2 * S + S / 2);
    uint32_t* maps = reinterpret_cast<uint32_t*>(keys + S);
    int* oslot = keys + 2 * S;  // step 2, rows with records: hash slot of each compressed entry
    const int64_t wg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (wg >= nrows) return;
    const int64_t I = rows[wg];
    for (int i = lane; i < S; i += 32) {
        keys[i] = EMPTY_KEY;
        maps[i] = 0;
    }
    __syncwarp();
    int64_t r0 = 0, r1 = 0;
    if (STEP == 2 && hr.rec) {
        r0 = hr.hoff[I];
        r1 = hr.hoff[I + 1];
    }
    int cnt = 0;
    if (STEP == 2 && r1 > r0) {  // records {hash slot, B tile, A tile, bitmap product} (R34)
        warp_pairs(c, I, lane, [&](int32_t J, uint32_t mc, int64_t t, int64_t j, int64_t pos) {
            const int h = hash_insert_at(keys, maps, LOGS, J, mc);
            hr.rec[r0 + pos] = make_int4(h, (int)j, (int)t, (int)mc);
        });
    } else {
        warp_pairs(c, I, lane, [&](int32_t J, uint32_t mc) { cnt += hash_insert(keys, maps, LOGS, J, mc, STEP == 2); });
    }
    __syncwarp();
    if (STEP == 1) {
#pragma unroll
        for (int d = 16; d; d >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, d);
        if (lane == 0) nnz_row[I] = cnt;
        return;
    }
    // compress in place (rounds of 32 slots; all reads of a round precede its writes)
    int n = 0;
    for (int base = 0; base < S; base += 32) {
        const int k = keys[base + lane];
        const uint32_t mp = maps[base + lane];
        const bool v = k != EMPTY_KEY;
        const uint32_t bal = __ballot_sync(0xffffffffu, v);
        __syncwarp();
        if (v) {
            const int pos = n + __popc(bal & ((1u << lane) - 1u));
            keys[pos] = k;
            maps[pos] = mp;
            oslot[pos] = base + lane;
        }
        n += __popc(bal);
        __syncwarp();
    }
    // rank sort (n <= S/2 distinct keys); with records, maps[i] <- rank of entry i
    const int64_t out = cptr[I];
    for (int i = lane; i < n; i += 32) {
        const int k = keys[i];
        int rank = 0;
        for (int j = 0; j < n; ++j) rank += keys[j] < k;
        cidx[out + rank] = k;
        cmap[out + rank] = (uint16_t)maps[i];
        maps[i] = (uint32_t)rank;
    }
    if (r1 > r0) {  // slot -> rank table in keys[], then the row's records get their C tiles
        __syncwarp();
        if (lane == 0) hr.rowf[I] = 1;
        int sl[S / 64 > 0 ? S / 64 : 1], rk[S / 64 > 0 ? S / 64 : 1];
#pragma unroll
        for (int u = 0; u < (S / 64 > 0 ? S / 64 : 1); ++u) {
            const int i = lane + 32 * u;
            sl[u] = i < n ? oslot[i] : -1;
            rk[u] = i < n ? (int)maps[i] : 0;
        }
        __syncwarp();
#pragma unroll
        for (int u = 0; u < (S / 64 > 0 ? S / 64 : 1); ++u)
            if (sl[u] >= 0) keys[sl[u]] = rk[u];
        __syncwarp();
        for (int64_t pb = r0 + lane; pb < r1; pb += 4 * 32) {  // four records per lane in flight
            int hv[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) hv[u] = pb + 32 * u < r1 ? reinterpret_cast<const int*>(hr.rec + pb + 32 * u)[0] : -1;
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                if (hv[u] < 0) continue;
                const int64_t q = out + keys[hv[u]];
                reinterpret_cast<int*>(hr.rec + pb + 32 * u)[0] = (int)q;
                atomicAdd(hr.cnt + q, 1u);
            }
        }
    }
}

// ---------------------------------------------------------------- step kernels: tiny rows
// Every block row goes through k_sym_flat, which also does the analysis and binning (L149-151:
// Cub(I) = sum_{K in A(I,:)} #tiles(B(K,:)), bin edges 128*2^b, reading R7).  One warp takes
// SF_ROWS = 16 consecutive block rows; their A tiles are one contiguous range, which the 32
// lanes walk 128 tiles at a time (4 per lane: columns, bitmaps, B-row ranges all requested
// together, so a few dependent round trips per warp instead of per tile).  Each lane appends its tile's (A tile, B tile) pairs to
// its row's candidate list in shared memory at the row-local pair position (A-tile order, then
// B order): the candidate is the tile column J when BITMAPMULTIPLY(mapA, mapB) != 0 (Alg. 3
// lines 7-8).  The list length is Cub.  Rows with Cub <= 32 (category 8) are finished here by
// one 4-lane group: a candidate counts when it is the first occurrence of its J (the
// collision-free degenerate form of the paper's hash table, Alg. 3 lines 9-11); step 1 writes
// the distinct count, step 2 writes each distinct J at its rank with the OR of the bitmaps of
// all its occurrences (lines 13-14, R15).  Deterministic, no atomics on the data.  Rows with
// Cub > 32 are only binned here (bin_of, stats) and left to the per-bin hash kernels.
// (A 4-lane group per row walking its own tiles measured 92 + 104 us for the config-2 A*P
// steps: latency-bound dependent chains.)
constexpr int SF_ROWS = 16;  // block rows per warp in k_sym_flat
constexpr int SF_U = 4;      // A tiles per lane per round (all their loads in flight together)
// sidx/smap (step 1, optional): the finished sorted list of every category-8 row is also
// written to its slot [32 I, 32 I + n) of these scratch arrays, and k_sym_copy moves it into C
// once the row offsets exist — step 2's re-expansion of the pairs is then skipped.
template <int STEP>
__global__ void __launch_bounds__(256) k_sym_flat(int64_t BR, SymCtx c, int64_t* __restrict__ nnz_row,
                                                  const int64_t* __restrict__ cptr, int32_t* __restrict__ cidx,
                                                  uint16_t* __restrict__ cmap, int64_t* __restrict__ bin_of,
                                                  unsigned long long* __restrict__ stats,
                                                  int32_t* __restrict__ sidx = nullptr,
                                                  uint16_t* __restrict__ smap = nullptr,
                                                  const int64_t* __restrict__ pp = nullptr,
                                                  int64_t* __restrict__ cub_row = nullptr) {
    // pp (optional): pair prefix over A tiles -> Cub(I) = pp[aptr[I+1]] - pp[aptr[I]] directly;
    // the tiles of rows with Cub > SMALL_CUB (power-law rows of thousands of tiles) are then
    // jumped over instead of walked.
    // row stride padded by one word: the 8 groups of a warp read the same position of 8
    // different rows at once (an unpadded 128-B stride puts them all in one bank)
    __shared__ int keys[8][SF_ROWS][SMALL_CUB + 1];
    __shared__ uint32_t maps[8][SF_ROWS][SMALL_CUB + 1];
    __shared__ unsigned char first[8][SF_ROWS][SMALL_CUB + 4];
    __shared__ int npair[8][SF_ROWS];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, g = lane >> 2, r = lane & 3;
    const unsigned gm = 0xFu << (lane & ~3);
    const int64_t I0 = ((int64_t)blockIdx.x * 8 + w) * SF_ROWS;
    if (I0 >= BR) return;  // whole warp
    const int nr = (int)min((int64_t)SF_ROWS, BR - I0);
    const int64_t ap = lane <= nr ? c.aptr[I0 + lane] : 0;  // lane k: start of row I0 + k
    const int64_t T0 = __shfl_sync(0xffffffffu, ap, 0), T1 = __shfl_sync(0xffffffffu, ap, nr);
    // lane k < nr: Cub of row I0 + k from pp (pp[ap] at lane k, pp[ap of k+1] from lane k+1)
    int64_t pcub = 0;
    if (pp) {
        const int64_t pk = lane <= nr ? pp[ap] : 0;
        const int64_t pk1 = __shfl_down_sync(0xffffffffu, pk, 1);
        pcub = lane < nr ? pk1 - pk : 0;
    }
    const unsigned bigrows = __ballot_sync(0xffffffffu, pp != nullptr && lane < nr && pcub > SMALL_CUB);
    if (lane < SF_ROWS) npair[w][lane] = 0;
    __syncwarp();
    for (int64_t base = T0; base < T1; base += 32 * SF_U) {
        if (bigrows) {  // warp-uniform: skip whole chunks that start inside a big row
            int rb = 0;
#pragma unroll
            for (int k = 1; k < SF_ROWS; ++k) {
                const int64_t sk = __shfl_sync(0xffffffffu, ap, k);
                rb += (k < nr && sk <= base);
            }
            bool jumped = false;
            while (rb < nr && ((bigrows >> rb) & 1u)) {
                base = __shfl_sync(0xffffffffu, ap, rb + 1);  // start of the next row
                ++rb;
                jumped = true;
            }
            if (base >= T1) break;
            (void)jumped;
        }
        int32_t K[SF_U];
        uint32_t ma[SF_U];
        int64_t b0[SF_U];
        int len[SF_U];
#pragma unroll
        for (int u = 0; u < SF_U; ++u) {  // tile base + 32u + lane
            const int64_t t = base + 32 * u + lane;
            K[u] = t < T1 ? c.aidx[t] : -1;
            ma[u] = t < T1 ? c.amap[t] : 0u;
        }
#pragma unroll
        for (int u = 0; u < SF_U; ++u) {
            b0[u] = K[u] >= 0 ? c.bptr[K[u]] : 0;
            len[u] = K[u] >= 0 ? (int)(c.bptr[K[u] + 1] - b0[u]) : 0;
        }
#pragma unroll
        for (int u = 0; u < SF_U; ++u) {
            const int64_t t = base + 32 * u + lane;
            if (__all_sync(0xffffffffu, t >= T1)) break;
            int row = 0;  // the tile's row within the warp: #{k in 1..nr-1 : start(k) <= t}
#pragma unroll
            for (int k = 1; k < SF_ROWS; ++k) {
                const int64_t sk = __shfl_sync(0xffffffffu, ap, k);
                row += (k < nr && sk <= t);
            }
            int incl = len[u];
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const int y = __shfl_up_sync(0xffffffffu, incl, d);
                if (lane >= d) incl += y;
            }
            const int excl = incl - len[u];
            const int prow = __shfl_up_sync(0xffffffffu, row, 1);
            const unsigned seg = __ballot_sync(0xffffffffu, lane == 0 || row != prow);  // segment starts
            const int start = 31 - __clz(seg & (0xffffffffu >> (31 - lane)));
            const int excl0 = __shfl_sync(0xffffffffu, excl, start);
            const int off = npair[w][row] + excl - excl0;
            int* Kl = keys[w][row];
            uint32_t* Ml = maps[w][row];
            for (int jj = 0; jj < len[u] && off + jj < SMALL_CUB; ++jj) {
                const int64_t j = b0[u] + jj;
                const uint32_t mc = bitmap_multiply(ma[u], c.bmap[j]);
                Kl[off + jj] = mc ? c.bidx[j] : -1;
                Ml[off + jj] = mc;
            }
            const bool last = lane == 31 || ((seg >> (lane + 1)) & 1u);
            __syncwarp();
            if (last) npair[w][row] += incl - excl0;
            __syncwarp();
        }
    }
    // rows g and g + 8 of the warp: one 4-lane group each, in turn
    for (int h = 0; h < SF_ROWS / 8; ++h) {
        const int gr = g + 8 * h;
        const bool own = gr < nr;
        const int64_t I = I0 + gr;
        const int64_t pc = __shfl_sync(0xffffffffu, pcub, gr);
        const int64_t cub = own ? (pp ? pc : (int64_t)npair[w][gr]) : 0;
        bool small = false;
        if (STEP == 1) {
            int b = 0;
            while (b < NBINS - 1 && cub >= (128ll << b)) ++b;
            if (b == 0 && cub <= SMALL_CUB) b = NBINS;  // category 8
            small = b == NBINS;
            const bool lead = own && r == 0;
            if (lead) {
                bin_of[I] = b;
                if (!small) {
                    nnz_row[I] = 0;  // counted by its bin's kernel
                    atomicAdd(&stats[cat_stat(b)], 1ull);
                    if (cub_row) cub_row[I] = cub;
                }
            }
            const unsigned n8 = __ballot_sync(0xffffffffu, lead && small);
            unsigned long long ct = lead ? (unsigned long long)cub : 0ull;
            for (int d = 16; d; d >>= 1) ct += __shfl_xor_sync(0xffffffffu, ct, d);
            if (lane == 0) {
                if (n8) atomicAdd(&stats[cat_stat(NBINS)], (unsigned long long)__popc(n8));
                if (ct) atomicAdd(&stats[8], ct);
            }
        } else {
            small = own && cub <= SMALL_CUB;  // same classification as step 1
        }
        if (!own || !small) continue;  // group-uniform
        const int* Kr = keys[w][gr];
        const uint32_t* Mr = maps[w][gr];
        unsigned char* F = first[w][gr];
        const int n = (int)cub;
        int cnt = 0;
        for (int i = r; i < n; i += 4) {  // first occurrences
            const int k = Kr[i];
            bool f = k >= 0;
            for (int j = 0; j < i && f; ++j) f = Kr[j] != k;
            F[i] = f;
            cnt += f;
        }
        cnt += __shfl_xor_sync(gm, cnt, 1, 4);
        cnt += __shfl_xor_sync(gm, cnt, 2, 4);
        if (STEP == 1) {
            if (r == 0) nnz_row[I] = cnt;
            if (!sidx) continue;
        }
        __syncwarp(gm);
        int32_t* oi = STEP == 1 ? sidx + SMALL_CUB * I : cidx + cptr[I];
        uint16_t* om = STEP == 1 ? smap + SMALL_CUB * I : cmap + cptr[I];
        for (int i = r; i < n; i += 4) {
            if (!F[i]) continue;
            const int k = Kr[i];
            int rank = 0;
            uint32_t m = 0;
            for (int j = 0; j < n; ++j) {
                const int kj = Kr[j];
                rank += (F[j] && kj < k);
                m |= (kj == k) ? Mr[j] : 0u;
            }
            oi[rank] = k;
            om[rank] = (uint16_t)m;
        }
    }
}

// Symbolic step 1 when every block row of B holds at most one tile (A P with an aggregation P,
// R19) and every row of A at most 32 tiles: Cub(I) = the A tiles of row I whose B row is not
// empty (all category 8).  A 4-lane group per row resolves them (lane r: tiles 4s + r, s < 8 —
// column and bitmap, B row pointers, B column and bitmap: three rounds of independent loads) and
// extracts the distinct columns J with BITMAPMULTIPLY != 0 in ascending order, each with the OR
// of its bitmap products (group min / OR by shuffles; no shared memory, no pair lists).  The
// sorted list goes to the row's 32-slot scratch row for k_sym_copy, the count to nnz_row: the
// same outputs as k_sym_flat<1> for these rows.
__global__ void __launch_bounds__(256) k_sym_b1(int64_t BR, SymCtx c, int64_t* __restrict__ nnz_row,
                                                int64_t* __restrict__ bin_of, unsigned long long* __restrict__ stats,
                                                int32_t* __restrict__ sidx, uint16_t* __restrict__ smap) {
    const int lane = threadIdx.x & 31, r = lane & 3;
    const unsigned gm = 0xFu << (lane & ~3);
    unsigned long long rows8 = 0, cubs = 0;
    for (int64_t I = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 2; I < BR;
         I += ((int64_t)gridDim.x * blockDim.x) >> 2) {
        const int64_t t0 = c.aptr[I], t1 = c.aptr[I + 1];
        int32_t K[8], J[8];
        uint32_t ma[8], mc[8];
        int64_t b0[8];
        bool has[8];
#pragma unroll
        for (int s = 0; s < 8; ++s) {
            const int64_t t = t0 + 4 * s + r;
            K[s] = t < t1 ? __ldg(c.aidx + t) : -1;
            ma[s] = t < t1 ? __ldg(c.amap + t) : 0u;
        }
#pragma unroll
        for (int s = 0; s < 8; ++s) {
            b0[s] = K[s] >= 0 ? __ldg(c.bptr + K[s]) : 0;
            has[s] = K[s] >= 0 && __ldg(c.bptr + K[s] + 1) > b0[s];
        }
        int cub = 0;
#pragma unroll
        for (int s = 0; s < 8; ++s) {
            mc[s] = has[s] ? bitmap_multiply(ma[s], __ldg(c.bmap + b0[s])) : 0u;
            J[s] = mc[s] ? __ldg(c.bidx + b0[s]) : INT_MAX;
            cub += has[s];
        }
        cub += __shfl_xor_sync(gm, cub, 1, 4);
        cub += __shfl_xor_sync(gm, cub, 2, 4);
        int n = 0, prev = -1;
        for (;;) {  // group-uniform: ascending distinct columns
            int m = INT_MAX;
#pragma unroll
            for (int s = 0; s < 8; ++s) m = (J[s] > prev && J[s] < m) ? J[s] : m;
            m = min(m, __shfl_xor_sync(gm, m, 1, 4));
            m = min(m, __shfl_xor_sync(gm, m, 2, 4));
            if (m == INT_MAX) break;
            uint32_t o = 0;
#pragma unroll
            for (int s = 0; s < 8; ++s) o |= (J[s] == m) ? mc[s] : 0u;
            o |= __shfl_xor_sync(gm, o, 1, 4);
            o |= __shfl_xor_sync(gm, o, 2, 4);
            if (r == 0) {
                sidx[SMALL_CUB * I + n] = m;
                smap[SMALL_CUB * I + n] = (uint16_t)o;
            }
            ++n;
            prev = m;
        }
        if (r == 0) {
            nnz_row[I] = n;
            bin_of[I] = NBINS;
            rows8 += 1;
            cubs += (unsigned long long)cub;
        }
    }
    for (int d = 16; d; d >>= 1) {
        rows8 += __shfl_xor_sync(0xffffffffu, rows8, d);
        cubs += __shfl_xor_sync(0xffffffffu, cubs, d);
    }
    if (lane == 0) {
        if (rows8) atomicAdd(&stats[cat_stat(NBINS)], rows8);
        if (cubs) atomicAdd(&stats[8], cubs);
    }
}

// Step 2 of the category-8 rows when step 1 kept their sorted lists: copy slot [32 I, +n) to
// C at cptr[I] (4-lane group per row).
__global__ void __launch_bounds__(256) k_sym_copy(int64_t BR, const int64_t* __restrict__ bin_of,
                                                  const int64_t* __restrict__ cptr, const int32_t* __restrict__ sidx,
                                                  const uint16_t* __restrict__ smap, int32_t* __restrict__ cidx,
                                                  uint16_t* __restrict__ cmap) {
    const int r = threadIdx.x & 3;
    for (int64_t I = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 2; I < BR;
         I += ((int64_t)gridDim.x * blockDim.x) >> 2) {
        if (bin_of[I] != NBINS) continue;  // group-uniform
        const int64_t c0 = cptr[I];
        const int n = (int)(cptr[I + 1] - c0);
        for (int i = r; i < n; i += 4) {
            cidx[c0 + i] = sidx[SMALL_CUB * I + i];
            cmap[c0 + i] = smap[SMALL_CUB * I + i];
        }
    }
}

// ---------------------------------------------------------------- step kernels: block bins
template <int LOGS, int STEP>
__global__ void __launch_bounds__(LOGS >= 12 ? 512 : 256, LOGS >= 12 ? 2 : 5) k_sym_block(int64_t nrows, const int32_t* __restrict__ rows, SymCtx c, int64_t* __restrict__ nnz_row,
                            const int64_t* __restrict__ cptr, int32_t* __restrict__ cidx, uint16_t* __restrict__ cmap,
                            int jbits, HRec hr) {
    constexpr int S = 1 << LOGS;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    // layout: keys[S] | maps[S] | list u64[S/2] (step 2) ; pair-search scratch in static smem
    int* keys = reinterpret_cast<int*>(smem_raw);
    uint32_t* maps = reinterpret_cast<uint32_t*>(keys + S);
    unsigned long long* list = reinterpret_cast<unsigned long long*>(maps + S);
    __shared__ int64_t sh_excl[512], sh_b0[512], sh_tot[17], sh_aux[512];
    __shared__ uint32_t sh_ma[512];
    __shared__ int sh_cnt[17];
    const int tid = threadIdx.x, nt = blockDim.x, lane = tid & 31, w = tid >> 5, nw = nt >> 5;
    for (int64_t rr = blockIdx.x; rr < nrows; rr += gridDim.x) {
        const int64_t I = rows[rr];
        for (int i = tid; i < S; i += nt) {
            keys[i] = EMPTY_KEY;
            maps[i] = 0;
        }
        __syncthreads();
        int64_t r0 = 0, r1 = 0;
        if (STEP == 2 && LOGS <= 12 && hr.rec) {
            r0 = hr.hoff[I];
            r1 = hr.hoff[I + 1];
        }
        int cnt = 0;
        if (STEP == 2 && r1 > r0) {  // block-uniform: records {hash slot, B tile, A tile, product} (R34)
            block_pairs_aux(
                c, c.aptr[I], c.aptr[I + 1], sh_excl, sh_b0, sh_ma, sh_tot, sh_aux,
                [&](int64_t, int32_t, int64_t pos0) { return r0 + pos0; },
                [&](int32_t J, uint32_t mc, int64_t t, int64_t j, int64_t pos) {
                    const int h = hash_insert_at(keys, maps, LOGS, J, mc);
                    hr.rec[pos] = make_int4(h, (int)j, (int)t, (int)mc);
                });
        } else {
            block_pairs(c, I, sh_excl, sh_b0, sh_ma, sh_tot,
                        [&](int32_t J, uint32_t mc) { cnt += hash_insert(keys, maps, LOGS, J, mc, STEP == 2); });
        }
        __syncthreads();
        if (STEP == 1) {
#pragma unroll
            for (int d = 16; d; d >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, d);
            if (lane == 0) sh_cnt[w] = cnt;
            __syncthreads();
            if (tid == 0) {
                int s = 0;
                for (int k = 0; k < nw; ++k) s += sh_cnt[k];
                nnz_row[I] = s;
            }
            __syncthreads();
            continue;
        }
        if constexpr (LOGS <= 12) {
            // sort the whole table as packed keys (J << 16 | map; empty slots = ~0 sort last)
            // with a block radix sort over J's bits: no compress pass, ~nbits/4 passes instead
            // of the log^2 N stages of a bitonic network (Alg. 3 line 14)
            constexpr int THREADS = LOGS >= 12 ? 512 : 256;
            constexpr int IPT = S / THREADS;
            using Sorter = cub::BlockRadixSort<unsigned long long, THREADS, IPT, int>;  // value: hash slot
            __shared__ typename Sorter::TempStorage rs_tmp;
            unsigned long long kv[IPT];
            int sv[IPT];
            int nv = 0;
#pragma unroll
            for (int u = 0; u < IPT; ++u) {
                const int slot = tid * IPT + u;
                const int k = keys[slot];
                nv += k != EMPTY_KEY;
                kv[u] = k != EMPTY_KEY ? (((unsigned long long)(uint32_t)k << 16) | (maps[slot] & 0xFFFFu)) : ~0ull;
                sv[u] = slot;
            }
#pragma unroll
            for (int d = 16; d; d >>= 1) nv += __shfl_xor_sync(0xffffffffu, nv, d);
            if (lane == 0) sh_cnt[w] = nv;
            __syncthreads();  // keys/maps read into registers; sh_cnt complete
            int n = 0;
            for (int q = 0; q < nw; ++q) n += sh_cnt[q];
            Sorter(rs_tmp).Sort(kv, sv, 16, 17 + jbits);  // one bit above J: empty slots (~0) last
            const int64_t out = cptr[I];
#pragma unroll
            for (int u = 0; u < IPT; ++u) {
                const int pos = tid * IPT + u;
                if (pos < n) {
                    cidx[out + pos] = (int32_t)(kv[u] >> 16);
                    cmap[out + pos] = (uint16_t)(kv[u] & 0xFFFFu);
                    if (r1 > r0) keys[sv[u]] = pos;  // slot -> rank (keys were read before the sort)
                }
            }
            __syncthreads();
            if (r1 > r0) {  // the row's records get their C tiles
                if (tid == 0) hr.rowf[I] = 1;
                for (int64_t pb = r0 + tid; pb < r1; pb += 4 * (int64_t)nt) {  // four records per thread in flight
                    int hv[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u)
                        hv[u] = pb + (int64_t)nt * u < r1 ? reinterpret_cast<const int*>(hr.rec + pb + (int64_t)nt * u)[0] : -1;
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        if (hv[u] < 0) continue;
                        const int64_t q = out + keys[hv[u]];
                        reinterpret_cast<int*>(hr.rec + pb + (int64_t)nt * u)[0] = (int)q;
                        atomicAdd(hr.cnt + q, 1u);
                    }
                }
                __syncthreads();
            }
            continue;
        }
        // compress into list (packed key<<16 | map), block-wide ballot prefix per round
        int n = 0;
        for (int base = 0; base < S; base += nt) {
            const int k = keys[base + tid];
            const bool v = k != EMPTY_KEY;
            const uint32_t bal = __ballot_sync(0xffffffffu, v);
            if (lane == 0) sh_cnt[w] = __popc(bal);
            __syncthreads();
            if (tid == 0) {
                int s = 0;
                for (int q = 0; q < nw; ++q) { const int x = sh_cnt[q]; sh_cnt[q] = s; s += x; }
                sh_cnt[nw] = s;
            }
            __syncthreads();
            if (v) {
                const int pos = n + sh_cnt[w] + __popc(bal & ((1u << lane) - 1u));
                list[pos] = ((unsigned long long)(uint32_t)k << 16) | (maps[base + tid] & 0xFFFFu);
            }
            n += sh_cnt[nw];
            __syncthreads();
        }
        int N = 1;
        while (N < n) N <<= 1;
        for (int i = n + tid; i < N; i += nt) list[i] = ~0ull;
        __syncthreads();
        for (int k = 2; k <= N; k <<= 1)  // bitonic sort, ascending
            for (int j = k >> 1; j > 0; j >>= 1) {
                for (int i = tid; i < N; i += nt) {
                    const int ixj = i ^ j;
                    if (ixj > i) {
                        const unsigned long long a = list[i], b = list[ixj];
                        const bool up = (i & k) == 0;
                        if ((a > b) == up) { list[i] = b; list[ixj] = a; }
                    }
                }
                __syncthreads();
            }
        const int64_t out = cptr[I];
        for (int i = tid; i < n; i += nt) {
            const unsigned long long e = list[i];
            cidx[out + i] = (int32_t)(e >> 16);
            cmap[out + i] = (uint16_t)(e & 0xFFFFu);
        }
        __syncthreads();
    }
}

// ---------------------------------------------------------------- step kernels: bin 7 (dense bitmap)
template <int STEP>
__global__ void __launch_bounds__(512) k_sym_dense(int64_t nrows, const int32_t* __restrict__ rows, SymCtx c,
                                                   int64_t W, uint32_t* __restrict__ gws, int64_t* __restrict__ nnz_row,
                                                   const int64_t* __restrict__ cptr, int32_t* __restrict__ cidx,
                                                   uint16_t* __restrict__ cmap) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ int64_t sh_excl[512], sh_b0[512], sh_tot[17];
    __shared__ uint32_t sh_ma[512];
    __shared__ long long sh_sum[17];
    uint32_t* bm;
    uint32_t* pre;
    if (gws) {
        bm = gws + (int64_t)blockIdx.x * 2 * W;
        pre = bm + W;
    } else {
        bm = reinterpret_cast<uint32_t*>(smem_raw);
        pre = bm + W;
    }
    const int tid = threadIdx.x, nt = blockDim.x, lane = tid & 31, w = tid >> 5, nw = nt >> 5;
    for (int64_t rr = blockIdx.x; rr < nrows; rr += gridDim.x) {
        const int64_t I = rows[rr];
        for (int64_t i = tid; i < W; i += nt) bm[i] = 0;
        __syncthreads();
        block_pairs(c, I, sh_excl, sh_b0, sh_ma, sh_tot,
                    [&](int32_t J, uint32_t) { atomicOr(bm + (J >> 5), 1u << (J & 31)); });
        __syncthreads();
        // per-thread contiguous word ranges -> block scan of popcounts
        const int64_t per = (W + nt - 1) / nt;
        const int64_t w0 = min(W, per * (int64_t)tid), w1 = min(W, w0 + per);
        long long s = 0;
        for (int64_t i = w0; i < w1; ++i) s += __popc(bm[i]);
        long long incl = s;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const long long y = __shfl_up_sync(0xffffffffu, incl, d);
            if (lane >= d) incl += y;
        }
        if (lane == 31) sh_sum[w] = incl;
        __syncthreads();
        if (tid == 0) {
            long long a = 0;
            for (int k = 0; k < nw; ++k) { const long long x = sh_sum[k]; sh_sum[k] = a; a += x; }
            sh_sum[nw] = a;
        }
        __syncthreads();
        if (STEP == 1) {
            if (tid == 0) nnz_row[I] = sh_sum[nw];
            __syncthreads();
            continue;
        }
        long long run = sh_sum[w] + incl - s;
        const int64_t out = cptr[I];
        for (int64_t i = w0; i < w1; ++i) {
            pre[i] = (uint32_t)run;
            uint32_t bits = bm[i];
            while (bits) {
                const int b = __ffs(bits) - 1;
                bits &= bits - 1;
                cidx[out + run] = (int32_t)(32 * i + b);
                ++run;
            }
        }
        __syncthreads();
        block_pairs(c, I, sh_excl, sh_b0, sh_ma, sh_tot, [&](int32_t J, uint32_t mc) {
            const int64_t q = out + pre[J >> 5] + __popc(bm[J >> 5] & ((1u << (J & 31)) - 1u));
            atomicOr(reinterpret_cast<unsigned int*>(cmap) + (q >> 1), mc << (16 * (q & 1)));
        });
        __syncthreads();
    }
}

// ---------------------------------------------------------------- dense rows, whole-GPU form
// Same bitmap idea as k_sym_dense, with the row bitmaps in global memory (W words per dense
// row) so that one row is spread over many CTAs: work items are (row, GD_CH consecutive A
// tiles), each expanded by block_pairs_range.  Step 1 ORs the bit of every candidate column
// J into its row's bitmap; k_gdense_count turns each bitmap into per-word exclusive prefix
// counts and the row's distinct count (Alg. 3 lines 9-12); step 2 writes the columns in word
// order (sorted by construction, line 14) and ORs each pair's bitmap product into its C tile
// at rank(J) = prefix(word) + popcount of the lower bits (R15).  No per-row serial walk: the
// 107K-pair rows of config 4 take ~400 items instead of one CTA.
constexpr int GD_CH = 256;  // A tiles per work item (= the block size: one block_pairs round)

__global__ void k_gdense_items(int64_t nd, const int32_t* __restrict__ rows, const int64_t* __restrict__ aptr,
                               int64_t* __restrict__ nitem) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nd; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t I = rows[i];
        nitem[i] = (aptr[I + 1] - aptr[I] + GD_CH - 1) / GD_CH;
    }
}

__global__ void k_gdense_item_rows(int64_t nd, const int64_t* __restrict__ ioff, int32_t* __restrict__ item_row) {
    for (int64_t i = blockIdx.x; i < nd; i += gridDim.x)
        for (int64_t k = ioff[i] + threadIdx.x; k < ioff[i + 1]; k += blockDim.x) item_row[k] = (int32_t)i;
}

// Numeric plan records written by step 2 (band-major positions, see SpgemmPlan below).
struct PlanRec {
    const int64_t* pp;    // [TA+1] global pair prefix over A tiles
    const int64_t* tl;    // [nd][nb+1] pair index of the row's first tile in band b
    const int64_t* ioffB; // [nb*nd+1] band-major offsets of the (band, row) items
    int64_t nd, BW;
    int nb;
    int4* rec;      // {C tile q, B tile j, A tile t, bitmap product}; q = -1: empty product
    uint32_t* cnt;  // [TC] products per C tile
};

// Deterministic multi-product tiles (R34): the multi tiles are numbered in C order
// (mi = prefix of popcount(mflag) words + rank in the word); k_plan_mlist lists their C tile
// and product count, a scan gives each its slot range, and k_plan_slots rewrites every record of
// a multi tile to -(slot + 2) — the numeric pass writes those products to their slots and
// k_plan_msum adds each tile's products in ascending A-tile order (the pair order of Alg. 4), so
// the sum no longer depends on scheduling.
__global__ void k_plan_wpop(int64_t nw, const uint32_t* __restrict__ mflag, int64_t* __restrict__ wpop) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nw; i += (int64_t)gridDim.x * blockDim.x)
        wpop[i] = __popc(mflag[i]);
}
__device__ __forceinline__ int64_t multi_index(const uint32_t* mflag, const int64_t* mwpre, int64_t q) {
    return mwpre[q >> 5] + __popc(mflag[q >> 5] & ((1u << (q & 31)) - 1u));
}
__global__ void k_plan_mlist(int64_t TC, const uint32_t* __restrict__ mflag, const int64_t* __restrict__ mwpre,
                             const uint32_t* __restrict__ cnt, int32_t* __restrict__ mq, int64_t* __restrict__ mcnt) {
    const int64_t nw = (TC + 31) / 32;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nw; i += (int64_t)gridDim.x * blockDim.x) {
        uint32_t f = mflag[i];
        int64_t mi = mwpre[i];
        while (f) {
            const int b = __ffs(f) - 1;
            f &= f - 1;
            const int64_t q = 32 * i + b;
            mq[mi] = (int32_t)q;
            mcnt[mi] = cnt[q];
            ++mi;
        }
    }
}
__global__ void k_plan_slots(int64_t n, int4* __restrict__ rec, const uint32_t* __restrict__ mflag,
                             const int64_t* __restrict__ mwpre, const int64_t* __restrict__ moff,
                             uint32_t* __restrict__ mfill) {
    for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < n; p += (int64_t)gridDim.x * blockDim.x) {
        const int q = reinterpret_cast<const int*>(rec + p)[0];
        if (q < 0 || !((mflag[q >> 5] >> (q & 31)) & 1u)) continue;
        const int64_t mi = multi_index(mflag, mwpre, q);
        const int64_t slot = moff[mi] + atomicAdd(mfill + mi, 1u);
        reinterpret_cast<int*>(rec + p)[0] = (int)(-(slot + 2));
    }
}

// mflag bit q <- C tile q takes more than one product
__global__ void k_plan_mark(int64_t TC, const uint32_t* __restrict__ cnt, uint32_t* __restrict__ mflag) {
    const int64_t nw = (TC + 31) / 32;
    const int lane = threadIdx.x & 31;
    for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < 32 * nw; q += (int64_t)gridDim.x * blockDim.x) {
        const bool m = q < TC && cnt[q] > 1u;
        const unsigned b = __ballot_sync(0xffffffffu, m);
        if (lane == 0) mflag[q >> 5] = b;
    }
}

template <int STEP>
__global__ void __launch_bounds__(GD_CH) k_gdense_pairs(const int64_t* __restrict__ nitems_dev,
                                                      const int32_t* __restrict__ item_row,
                                                      const int64_t* __restrict__ ioff, const int32_t* __restrict__ rows,
                                                      SymCtx c, int64_t W, uint32_t* __restrict__ gbm,
                                                      const uint32_t* __restrict__ gpre, const int64_t* __restrict__ cptr,
                                                      uint32_t* __restrict__ cmap32, PlanRec pr,
                                                      unsigned long long* __restrict__ npairs) {
    __shared__ int64_t sh_excl[GD_CH], sh_b0[GD_CH], sh_tot[GD_CH / 32 + 1], sh_aux[GD_CH];
    __shared__ uint32_t sh_ma[GD_CH];
    const int64_t nitems = *nitems_dev;
    for (int64_t item = blockIdx.x; item < nitems; item += gridDim.x) {
        const int64_t li = item_row[item];
        const int64_t I = rows[li];
        const int64_t a0 = c.aptr[I] + (item - ioff[li]) * GD_CH;
        const int64_t a1 = min(c.aptr[I + 1], a0 + GD_CH);
        uint32_t* bm = gbm + li * W;
        if (STEP == 1) {
            if (npairs) {  // the item's (A tile, B tile) pairs: the plan's record count
                const int64_t t = a0 + threadIdx.x;
                unsigned long long len = 0;
                if (t < a1) {
                    const int32_t K = c.aidx[t];
                    len = (unsigned long long)(c.bptr[K + 1] - c.bptr[K]);
                }
#pragma unroll
                for (int d = 16; d; d >>= 1) len += __shfl_xor_sync(0xffffffffu, len, d);
                if ((threadIdx.x & 31) == 0 && len) atomicAdd(npairs, len);
            }
            block_pairs_range(c, a0, a1, sh_excl, sh_b0, sh_ma, sh_tot,
                              [&](int32_t J, uint32_t) { atomicOr(bm + (J >> 5), 1u << (J & 31)); });
        } else {
            const uint32_t* pre = gpre + li * W;
            const int64_t c0 = cptr[I];
            auto rank = [&](int32_t J) {
                const int wd = J >> 5;
                return c0 + pre[wd] + __popc(bm[wd] & ((1u << (J & 31)) - 1u));
            };
            if (pr.rec) {
                const int64_t* tlr = pr.tl + li * (pr.nb + 1);
                block_pairs_aux(
                    c, a0, a1, sh_excl, sh_b0, sh_ma, sh_tot, sh_aux,
                    [&](int64_t t, int32_t K, int64_t) {
                        const int b = (int)(K / pr.BW);
                        return pr.ioffB[(int64_t)b * pr.nd + li] + (pr.pp[t] - tlr[b]);
                    },
                    [&](int32_t J, uint32_t mc, int64_t t, int64_t j, int64_t pos) {
                        const int64_t q = rank(J);
                        atomicOr(cmap32 + (q >> 1), mc << (16 * (q & 1)));
                        atomicAdd(pr.cnt + q, 1u);  // products per C tile (k_plan_mark)
                        pr.rec[pos] = make_int4((int)q, (int)j, (int)t, (int)mc);
                    });
            } else {
                block_pairs_range(c, a0, a1, sh_excl, sh_b0, sh_ma, sh_tot, [&](int32_t J, uint32_t mc) {
                    const int64_t q = rank(J);
                    atomicOr(cmap32 + (q >> 1), mc << (16 * (q & 1)));
                });
            }
        }
    }
}

// per dense row: exclusive prefix popcount per bitmap word (gpre) and the distinct count
constexpr int GD_CNT_THREADS = 512;
__global__ void __launch_bounds__(GD_CNT_THREADS) k_gdense_count(int64_t nd, const int32_t* __restrict__ rows, int64_t W,
                                                                 const uint32_t* __restrict__ gbm,
                                                                 uint32_t* __restrict__ gpre, int64_t* __restrict__ nnz_row) {
    __shared__ uint32_t sh[GD_CNT_THREADS / 32 + 1];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    constexpr int NW = GD_CNT_THREADS / 32;
    for (int64_t li = blockIdx.x; li < nd; li += gridDim.x) {
        const uint32_t* bm = gbm + li * W;
        uint32_t* pre = gpre + li * W;
        uint32_t run = 0;
        // four consecutive words per thread per round (one 16-B load when W is a multiple of 4)
        for (int64_t base = 0; base < W; base += 4 * GD_CNT_THREADS) {
            const int64_t i = base + 4 * tid;
            uint32_t wv[4];
            if ((W & 3) == 0 && i + 3 < W) {
                const uint4 q4 = *reinterpret_cast<const uint4*>(bm + i);
                wv[0] = q4.x; wv[1] = q4.y; wv[2] = q4.z; wv[3] = q4.w;
            } else {
#pragma unroll
                for (int u = 0; u < 4; ++u) wv[u] = i + u < W ? bm[i + u] : 0u;
            }
            uint32_t pc[4], v = 0;
#pragma unroll
            for (int u = 0; u < 4; ++u) { pc[u] = (uint32_t)__popc(wv[u]); v += pc[u]; }
            uint32_t incl = v;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t y = __shfl_up_sync(0xffffffffu, incl, d);
                if (lane >= d) incl += y;
            }
            if (lane == 31) sh[w] = incl;
            __syncthreads();
            if (w == 0) {
                const uint32_t x = lane < NW ? sh[lane] : 0u;
                uint32_t xi = x;
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {
                    const uint32_t y = __shfl_up_sync(0xffffffffu, xi, d);
                    if (lane >= d) xi += y;
                }
                if (lane < NW) sh[lane] = xi - x;
                if (lane == NW - 1) sh[NW] = xi;
            }
            __syncthreads();
            uint32_t ex = run + sh[w] + incl - v;
            if ((W & 3) == 0 && i + 3 < W) {
                uint4 o;
                o.x = ex; ex += pc[0];
                o.y = ex; ex += pc[1];
                o.z = ex; ex += pc[2];
                o.w = ex;
                *reinterpret_cast<uint4*>(pre + i) = o;
            } else {
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    if (i + u < W) pre[i + u] = ex;
                    ex += pc[u];
                }
            }
            run += sh[NW];
            __syncthreads();
        }
        if (tid == 0) nnz_row[rows[li]] = run;
    }
}

// step 2 columns: every set bit of word i of dense row li goes to cptr + gpre + its rank
__global__ void k_gdense_out(int64_t nd, const int32_t* __restrict__ rows, int64_t W, const uint32_t* __restrict__ gbm,
                             const uint32_t* __restrict__ gpre, const int64_t* __restrict__ cptr,
                             int32_t* __restrict__ cidx) {
    // four consecutive words of one row per thread (W a multiple of 4), else one
    const int64_t n = nd * W;
    const int V = (W & 3) == 0 ? 4 : 1;
    for (int64_t g = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * V; g < n;
         g += (int64_t)gridDim.x * blockDim.x * V) {
        uint32_t wv[4] = {0u, 0u, 0u, 0u}, pv[4] = {0u, 0u, 0u, 0u};
        if (V == 4) {
            const uint4 b4 = *reinterpret_cast<const uint4*>(gbm + g);
            if ((b4.x | b4.y | b4.z | b4.w) == 0u) continue;
            const uint4 p4 = *reinterpret_cast<const uint4*>(gpre + g);
            wv[0] = b4.x; wv[1] = b4.y; wv[2] = b4.z; wv[3] = b4.w;
            pv[0] = p4.x; pv[1] = p4.y; pv[2] = p4.z; pv[3] = p4.w;
        } else {
            wv[0] = gbm[g];
            if (!wv[0]) continue;
            pv[0] = gpre[g];
        }
        const int64_t li = g / W, wd0 = g - li * W;
        const int64_t c0 = cptr[rows[li]];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            uint32_t bits = wv[u];
            int64_t q = c0 + pv[u];
            while (bits) {
                const int b = __ffs(bits) - 1;
                bits &= bits - 1;
                cidx[q++] = (int32_t)(32 * (wd0 + u) + b);
            }
        }
    }
}

__global__ void k_numeric_rows_stats(int64_t BR, const int64_t* __restrict__ cptr, unsigned long long* __restrict__ out) {
    unsigned long long a = 0, b = 0, e = 0;
    for (int64_t I = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; I < BR; I += (int64_t)gridDim.x * blockDim.x) {
        const int64_t n = cptr[I + 1] - cptr[I];
        if (n == 0) ++e; else if (n <= 32) ++a; else ++b;
    }
    for (int d = 16; d; d >>= 1) {
        a += __shfl_xor_sync(0xffffffffu, a, d);
        b += __shfl_xor_sync(0xffffffffu, b, d);
        e += __shfl_xor_sync(0xffffffffu, e, d);
    }
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(out, a);
        atomicAdd(out + 1, b);
        atomicAdd(out + 2, e);
    }
}

// ---------------------------------------------------------------- numeric
template <typename T> struct TileIO;
template <> struct TileIO<double> {
    static __device__ __forceinline__ void load(const double* p, double (&v)[16]) {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const double2 d = __ldg(reinterpret_cast<const double2*>(p) + i);
            v[2 * i] = d.x;
            v[2 * i + 1] = d.y;
        }
    }
};
template <> struct TileIO<float> {
    static __device__ __forceinline__ void load(const float* p, float (&v)[16]) {
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const float4 d = __ldg(reinterpret_cast<const float4*>(p) + i);
            v[4 * i] = d.x; v[4 * i + 1] = d.y; v[4 * i + 2] = d.z; v[4 * i + 3] = d.w;
        }
    }
};
template <> struct TileIO<__half> {
    static __device__ __forceinline__ void load(const __half* p, float (&v)[16]) {
#pragma unroll
        for (int i = 0; i < 2; ++i) {
            const uint4 u = __ldg(reinterpret_cast<const uint4*>(p) + i);
            const uint32_t w[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const float2 f = __half22float2(*reinterpret_cast<const __half2*>(&w[k]));
                v[8 * i + 2 * k] = f.x;
                v[8 * i + 2 * k + 1] = f.y;
            }
        }
    }
};

template <typename T> struct RowIO;
template <> struct RowIO<double> {
    static __device__ __forceinline__ void load(const double* p, double (&v)[4]) {
        const double2 a = __ldg(reinterpret_cast<const double2*>(p));
        const double2 b = __ldg(reinterpret_cast<const double2*>(p) + 1);
        v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
    }
    static __device__ __forceinline__ void store(double* p, const double (&v)[4]) {
        reinterpret_cast<double2*>(p)[0] = make_double2(v[0], v[1]);
        reinterpret_cast<double2*>(p)[1] = make_double2(v[2], v[3]);
    }
};
template <> struct RowIO<float> {
    static __device__ __forceinline__ void load(const float* p, float (&v)[4]) {
        const float4 a = __ldg(reinterpret_cast<const float4*>(p));
        v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
    }
    static __device__ __forceinline__ void store(float* p, const float (&v)[4]) {
        *reinterpret_cast<float4*>(p) = make_float4(v[0], v[1], v[2], v[3]);
    }
};
template <> struct RowIO<__half> {
    static __device__ __forceinline__ void load(const __half* p, float (&v)[4]) {
        const uint2 u = __ldg(reinterpret_cast<const uint2*>(p));
        const float2 lo = __half22float2(*reinterpret_cast<const __half2*>(&u.x));
        const float2 hi = __half22float2(*reinterpret_cast<const __half2*>(&u.y));
        v[0] = lo.x; v[1] = lo.y; v[2] = hi.x; v[3] = hi.y;
    }
    static __device__ __forceinline__ void store(__half* p, const float (&v)[4]) {
        __half2 a = __floats2half2_rn(v[0], v[1]), b = __floats2half2_rn(v[2], v[3]);
        uint2 u;
        u.x = *reinterpret_cast<uint32_t*>(&a);
        u.y = *reinterpret_cast<uint32_t*>(&b);
        *reinterpret_cast<uint2*>(p) = u;
    }
};

template <typename Acc, typename T> __device__ __forceinline__ Acc to_acc(T v) { return (Acc)v; }
template <> __device__ __forceinline__ float to_acc<float, __half>(__half v) { return __half2float(v); }
__device__ __forceinline__ double fma_acc(double a, double b, double c) { return fma(a, b, c); }
__device__ __forceinline__ float fma_acc(float a, float b, float c) { return fmaf(a, b, c); }

// C tile += A tile * B tile on CUDA cores (64 FMAs, fixed order k = 0..3).
template <typename Acc>
__device__ __forceinline__ void tile_mma(const Acc (&a)[16], const Acc (&b)[16], Acc (&c)[16]) {
#pragma unroll
    for (int r = 0; r < 4; ++r)
#pragma unroll
        for (int col = 0; col < 4; ++col) {
            Acc s = a[4 * r] * b[col];
            s = fma(a[4 * r + 1], b[4 + col], s);
            s = fma(a[4 * r + 2], b[8 + col], s);
            s = fma(a[4 * r + 3], b[12 + col], s);
            c[4 * r + col] = s;
        }
}

__device__ __forceinline__ int bsearch_row(const int32_t* idx, int n, int32_t J) {
    int lo = 0, hi = n - 1;
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (idx[mid] < J) lo = mid + 1; else hi = mid;
    }
    return lo;
}

constexpr int NUM_WARPS = 4;
constexpr int CAP = 32;  // C tiles per row accumulated in shared memory

template <typename Acc> struct NumSmem {
    Acc acc[CAP][17];  // C tiles of the row; padded: lanes adding different tiles spread over banks
    int32_t cidx[CAP];
};

// DMMA m8n8k4 FP64 (sm_80+ DMMA; native DMMA.8x8x4 on sm_100a).
__device__ __forceinline__ void dmma(double& c0, double& c1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};"
                 : "+d"(c0), "+d"(c1)
                 : "d"(a), "d"(b));
}

// T = storage type, Acc = accumulation type (double for FP64, float otherwise).
// gacc: FP32 accumulation workspace for FP16 global-path rows (indexed like C values).
template <typename T, typename Acc>
__device__ __forceinline__ void numeric_warp_row(int64_t I, const SymCtx& c, const T* __restrict__ aval,
                                                 const T* __restrict__ bval, const int64_t* __restrict__ cptr,
                                                 const int32_t* __restrict__ cidx_g,
                                                 const uint16_t* __restrict__ cmap_g, T* __restrict__ cval,
                                                 Acc* __restrict__ gacc, int tc_thr, NumSmem<Acc>& S, int lane) {
    const int64_t c0 = cptr[I];
    const int nC = (int)(cptr[I + 1] - c0);
    if (nC == 0) return;
    const int64_t a0 = c.aptr[I], a1 = c.aptr[I + 1];
    // nC <= CAP (longer rows go to the mid/long-row kernels): shared-memory accumulators
    if (lane < nC) S.cidx[lane] = cidx_g[c0 + lane];
    for (int e = lane; e < nC * 16; e += 32) S.acc[e >> 4][e & 15] = Acc(0);
    __syncwarp();
    const int32_t* rowidx = S.cidx;
    auto accp = [&](int q) -> Acc* { return S.acc[q]; };

    // ---- tensor-core route (FP64 only): A tiles with POPCOUNT >= tc_thr, one at a time.
    if constexpr (sizeof(T) == 8) {
        for (int64_t base = a0; base < a1; base += 32) {
            const int64_t t = base + lane;
            const uint32_t ma = t < a1 ? c.amap[t] : 0u;
            uint32_t dense = __ballot_sync(0xffffffffu, t < a1 && __popc(ma) >= tc_thr);
            while (dense) {
                const int src = __ffs(dense) - 1;
                dense &= dense - 1;
                const int64_t ta = base + src;
                const uint32_t mA = __shfl_sync(0xffffffffu, ma, src);
                const int32_t K = c.aidx[ta];
                // fragA[row][k] = A[row & 3][k]: lane l -> element (l>>2 & 3, l&3)
                const double fa = (double)aval[16 * ta + 4 * ((lane >> 2) & 3) + (lane & 3)];
                const int64_t b0 = c.bptr[K], b1 = c.bptr[K + 1];
                for (int64_t jb = b0; jb < b1; jb += 32) {
                    const int64_t j = jb + lane;
                    const uint32_t mb = j < b1 ? c.bmap[j] : 0u;
                    const uint32_t mc = j < b1 ? bitmap_multiply(mA, mb) : 0u;
                    const int q = mc ? bsearch_row(rowidx, nC, c.bidx[j]) : -1;
                    uint32_t valid = __ballot_sync(0xffffffffu, mc != 0);
                    while (valid) {
                        const int l1 = __ffs(valid) - 1;
                        valid &= valid - 1;
                        int l2 = -1;
                        if (valid) { l2 = __ffs(valid) - 1; valid &= valid - 1; }
                        const int q1 = __shfl_sync(0xffffffffu, q, l1);
                        const int q2 = __shfl_sync(0xffffffffu, q, l2 < 0 ? l1 : l2);
                        // fragB[k][n]: lane l -> (k = l&3, n = l>>2); n<4 -> B_j1[k][n], else B_j2[k][n-4]
                        const int n8 = lane >> 2, k4 = lane & 3;
                        double fb = 0.0;
                        if (n8 < 4) fb = (double)bval[16 * (jb + l1) + 4 * k4 + n8];
                        else if (l2 >= 0) fb = (double)bval[16 * (jb + l2) + 4 * k4 + (n8 - 4)];
                        double d0 = 0.0, d1 = 0.0;
                        dmma(d0, d1, fa, fb);
                        // C[g][2t..2t+1] in lane 4g+t; quadrant (0:4,0:4) -> tile q1, (4:8,4:8) -> q2
                        if (n8 < 4 && k4 < 2) {
                            Acc* p = accp(q1) + 4 * n8 + 2 * k4;
                            p[0] += d0;
                            p[1] += d1;
                        } else if (n8 >= 4 && k4 >= 2 && l2 >= 0) {
                            Acc* p = accp(q2) + 4 * (n8 - 4) + 2 * (k4 - 2);
                            p[0] += d0;
                            p[1] += d1;
                        }
                        __syncwarp();
                    }
                }
            }
        }
    }

    // ---- CUDA-core route: pairs of the remaining A tiles.
    const int thr = (sizeof(T) == 8) ? tc_thr : 17;
    {
        // flattened pairs: one lane per (A tile, B tile) pair, products staged per lane
        for (int64_t base = a0; base < a1; base += 32) {
            const int64_t t = base + lane;
            const bool v = t < a1;
            const uint32_t ma = v ? c.amap[t] : 0u;
            const bool sp = v && __popc(ma) < thr;
            const int32_t K = sp ? c.aidx[t] : 0;
            const int64_t b0 = sp ? c.bptr[K] : 0;
            const int64_t len = sp ? c.bptr[K + 1] - b0 : 0;
            int64_t incl = len;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const int64_t y = __shfl_up_sync(0xffffffffu, incl, d);
                if (lane >= d) incl += y;
            }
            const int64_t excl = incl - len;
            const int64_t total = __shfl_sync(0xffffffffu, incl, 31);
            for (int64_t p0 = 0; p0 < total; p0 += 32) {
                const int64_t p = p0 + lane;
                int lo = 0;
#pragma unroll
                for (int step = 16; step; step >>= 1) {
                    const int cand = lo + step;
                    const int64_t e = __shfl_sync(0xffffffffu, excl, cand & 31);
                    if (cand < 32 && e <= p) lo = cand;
                }
                const int64_t ob0 = __shfl_sync(0xffffffffu, b0, lo);
                const int64_t oex = __shfl_sync(0xffffffffu, excl, lo);
                const uint32_t oma = __shfl_sync(0xffffffffu, ma, lo);
                const int64_t ot = base + lo;
                int q = -1;
                Acc pr[16];
                if (p < total) {
                    const int64_t j = ob0 + (p - oex);
                    const uint32_t mc = bitmap_multiply(oma, c.bmap[j]);
                    if (mc) {
                        q = bsearch_row(rowidx, nC, c.bidx[j]);
                        Acc bv[16];
                        TileIO<T>::load(bval + 16 * j, bv);
                        const T* ap = aval + 16 * ot;
#pragma unroll
                        for (int r = 0; r < 4; ++r) {  // the product in registers (tile_mma order)
                            Acc ar[4];
                            RowIO<T>::load(ap + 4 * r, ar);
#pragma unroll
                            for (int col = 0; col < 4; ++col) {
                                Acc sv = ar[0] * bv[col];
                                sv = fma(ar[1], bv[4 + col], sv);
                                sv = fma(ar[2], bv[8 + col], sv);
                                sv = fma(ar[3], bv[12 + col], sv);
                                pr[4 * r + col] = sv;
                            }
                        }
                    }
                }
                // accumulate in lane order per C tile (deterministic): the k-th lane of a group
                // of lanes with the same tile adds in round k, so lanes of different tiles add
                // concurrently (usually one to three rounds instead of 32 serial steps)
                const unsigned peers = __match_any_sync(0xffffffffu, q);
                const int rank = __popc(peers & ((1u << lane) - 1u));
                const int rmax = (int)__reduce_max_sync(0xffffffffu, q >= 0 ? (unsigned)rank : 0u);
                for (int k = 0; k <= rmax; ++k) {
                    if (q >= 0 && rank == k) {
#pragma unroll
                        for (int x = 0; x < 16; ++x) S.acc[q][x] += pr[x];
                    }
                    __syncwarp();
                }
            }
        }
    }
    __syncwarp();
    // ---- write out, +0.0 where the bitmap bit is clear (R2)
    for (int64_t e = lane; e < 16 * (int64_t)nC; e += 32) {
        const int q = (int)(e >> 4), b = (int)(e & 15);
        const bool bit = (cmap_g[c0 + q] >> b) & 1u;
        const Acc v = S.acc[q][b];
        cval[16 * c0 + e] = bit ? from_acc<T>(v) : from_acc<T>(Acc(0));
    }
}

// Warp per C block row for the rows in `rows` (count read from the device: the rows the
// group kernel could not take, nC > GROUP_NC).  Persistent grid-stride over the list.
template <typename T, typename Acc>
__global__ void __launch_bounds__(NUM_WARPS * 32) k_numeric(const int32_t* __restrict__ rows,
                                                            const unsigned long long* __restrict__ nrows_dev, SymCtx c,
                                                            const T* __restrict__ aval, const T* __restrict__ bval,
                                                            const int64_t* __restrict__ cptr,
                                                            const int32_t* __restrict__ cidx_g,
                                                            const uint16_t* __restrict__ cmap_g, T* __restrict__ cval,
                                                            Acc* __restrict__ gacc, int tc_thr) {
    __shared__ NumSmem<Acc> sm[NUM_WARPS];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t nrows = (int64_t)*nrows_dev;
    for (int64_t wi = (int64_t)blockIdx.x * NUM_WARPS + w; wi < nrows; wi += (int64_t)gridDim.x * NUM_WARPS) {
        numeric_warp_row<T, Acc>(rows[wi], c, aval, bval, cptr, cidx_g, cmap_g, cval, gacc, tc_thr, sm[w], lane);
        __syncwarp();
    }
}

// ---------------------------------------------------------------- numeric: long rows
// C block rows with more than CAP tiles (power-law rows of config 4): one CTA per row.  The
// row's C tile columns are copied to shared memory (when <= LONG_SMEM tiles) for the
// position search; the row's pairs are flattened across the CTA (no serialisation over A
// tiles).  Dense A tiles (POPCOUNT >= threshold, FP64) go to DMMA m8n8k4 exactly as Alg. 4:
// fragA = [A;A], fragB = [B_j | B_j'], two quadrants kept; warps take the dense tiles
// round-robin.  Accumulation: FP64/FP32 atomics into the output (FP32 workspace for FP16),
// only at the bitmap positions a product can touch — the order of additions is not fixed,
// so these rows are reproducible up to rounding (exact on integer/dyadic data).
constexpr int LONG_SMEM = 8192;

// last i with idx[i] <= J (idx ascending, idx[0] <= J)
__device__ __forceinline__ int bsearch_le(const int32_t* idx, int n, int32_t J) {
    int lo = 0, hi = n - 1;
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (idx[mid] <= J) lo = mid; else hi = mid - 1;
    }
    return lo;
}
// warp-cooperative: largest i in [lo, hi] with key(i) <= x (key nondecreasing, key(lo) <= x);
// each round the 32 lanes probe 32 evenly spaced candidates
template <typename F>
__device__ __forceinline__ int64_t warp_search_le(int64_t lo, int64_t hi, int64_t x, F key, int lane) {
    while (hi > lo) {
        const int64_t step = (hi - lo + 31) / 32;
        const int64_t pos = lo + (int64_t)(lane + 1) * step;
        const bool ok = pos <= hi && key(pos) <= x;
        const int cnt = __popc(__ballot_sync(0xffffffffu, ok));
        lo += cnt * step;
        hi = min(hi, lo + step - 1);
    }
    return lo;
}

constexpr int LONG_PAIRS = 2048;  // (A tile, B tile) pairs per work item of a long row
constexpr int LONG_CTILES = 512;  // C tiles per finalising work item of a long row

// pairs per A tile of the long rows (the other entries were zeroed)
__global__ void k_long_plen(const int32_t* __restrict__ rows, const unsigned long long* __restrict__ nrows_dev,
                            SymCtx c, int64_t* __restrict__ plen) {
    const int64_t n = (int64_t)*nrows_dev;
    const int lane = threadIdx.x & 31;
    for (int64_t wi = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; wi < n;
         wi += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int64_t I = rows[wi];
        for (int64_t t = c.aptr[I] + lane; t < c.aptr[I + 1]; t += 32) {
            const int32_t K = c.aidx[t];  // an empty B row still counts one (void) pair, so a
            plen[t] = max(c.bptr[K + 1] - c.bptr[K], (int64_t)1);  // chunk spans <= LONG_PAIRS + 1 A tiles
        }
    }
}

// work items per long row: ceil(pairs / LONG_PAIRS) (entries past the device-side count are 0)
__global__ void k_long_prep(int64_t cap, const int32_t* __restrict__ rows, const unsigned long long* __restrict__ nrows_dev,
                            const int64_t* __restrict__ aptr, const int64_t* __restrict__ pp,
                            int64_t* __restrict__ nch) {
    const int64_t n = (int64_t)*nrows_dev;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cap; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t c = 0;
        if (i < n) {
            const int64_t I = rows[i];
            c = (pp[aptr[I + 1]] - pp[aptr[I]] + LONG_PAIRS - 1) / LONG_PAIRS;
        }
        nch[i] = c;
    }
}


__global__ void k_long_prep_c(int64_t cap, const int32_t* __restrict__ rows, const unsigned long long* __restrict__ nrows_dev,
                              const int64_t* __restrict__ cptr, int64_t* __restrict__ nch) {
    const int64_t n = (int64_t)*nrows_dev;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < cap; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t c = 0;
        if (i < n) {
            const int64_t I = rows[i];
            c = (cptr[I + 1] - cptr[I] + LONG_CTILES - 1) / LONG_CTILES;
        }
        nch[i] = c;
    }
}

// FP16 rows accumulated with atomics: round the FP32 workspace, +0.0 where the bit is
// clear; work items = (row, 512-C-tile chunk) over a persistent grid
template <typename T, typename Acc>
__global__ void k_long_rows_finalize(const int32_t* __restrict__ rows, const unsigned long long* __restrict__ nrows_dev,
                                     const int64_t* __restrict__ choff, int64_t cap, const int64_t* __restrict__ cptr,
                                     const uint16_t* __restrict__ cmap, T* __restrict__ cval, const Acc* __restrict__ gacc) {
    const int64_t nrows = (int64_t)*nrows_dev;
    const int64_t nitems = choff[cap];
    for (int64_t item = blockIdx.x; item < nitems; item += gridDim.x) {
        int64_t lo = 0, hi = nrows - 1;
        while (lo < hi) {
            const int64_t mid = (lo + hi + 1) >> 1;
            if (choff[mid] <= item) lo = mid; else hi = mid - 1;
        }
        const int64_t I = rows[lo];
        const int64_t c0 = cptr[I], q0 = c0 + (item - choff[lo]) * LONG_CTILES;
        const int64_t q1 = min(cptr[I + 1], q0 + LONG_CTILES);
        for (int64_t e = 16 * q0 + threadIdx.x; e < 16 * q1; e += blockDim.x) {
            const bool bit = (cmap[e >> 4] >> (e & 15)) & 1u;
            cval[e] = bit ? from_acc<T>(gacc[e]) : from_acc<T>(Acc(0));
        }
    }
}

// Pair records written by pass 0 when the long rows' pair count fits their capacity: per
// global pair index P, the C tile (global index, -1 if the product is empty), B tile, A
// tile and bitmap product — pass 1 then streams them (k_long_flat) with no searches.
struct PairRec {
    int32_t* q;
    int32_t* j;
    int32_t* t;
    uint16_t* m;
    int64_t cap;
};

template <typename T, typename Acc, int PASS>
__global__ void __launch_bounds__(256) k_numeric_long(const int32_t* __restrict__ rows,
                                                      const unsigned long long* __restrict__ nrows_dev,
                                                      const int64_t* __restrict__ choff, int64_t cap,
                                                      const int64_t* __restrict__ pp, const int64_t* __restrict__ pp_total,
                                                      unsigned long long* __restrict__ next, int32_t* __restrict__ cnt,
                                                      PairRec rec, SymCtx c, const T* __restrict__ aval,
                                                      const T* __restrict__ bval, const int64_t* __restrict__ cptr,
                                                      const int32_t* __restrict__ cidx_g, T* __restrict__ cval,
                                                      Acc* __restrict__ gacc) {
    extern __shared__ __align__(16) int32_t sidx[];
    __shared__ int32_t sh_pp[LONG_PAIRS + 2];  // pair prefix of the chunk's A tiles, relative to P0
    __shared__ int64_t sh_d[6];
    const int tid = threadIdx.x, nt = blockDim.x, lane = tid & 31, w = tid >> 5;
    const int hl = tid & 15, hsh = tid & 16;
    const int64_t nrows = (int64_t)*nrows_dev;
    const int64_t nitems = choff[cap];
    const bool records = *pp_total <= rec.cap;
    if (PASS == 1 && records) return;  // k_long_flat streams the records instead
    Acc* stg = reinterpret_cast<Acc*>(sidx + LONG_SMEM) + w * (32 * 16);
    for (;;) {
        // item descriptor (warp 0): dequeue, then 32-ary searches for the row and for the
        // chunk's A tiles (a few dependent loads instead of ~log2 n)
        if (w == 0) {
            int64_t item = 0;
            if (lane == 0) item = (int64_t)atomicAdd(next, 1ull);
            item = __shfl_sync(0xffffffffu, item, 0);
            if (lane == 0) sh_d[0] = item;
            if (item < nitems) {
                const int64_t li = warp_search_le(0, nrows - 1, item, [&](int64_t m) { return choff[m]; }, lane);
                const int64_t I = rows[li];
                const int64_t ta0 = c.aptr[I], ta1 = c.aptr[I + 1];
                const int64_t P0 = pp[ta0] + (item - choff[li]) * LONG_PAIRS, P1 = min(pp[ta1], P0 + LONG_PAIRS);
                auto key = [&](int64_t m) { return pp[m]; };
                const int64_t a0 = warp_search_le(ta0, ta1 - 1, P0, key, lane);
                const int64_t a1 = warp_search_le(a0, ta1 - 1, P1 - 1, key, lane) + 1;
                if (lane == 0) { sh_d[1] = I; sh_d[2] = a0; sh_d[3] = a1; sh_d[4] = P0; sh_d[5] = P1; }
            }
        }
        __syncthreads();
        if (sh_d[0] >= nitems) break;
        const int64_t I = sh_d[1], a0 = sh_d[2], a1 = sh_d[3], P0 = sh_d[4], P1 = sh_d[5];
        const int64_t c0 = cptr[I];
        const int nC = (int)(cptr[I + 1] - c0);
        Acc* acc = gacc ? gacc + 16 * c0 : reinterpret_cast<Acc*>(cval + 16 * c0);
        int32_t* rcnt = cnt + c0;
        // position search: every S-th C tile column in shared memory (S = 1 when the row
        // fits), then a short forward scan over the global column list
        const int S = (nC + LONG_SMEM - 1) / LONG_SMEM, ns = (nC + S - 1) / S;
        for (int q = tid; q < ns; q += nt) sidx[q] = cidx_g[c0 + (int64_t)q * S];
        const int na = (int)(a1 - a0);
        for (int i = tid; i <= na; i += nt) sh_pp[i] = (int32_t)(pp[a0 + i] - P0);
        __syncthreads();
        auto find_q = [&](int32_t J) {
            int q = bsearch_le(sidx, ns, J) * S;
            if (S > 1) {
                const int e1 = min(nC, q + S);
                while (q + 1 < e1 && cidx_g[c0 + q] != J) ++q;
            }
            return q;
        };
        auto tile_of = [&](int64_t P) {  // last chunk A tile i with pp[a0 + i] <= P
            const int32_t x = (int32_t)(P - P0);
            int l = 0, h = na - 1;
            while (l < h) {
                const int m = (l + h + 1) >> 1;
                if (sh_pp[m] <= x) l = m; else h = m - 1;
            }
            return l;
        };
        // ---- one pair per thread per round.  Pass 0: count the products per C tile, zero
        // the tiles that will take REDs (a second product) and write the pair records.
        // Pass 1 (no records): the B tile and the A rows in registers, every load in flight
        // at once; each warp stages its 32 tile products in shared memory and writes them
        // with 16-lane coalesced accesses, two products per instruction — a plain store
        // (+0.0 at the clear bits) into a tile with one product, REDs at the bitmap
        // positions otherwise.
        for (int64_t pb = P0; pb < P1; pb += nt) {
            const int64_t p = pb + tid;
            uint32_t mc = 0u;
            int q = 0;
            if (p < P1) {
                const int i = tile_of(p);
                const int64_t t = a0 + i;
                const uint32_t ma = c.amap[t];
                const int32_t K = c.aidx[t];
                const int64_t j = c.bptr[K] + (p - P0 - sh_pp[i]);
                if (j < c.bptr[K + 1]) {
                    mc = bitmap_multiply(ma, c.bmap[j]);
                    if (mc) {
                        q = find_q(c.bidx[j]);
                        if constexpr (PASS == 0) {
                            const int old = atomicAdd(rcnt + q, 1);
                            if (old == 1) {
                                uint4* v = reinterpret_cast<uint4*>(acc + 16 * (int64_t)q);
#pragma unroll
                                for (int e = 0; e < (int)sizeof(Acc); ++e) v[e] = make_uint4(0u, 0u, 0u, 0u);
                            }
                            if (records) {
                                rec.j[p] = (int32_t)j;
                                rec.t[p] = (int32_t)t;
                                rec.m[p] = (uint16_t)mc;
                            }
                        } else {
                            Acc bv[16];
                            TileIO<T>::load(bval + 16 * j, bv);
#pragma unroll
                            for (int r = 0; r < 4; ++r) {
                                Acc ar[4];
                                RowIO<T>::load(aval + 16 * t + 4 * r, ar);
#pragma unroll
                                for (int col = 0; col < 4; ++col) {
                                    Acc s = ar[0] * bv[col];
                                    s = fma_acc(ar[1], bv[4 + col], s);
                                    s = fma_acc(ar[2], bv[8 + col], s);
                                    s = fma_acc(ar[3], bv[12 + col], s);
                                    stg[lane * 16 + 4 * r + col] = s;
                                }
                            }
                        }
                    }
                }
                if (PASS == 0 && records) rec.q[p] = mc ? (int32_t)(c0 + q) : -1;
            }
            if constexpr (PASS == 1) {
                int single = 0;
                if (mc) single = rcnt[q] == 1;
                __syncwarp();
                uint32_t todo = __ballot_sync(0xffffffffu, mc != 0u);
                while (todo) {
                    const int s1 = __ffs(todo) - 1;
                    todo &= todo - 1;
                    const int s2 = todo ? __ffs(todo) - 1 : -1;
                    if (todo) todo &= todo - 1;
                    const int src = hsh ? s2 : s1;
                    const int sl = src < 0 ? s1 : src;
                    const uint32_t ms = __shfl_sync(0xffffffffu, mc, sl);
                    const int qs = __shfl_sync(0xffffffffu, q, sl);
                    const int one = __shfl_sync(0xffffffffu, single, sl);
                    if (src >= 0) {
                        const bool bit = (ms >> hl) & 1u;
                        const Acc val = stg[src * 16 + hl];
                        Acc* dst = acc + 16 * (int64_t)qs + hl;
                        if (one) *dst = bit ? val : Acc(0);
                        else if (bit) atomicAdd(dst, val);
                    }
                }
                __syncwarp();
            }
        }
        __syncthreads();  // sidx / sh_pp / sh_d are rewritten by the next item
    }
}

// Pass 1 over the pair records: a half-warp per record, lane e = 4r+c computing entry
// (r,c) of the tile product (A row r, B column c), FLAT_U records per half-warp in flight;
// the tile is written with one coalesced 16-lane access — a plain store (+0.0 at the clear
// bits) into a single-product tile, REDs at the bitmap positions otherwise.
constexpr int FLAT_U = 4;

template <typename T, typename Acc>
__global__ void __launch_bounds__(256, 4) k_long_flat(const int64_t* __restrict__ pp_total, PairRec rec,
                                                   const int32_t* __restrict__ cnt, const T* __restrict__ aval,
                                                   const T* __restrict__ bval, T* __restrict__ cval,
                                                   Acc* __restrict__ gacc) {
    const int64_t total = *pp_total;
    if (total > rec.cap) return;  // no records: the item kernel's pass 1 ran
    const int hl = threadIdx.x & 15, er = hl >> 2, ec = hl & 3;
    Acc* acc = gacc ? gacc : reinterpret_cast<Acc*>(cval);
    const int64_t hw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 4;
    const int64_t nhw = ((int64_t)gridDim.x * blockDim.x) >> 4;
    for (int64_t base = hw * FLAT_U; base < total; base += nhw * FLAT_U) {
        int32_t q[FLAT_U];
        int64_t t[FLAT_U], j[FLAT_U];
        uint32_t m[FLAT_U];
#pragma unroll
        for (int u = 0; u < FLAT_U; ++u) {
            const int64_t p = base + u;
            q[u] = p < total ? __ldg(rec.q + p) : -1;
            j[u] = q[u] >= 0 ? __ldg(rec.j + p) : 0;
            t[u] = q[u] >= 0 ? __ldg(rec.t + p) : 0;
            m[u] = q[u] >= 0 ? __ldg(rec.m + p) : 0u;
        }
        Acc bc[FLAT_U][4];
        int one[FLAT_U];
#pragma unroll
        for (int u = 0; u < FLAT_U; ++u) {
#pragma unroll
            for (int k = 0; k < 4; ++k) bc[u][k] = q[u] >= 0 ? to_acc<Acc>(bval[16 * j[u] + 4 * k + ec]) : Acc(0);
            one[u] = q[u] >= 0 ? cnt[q[u]] == 1 : 0;
        }
#pragma unroll
        for (int u = 0; u < FLAT_U; ++u) {
            if (q[u] < 0) continue;
            Acc ar[4];
            RowIO<T>::load(aval + 16 * t[u] + 4 * er, ar);
            Acc sv = ar[0] * bc[u][0];
            sv = fma_acc(ar[1], bc[u][1], sv);
            sv = fma_acc(ar[2], bc[u][2], sv);
            sv = fma_acc(ar[3], bc[u][3], sv);
            const bool bit = (m[u] >> hl) & 1u;
            Acc* dst = acc + 16 * (int64_t)q[u] + hl;
            if (one[u]) *dst = bit ? sv : Acc(0);
            else if (bit) atomicAdd(dst, sv);
        }
    }
}

// ---------------------------------------------------------------- numeric: mid rows
// C block rows with CAP < nC <= MIDCAP tiles (most long rows of power-law matrices): one
// warp per row, rows dequeued dynamically, no CTA barriers.  Two passes over the row's
// pairs (one pair per lane per round): pass 0 counts the products landing on each C tile
// (shared-memory atomics); pass 1 computes them, stages each warp's 32 tile products in
// shared memory and writes them with 16-lane coalesced accesses — a plain store (+0.0 at
// the clear bits) for a tile with one product, REDs at the bitmap positions into a
// zeroed tile otherwise.  On power-law rows almost every C tile has one product, so the
// row is written once, without atomics.  CUDA cores only.
constexpr int MIDCAP = 512;
constexpr int MID_WARPS = 8;

template <typename T, typename Acc>
__global__ void __launch_bounds__(MID_WARPS * 32) k_numeric_mid(const int32_t* __restrict__ rows,
                                                                const unsigned long long* __restrict__ nrows_dev,
                                                                unsigned long long* __restrict__ cursor, SymCtx c,
                                                                const T* __restrict__ aval, const T* __restrict__ bval,
                                                                const int64_t* __restrict__ cptr,
                                                                const int32_t* __restrict__ cidx_g, T* __restrict__ cval,
                                                                Acc* __restrict__ gacc) {
    extern __shared__ __align__(16) unsigned char mid_smem[];  // per warp: staging, columns, counts
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, hl = lane & 15, hsh = lane & 16;
    const int64_t nrows = (int64_t)*nrows_dev;
    Acc* stg = reinterpret_cast<Acc*>(mid_smem) + w * (32 * 16);
    int32_t* sidx = reinterpret_cast<int32_t*>(mid_smem + MID_WARPS * 32 * 16 * sizeof(Acc)) + w * (2 * MIDCAP);
    int32_t* scnt = sidx + MIDCAP;
    for (;;) {
        int64_t wi = 0;
        if (lane == 0) wi = (int64_t)atomicAdd(cursor, 1ull);
        wi = __shfl_sync(0xffffffffu, wi, 0);
        if (wi >= nrows) break;
        const int64_t I = rows[wi], c0 = cptr[I];
        const int nC = (int)(cptr[I + 1] - c0);
        for (int q = lane; q < nC; q += 32) {
            sidx[q] = cidx_g[c0 + q];
            scnt[q] = 0;
        }
        __syncwarp();
        Acc* acc = gacc ? gacc + 16 * c0 : reinterpret_cast<Acc*>(cval + 16 * c0);
        const int64_t a0 = c.aptr[I], a1 = c.aptr[I + 1];
        for (int pass = 0; pass < 2; ++pass) {
            if (pass == 1) {  // zero the tiles that take several products
                for (int q = lane; q < nC; q += 32)
                    if (scnt[q] > 1) {
                        uint4* v = reinterpret_cast<uint4*>(acc + 16 * q);
#pragma unroll
                        for (int e = 0; e < (int)sizeof(Acc); ++e) v[e] = make_uint4(0u, 0u, 0u, 0u);
                    }
                __threadfence();
                __syncwarp();
            }
            for (int64_t base = a0; base < a1; base += 32) {
                const int64_t t = base + lane;
                const bool v = t < a1;
                const int32_t K = v ? c.aidx[t] : 0;
                const uint32_t ma = v ? c.amap[t] : 0u;
                const int64_t b0 = v ? c.bptr[K] : 0;
                const int64_t len = v ? c.bptr[K + 1] - b0 : 0;
                int64_t incl = len;
#pragma unroll
                for (int d = 1; d < 32; d <<= 1) {
                    const int64_t y = __shfl_up_sync(0xffffffffu, incl, d);
                    if (lane >= d) incl += y;
                }
                const int64_t excl = incl - len;
                const int64_t total = __shfl_sync(0xffffffffu, incl, 31);
                for (int64_t p0 = 0; p0 < total; p0 += 32) {
                    const int64_t p = p0 + lane;
                    int lo = 0;  // owner lane: last with excl <= p
#pragma unroll
                    for (int step = 16; step; step >>= 1) {
                        const int cand = lo + step;
                        const int64_t e = __shfl_sync(0xffffffffu, excl, cand & 31);
                        if (cand < 32 && e <= p) lo = cand;
                    }
                    const int64_t ob0 = __shfl_sync(0xffffffffu, b0, lo);
                    const int64_t oex = __shfl_sync(0xffffffffu, excl, lo);
                    const uint32_t oma = __shfl_sync(0xffffffffu, ma, lo);
                    uint32_t mc = 0u;
                    int q = 0;
                    if (p < total) {
                        const int64_t j = ob0 + (p - oex);
                        mc = bitmap_multiply(oma, c.bmap[j]);
                        if (mc) {
                            q = bsearch_row(sidx, nC, c.bidx[j]);
                            if (pass == 0) {
                                atomicAdd(scnt + q, 1);
                            } else {
                                Acc bv[16];
                                TileIO<T>::load(bval + 16 * j, bv);
                                const T* ap = aval + 16 * (base + lo);
#pragma unroll
                                for (int r = 0; r < 4; ++r) {
                                    Acc ar[4];
                                    RowIO<T>::load(ap + 4 * r, ar);
#pragma unroll
                                    for (int col = 0; col < 4; ++col) {
                                        Acc s = ar[0] * bv[col];
                                        s = fma_acc(ar[1], bv[4 + col], s);
                                        s = fma_acc(ar[2], bv[8 + col], s);
                                        s = fma_acc(ar[3], bv[12 + col], s);
                                        stg[lane * 16 + 4 * r + col] = s;
                                    }
                                }
                            }
                        }
                    }
                    if (pass == 0) continue;
                    __syncwarp();
                    uint32_t todo = __ballot_sync(0xffffffffu, mc != 0u);
                    while (todo) {  // two staged products per instruction
                        const int s1 = __ffs(todo) - 1;
                        todo &= todo - 1;
                        const int s2 = todo ? __ffs(todo) - 1 : -1;
                        if (todo) todo &= todo - 1;
                        const int src = hsh ? s2 : s1;
                        const uint32_t ms = __shfl_sync(0xffffffffu, mc, src < 0 ? s1 : src);
                        const int qs = __shfl_sync(0xffffffffu, q, src < 0 ? s1 : src);
                        if (src >= 0) {
                            const bool bit = (ms >> hl) & 1u;
                            const Acc val = stg[src * 16 + hl];
                            Acc* dst = acc + 16 * (int64_t)qs + hl;
                            if (scnt[qs] == 1) *dst = bit ? val : Acc(0);
                            else if (bit) atomicAdd(dst, val);
                        }
                    }
                    __syncwarp();
                }
            }
            __syncwarp();
        }
    }
}

// ---------------------------------------------------------------- numeric: group kernel
// One 4-lane group per C block row with <= GROUP_NC tiles, 8 rows per warp.  Lane r owns
// row r of every C tile of its row (accumulators in registers).  The group walks its
// (A tile, B tile) pairs in order (A tiles ascending, B tiles ascending): deterministic,
// no conflicts.  Warp-synchronous rounds (one pair per group per round) let the groups
// whose pair has a dense A tile (POPCOUNT >= tc_thr, FP64) share DMMA m8n8k4 instructions
// two at a time: fragA = [A_a; A_b], fragB = [B_a | B_b], and the diagonal quadrants of
// fragC are A_a B_a and A_b B_b (L157-171; the paper pairs two B tiles of one A tile, we
// pair two groups' tile products — same instruction, same "keep half" extraction).
// Rows with more tiles are appended to `big` for k_numeric.
constexpr int GROUP_NC = 8;


template <typename T, typename Acc>
__global__ void __launch_bounds__(256) k_numeric_group(int64_t BR, SymCtx c, const T* __restrict__ aval,
                                                       const T* __restrict__ bval, const int64_t* __restrict__ cptr,
                                                       const int32_t* __restrict__ cidx_g,
                                                       const uint16_t* __restrict__ cmap_g, T* __restrict__ cval,
                                                       int32_t* __restrict__ big, unsigned long long* __restrict__ nbig,
                                                       int32_t* __restrict__ lng, unsigned long long* __restrict__ nlng,
                                                       int32_t* __restrict__ mid, unsigned long long* __restrict__ nmid,
                                                       int tc_thr) {
    const int lane = threadIdx.x & 31, g = lane >> 2, r = lane & 3;
    const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (wid * 8 >= BR) return;
    const int64_t I = wid * 8 + g;
    int64_t c0 = 0;
    int nC = 0;
    if (I < BR) {
        c0 = cptr[I];
        nC = (int)(cptr[I + 1] - c0);
        if (nC > GROUP_NC) {  // <= CAP: warp kernel (deterministic); longer: block kernel
            if (r == 0) {
                if (nC <= CAP) big[atomicAdd(nbig, 1ull)] = (int32_t)I;
                else if (nC <= MIDCAP) mid[atomicAdd(nmid, 1ull)] = (int32_t)I;
                else lng[atomicAdd(nlng, 1ull)] = (int32_t)I;
            }
            nC = 0;
        }
    }
    int32_t cid[GROUP_NC];
#pragma unroll
    for (int k = 0; k < GROUP_NC; ++k) cid[k] = k < nC ? cidx_g[c0 + k] : INT_MAX;
    Acc acc[GROUP_NC][4];
#pragma unroll
    for (int k = 0; k < GROUP_NC; ++k)
#pragma unroll
        for (int e = 0; e < 4; ++e) acc[k][e] = Acc(0);
    // pair cursor
    int64_t t = 0, a1 = 0, j = 0, jend = 0;
    uint32_t mA = 0;
    Acc arow[4] = {Acc(0), Acc(0), Acc(0), Acc(0)};
    if (nC > 0) {
        t = c.aptr[I];
        a1 = c.aptr[I + 1];
    }
    // A-tile metadata cache: lane u of the group holds (bitmap, B-row range) of tile cbase + u,
    // loaded four tiles at a time (parallel loads) instead of one dependent chain per tile.
    const unsigned gm = 0xFu << (lane & ~3);
    int64_t cbase = INT64_MIN, cb0 = 0, cb1 = 0;
    uint32_t cma = 0;
    auto load_chunk = [&](int64_t base) {
        cbase = base;
        const int64_t tt = base + r;
        cb0 = cb1 = 0;
        cma = 0;
        if (tt < a1) {
            const int32_t K = c.aidx[tt];
            cma = c.amap[tt];
            cb0 = c.bptr[K];
            cb1 = c.bptr[K + 1];
        }
    };
    auto next_a = [&]() {  // move to the next A tile with a non-empty B row (group-uniform)
        while (t < a1) {
            if (t >= cbase + 4) load_chunk(t);
            const int u = (int)(t - cbase);
            j = __shfl_sync(gm, cb0, u, 4);
            jend = __shfl_sync(gm, cb1, u, 4);
            const uint32_t m = __shfl_sync(gm, cma, u, 4);
            if (j < jend) {
                mA = m;
                RowIO<T>::load(aval + 16 * t + 4 * r, arow);
                return;
            }
            ++t;
        }
    };
    next_a();
    for (;;) {
        const bool has = t < a1;
        if (!__any_sync(0xffffffffu, has)) break;
        uint32_t mC = 0;
        int q = 0;
        if (has) {
            mC = bitmap_multiply(mA, c.bmap[j]);
            if (mC) {
                const int32_t J = c.bidx[j];
#pragma unroll
                for (int k = 0; k < GROUP_NC; ++k) q = (cid[k] == J) ? k : q;
            }
        }
        bool dense = false;
        if constexpr (sizeof(T) == 8 || sizeof(T) == 2) dense = mC != 0 && __popc(mA) >= tc_thr;
        if (mC && !dense) {  // CUDA-core route: lane r computes row r of A_t * B_j
            Acc b0[4], b1[4], b2[4], b3[4], v[4];
            const T* bp = bval + 16 * j;
            RowIO<T>::load(bp, b0);
            RowIO<T>::load(bp + 4, b1);
            RowIO<T>::load(bp + 8, b2);
            RowIO<T>::load(bp + 12, b3);
#pragma unroll
            for (int e = 0; e < 4; ++e) {
                Acc s_ = arow[0] * b0[e];
                s_ = fma(arow[1], b1[e], s_);
                s_ = fma(arow[2], b2[e], s_);
                s_ = fma(arow[3], b3[e], s_);
                v[e] = s_;
            }
#pragma unroll
            for (int k = 0; k < GROUP_NC; ++k)
                if (k == q)
#pragma unroll
                    for (int e = 0; e < 4; ++e) acc[k][e] += v[e];
        }
        if constexpr (sizeof(T) == 8) {
            uint32_t dm = __ballot_sync(0xffffffffu, dense && r == 0);
            while (dm) {  // tensor-core route, two groups per DMMA
                const int ga = (__ffs(dm) - 1) >> 2;
                dm &= dm - 1;
                int gb = -1;
                if (dm) { gb = (__ffs(dm) - 1) >> 2; dm &= dm - 1; }
                const int row8 = lane >> 2, k4 = lane & 3;
                const int64_t ta = __shfl_sync(0xffffffffu, t, 4 * ga);
                const int64_t ja = __shfl_sync(0xffffffffu, j, 4 * ga);
                const int64_t tb = __shfl_sync(0xffffffffu, t, 4 * (gb < 0 ? ga : gb));
                const int64_t jb = __shfl_sync(0xffffffffu, j, 4 * (gb < 0 ? ga : gb));
                double fa = 0.0, fb = 0.0;
                if (row8 < 4) {
                    fa = (double)aval[16 * ta + 4 * row8 + k4];
                    fb = (double)bval[16 * ja + 4 * k4 + row8];
                } else if (gb >= 0) {
                    fa = (double)aval[16 * tb + 4 * (row8 - 4) + k4];
                    fb = (double)bval[16 * jb + 4 * k4 + (row8 - 4)];
                }
                double d0 = 0.0, d1 = 0.0;
                dmma(d0, d1, fa, fb);
                // C_a row r: lanes (r, 0) and (r, 1); C_b row r: lanes (4+r, 2) and (4+r, 3)
                const bool isb = (g == gb);
                const int s0 = isb ? 4 * (4 + r) + 2 : 4 * r;
                const double x0 = __shfl_sync(0xffffffffu, d0, s0), x1 = __shfl_sync(0xffffffffu, d1, s0);
                const double x2 = __shfl_sync(0xffffffffu, d0, s0 + 1), x3 = __shfl_sync(0xffffffffu, d1, s0 + 1);
                if (g == ga || isb) {
#pragma unroll
                    for (int k = 0; k < GROUP_NC; ++k)
                        if (k == q) {
                            acc[k][0] += x0; acc[k][1] += x1; acc[k][2] += x2; acc[k][3] += x3;
                        }
                }
            }
        }
        if constexpr (sizeof(T) == 2) {
            // tensor-core route for FP16 (FP32 accumulation): HMMA m16n8k8 with
            //   A16x8 = rows 0-3 [A0|0], 4-7 [0|A1], 8-11 [A2|0], 12-15 [0|A3]
            //   B8x8  = [[B0|B2],[B1|B3]]
            // gives A0B0 (rows 0-3, cols 0-3), A1B1 (4-7, 0-3), A2B2 (8-11, 4-7), A3B3 (12-15, 4-7):
            // four groups' tile products per instruction.
            uint32_t dm = __ballot_sync(0xffffffffu, mC != 0 && __popc(mA) >= tc_thr && r == 0);
            // groups that took this route must skip the CUDA-core update above: handled by
            // `hdense` below (the CUDA-core block ran only for !hdense groups).
            while (dm) {
                int gs[4];
                int ns = 0;
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    gs[k] = -1;
                    if (dm) { gs[k] = (__ffs(dm) - 1) >> 2; dm &= dm - 1; ++ns; }
                }
                const int gid = lane >> 2, tid = lane & 3;
                int64_t ts[4], js[4];
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const int src = 4 * (gs[k] < 0 ? gs[0] : gs[k]);
                    ts[k] = __shfl_sync(0xffffffffu, t, src);
                    js[k] = __shfl_sync(0xffffffffu, j, src);
                }
                const __half* ah = reinterpret_cast<const __half*>(aval);
                const __half* bh = reinterpret_cast<const __half*>(bval);
                uint32_t a01 = 0u, a23 = 0u, b01 = 0u;
                // a0,a1: row gid (slot 0 if gid<4 with tid<2; slot 1 if gid>=4 with tid>=2)
                const int sA = gid < 4 ? 0 : 1;
                const bool onA = (gid < 4) == (tid < 2);
                if (onA && gs[sA] >= 0)
                    a01 = __ldg(reinterpret_cast<const unsigned int*>(ah + 16 * ts[sA] + 4 * (gid & 3) + 2 * (tid & 1)));
                const int sA2 = gid < 4 ? 2 : 3;
                if (onA && gs[sA2] >= 0)
                    a23 = __ldg(reinterpret_cast<const unsigned int*>(ah + 16 * ts[sA2] + 4 * (gid & 3) + 2 * (tid & 1)));
                // b0,b1: rows 2tid, 2tid+1 of B8, column gid
                const int sB = (tid < 2 ? 0 : 1) + (gid < 4 ? 0 : 2);
                if (gs[sB] >= 0) {
                    const __half* bp = bh + 16 * js[sB] + 4 * (2 * (tid & 1)) + (gid & 3);
                    const __half2 bb = __halves2half2(bp[0], bp[4]);
                    b01 = *reinterpret_cast<const uint32_t*>(&bb);
                }
                float d0 = 0.f, d1 = 0.f, d2 = 0.f, d3 = 0.f;
                asm volatile(
                    "mma.sync.aligned.m16n8k8.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};"
                    : "+f"(d0), "+f"(d1), "+f"(d2), "+f"(d3)
                    : "r"(a01), "r"(a23), "r"(b01));
                // my slot (if my group took part) and the lanes holding row r of its product
                int slot = -1;
#pragma unroll
                for (int k = 0; k < 4; ++k) slot = (gs[k] == g) ? k : slot;
                const int base = ((slot & 1) ? 16 : 0) + 4 * r + ((slot & 2) ? 2 : 0);
                const int src = slot < 0 ? lane : base;
                const float u0 = __shfl_sync(0xffffffffu, d0, src), u1 = __shfl_sync(0xffffffffu, d1, src);
                const float u2 = __shfl_sync(0xffffffffu, d2, src), u3 = __shfl_sync(0xffffffffu, d3, src);
                const float w0 = __shfl_sync(0xffffffffu, d0, src + 1), w1 = __shfl_sync(0xffffffffu, d1, src + 1);
                const float w2 = __shfl_sync(0xffffffffu, d2, src + 1), w3 = __shfl_sync(0xffffffffu, d3, src + 1);
                if (slot >= 0) {
                    const bool hi = (slot & 2) != 0;
                    const float x0 = hi ? u2 : u0, x1 = hi ? u3 : u1, x2 = hi ? w2 : w0, x3 = hi ? w3 : w1;
#pragma unroll
                    for (int k = 0; k < GROUP_NC; ++k)
                        if (k == q) {
                            acc[k][0] += x0; acc[k][1] += x1; acc[k][2] += x2; acc[k][3] += x3;
                        }
                }
                (void)ns;
            }
        }
        if (has) {  // advance the cursor
            if (++j == jend) {
                ++t;
                next_a();
            }
        }
    }
    // write out: lane r writes row r of each tile, +0.0 where the bit is clear (R2)
#pragma unroll
    for (int k = 0; k < GROUP_NC; ++k) {
        if (k < nC) {
            const uint32_t nib = (cmap_g[c0 + k] >> (4 * r)) & 0xFu;
            Acc o[4];
#pragma unroll
            for (int e = 0; e < 4; ++e) o[e] = ((nib >> e) & 1u) ? acc[k][e] : Acc(0);
            if constexpr (sizeof(T) == 8)
                group_store_tile_f64((double*)(cval + 16 * (c0 + k)), o, r, 0xFu << (lane & ~3), lane & ~3);
            else
                RowIO<T>::store(cval + 16 * (c0 + k) + 4 * r, o);
        }
    }
}

// ---------------------------------------------------------------- staged group kernel
// The CUDA-core route of k_numeric_group restructured for memory-level parallelism (the
// default when the tensor-core route is off).  Same row class (<= GROUP_NC C tiles), same
// lane roles (lane r of the group accumulates row r of every C tile in registers), same
// pair order and arithmetic — results are bit-identical to k_numeric_group's CUDA-core
// route.  What changes is how operands arrive: the group takes its (A tile, B tile) pairs
// four at a time, lane u resolving pair u of the batch (owner A tile from the cached
// metadata of four A tiles, B position, bitmap and column), and the four lanes copy the
// batch's eight operand tiles into shared memory with cp.async (16-B pieces, independent,
// no registers held).  Two buffers: batch k+1 is resolved and its copies issued before
// batch k's products are formed from shared memory, and the A-tile metadata is fetched one
// chunk ahead, so a batch costs about one exposed memory round trip instead of four
// dependent ones per pair (ncu on k_numeric_group: 16 warps/SM, 0.27 eligible warps per
// scheduler, DRAM 23% of peak).
template <typename T> struct SRow;  // row / tile reads from shared memory
template <> struct SRow<double> {
    static __device__ __forceinline__ void load(const double* p, double (&v)[4]) {
        const double2 a = reinterpret_cast<const double2*>(p)[0], b = reinterpret_cast<const double2*>(p)[1];
        v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
    }
};
template <> struct SRow<float> {
    static __device__ __forceinline__ void load(const float* p, float (&v)[4]) {
        const float4 a = *reinterpret_cast<const float4*>(p);
        v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
    }
};
template <> struct SRow<__half> {
    static __device__ __forceinline__ void load(const __half* p, float (&v)[4]) {
        const uint2 u = *reinterpret_cast<const uint2*>(p);
        const float2 lo = __half22float2(*reinterpret_cast<const __half2*>(&u.x));
        const float2 hi = __half22float2(*reinterpret_cast<const __half2*>(&u.y));
        v[0] = lo.x; v[1] = lo.y; v[2] = hi.x; v[3] = hi.y;
    }
};

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sa), "l"(gmem) : "memory");
}

constexpr int STAGED_WARPS = 4;  // warps per CTA of k_numeric_staged
constexpr int STAGED_RPG = 4;    // consecutive block rows streamed by one 4-lane group

// The group streams STAGED_RPG consecutive block rows: their A tiles are one contiguous range,
// walked four tiles per chunk, so the batch pipeline runs across row boundaries and the
// per-row chain (C row pointers and columns, A row pointers) is loaded once for the four rows
// up front (lane u: row R0 + u).  A pair carries its row; when the pair being multiplied
// belongs to a new row, the group writes out the finished row's tiles and switches its
// column list (kept in shared memory).  Rows with more than GROUP_NC C tiles are listed for
// the warp / mid / long-row kernels and their A tiles contribute no pairs here.
// NC: C tiles per row held in registers (4 when the longest C row has <= 4 tiles: fewer
// registers, more resident warps), rows with more than GROUP_NC tiles go to the other kernels.
template <typename T, typename Acc, int NC, int NBUF>
__global__ void __launch_bounds__(STAGED_WARPS * 32) k_numeric_staged(
    int64_t BR, SymCtx c, const T* __restrict__ aval, const T* __restrict__ bval, const int64_t* __restrict__ cptr,
    const int32_t* __restrict__ cidx_g, const uint16_t* __restrict__ cmap_g, T* __restrict__ cval,
    int32_t* __restrict__ big, unsigned long long* __restrict__ nbig, int32_t* __restrict__ lng,
    unsigned long long* __restrict__ nlng, int32_t* __restrict__ mid, unsigned long long* __restrict__ nmid,
    int rpg, const uint8_t* __restrict__ skip) {
    constexpr int TE = 16;                       // elements per tile
    constexpr int PIECES = TE * sizeof(T) / 16;  // 16-B pieces per tile
    extern __shared__ __align__(16) unsigned char smem_raw[];
    __shared__ int32_t s_cid[STAGED_WARPS * 8][STAGED_RPG][GROUP_NC];
    __shared__ uint16_t s_cmap[STAGED_WARPS * 8][STAGED_RPG][GROUP_NC];
    const int lane = threadIdx.x & 31, g = lane >> 2, r = lane & 3;
    const int gi = (threadIdx.x >> 5) * 8 + g;  // group index in the CTA
    const unsigned gm = 0xFu << (lane & ~3);
    constexpr int GROUP_BUF = NBUF * 4 * 2 * TE;  // NBUF buffers x 4 pairs x (A tile, B tile)
    T* buf = reinterpret_cast<T*>(smem_raw) + (size_t)gi * GROUP_BUF;
    const int64_t wid = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    if (wid * 8 * rpg >= BR) return;
    const int64_t R0 = (wid * 8 + g) * rpg;
    // lane u < rpg: row R0 + u (C range, class; A range start)
    const int64_t Ir = R0 + r;
    int64_t rc0 = 0, ra0 = 0;
    int rnC = 0;
    if (r < rpg && Ir < BR) {
        rc0 = cptr[Ir];
        rnC = (int)(cptr[Ir + 1] - rc0);
        ra0 = c.aptr[Ir];
        if (skip && skip[Ir]) {
            rnC = 0;  // computed from the symbolic phase's records (SpgemmPlan)
        } else if (rnC > GROUP_NC) {
            if (rnC <= CAP) big[atomicAdd(nbig, 1ull)] = (int32_t)Ir;
            else if (rnC <= MIDCAP) mid[atomicAdd(nmid, 1ull)] = (int32_t)Ir;
            else lng[atomicAdd(nlng, 1ull)] = (int32_t)Ir;
            rnC = 0;  // not this kernel's row: its A tiles give no pairs here
        }
    }
    const int64_t last = min(R0 + rpg, BR);  // one past the group's last row
    const int64_t A1 = R0 < BR ? c.aptr[last] : 0;
#pragma unroll
    for (int k = 0; k < GROUP_NC; ++k) {
        s_cid[gi][r][k] = k < rnC ? cidx_g[rc0 + k] : INT_MAX;
        s_cmap[gi][r][k] = k < rnC ? cmap_g[rc0 + k] : (uint16_t)0;
    }
    // row starts / sizes of the four rows, in every lane of the group
    int64_t rs[STAGED_RPG];
    int rn[STAGED_RPG];
#pragma unroll
    for (int u = 0; u < STAGED_RPG; ++u) {
        rs[u] = __shfl_sync(gm, ra0, u, 4);
        rn[u] = __shfl_sync(gm, rnC, u, 4);
    }
    const int nrows = (int)max(last - R0, (int64_t)0);
    Acc acc[NC][4];
#pragma unroll
    for (int k = 0; k < NC; ++k)
#pragma unroll
        for (int e = 0; e < 4; ++e) acc[k][e] = Acc(0);
    int32_t cid[NC];
    int cur = -1;  // row (0..3) whose C tiles acc holds
    // A-tile chunk cache: lane u holds tile cbase+u (bitmap, B-row start, exclusive pair
    // offset, row); the next chunk's column / bitmap are prefetched one chunk ahead (pK, pma).
    int64_t cbase = 0, myb0 = 0;
    int myE = 0, S = 0, pos = 0, myrow = 0;
    uint32_t mycma = 0, pma = 0;
    int32_t pK = -1;
    auto prefetch = [&](int64_t base) {
        const int64_t tt = base + r;
        pK = -1;
        if (tt < A1) {
            pK = c.aidx[tt];
            pma = c.amap[tt];
        }
    };
    auto load_chunk = [&](int64_t base) {  // consumes the prefetched metadata of `base`
        cbase = base;
        const int64_t tt = base + r;
        int ri = 0;
#pragma unroll
        for (int u = 1; u < STAGED_RPG; ++u) ri += (u < nrows && rs[u] <= tt);
        int rnc = 0;
#pragma unroll
        for (int u = 0; u < STAGED_RPG; ++u) rnc = (u == ri) ? rn[u] : rnc;
        myrow = ri;
        int len = 0;
        myb0 = 0;
        mycma = 0;
        if (pK >= 0 && rnc > 0) {
            mycma = pma;
            myb0 = c.bptr[pK];
            len = (int)(c.bptr[pK + 1] - myb0);
        }
        int incl = len, y = __shfl_up_sync(gm, incl, 1, 4);
        if (r >= 1) incl += y;
        y = __shfl_up_sync(gm, incl, 2, 4);
        if (r >= 2) incl += y;
        myE = incl - len;
        S = __shfl_sync(gm, incl, 3, 4);
        pos = 0;
        prefetch(base + 4);
    };
    const int64_t A0 = nrows > 0 ? rs[0] : 0;
    prefetch(A0);
    load_chunk(A0);
    // Batch = the group's next 4 pairs: lane u resolves pair u (A tile, B tile, bitmap,
    // column, row; the bitmap/column loads stay in flight until the batch is computed) and
    // the group issues the cp.async copies of the 8 operand tiles into buffer `nb`.
    struct Batch {
        bool valid;
        uint32_t ma;
        int row;
    };
    // first chunk base >= b that lies in a row of this kernel: the A tiles of rows handed to the
    // other kernels (rn = 0; power-law rows of thousands of tiles) are jumped over, not walked
    auto skip_rows = [&](int64_t b) {
        for (;;) {
            if (b >= A1) return b;
            int ri = 0;
#pragma unroll
            for (int u = 1; u < STAGED_RPG; ++u) ri += (u < nrows && rs[u] <= b);
            int rnc = 0;
            int64_t nxt = A1;
#pragma unroll
            for (int u = 0; u < STAGED_RPG; ++u) {
                rnc = (u == ri) ? rn[u] : rnc;
                nxt = (u == ri + 1 && u < nrows) ? rs[u] : nxt;
            }
            if (rnc > 0) return b;
            b = nxt;
        }
    };
    auto issue = [&](int nb, Batch& B, uint32_t& bm, int32_t& bj) {
        while (pos >= S) {  // group-uniform
            const int64_t nbse = skip_rows(cbase + 4);
            if (nbse >= A1) break;
            if (nbse != cbase + 4) prefetch(nbse);
            load_chunk(nbse);
        }
        const bool has = pos < S;
        const int p = pos + r;
        B.valid = has && p < S;
        const int E1 = __shfl_sync(gm, myE, 1, 4), E2 = __shfl_sync(gm, myE, 2, 4), E3 = __shfl_sync(gm, myE, 3, 4);
        const int o = (p >= E1) + (p >= E2) + (p >= E3);
        const int64_t ob0 = __shfl_sync(gm, myb0, o, 4);
        const int oE = __shfl_sync(gm, myE, o, 4);
        B.ma = __shfl_sync(gm, mycma, o, 4);
        B.row = __shfl_sync(gm, myrow, o, 4);
        const int64_t tu = cbase + o;
        const int64_t ju = ob0 + (p - oE);
        bm = 0;
        bj = 0;
        if (B.valid) {
            bm = c.bmap[ju];
            bj = c.bidx[ju];
        }
        T* bb = buf + nb * (GROUP_BUF / NBUF);
#pragma unroll
        for (int v = 0; v < 4; ++v) {
            const int src = (lane & ~3) + v;
            const bool vv = __shfl_sync(0xffffffffu, B.valid, src);
            const int64_t tv = __shfl_sync(0xffffffffu, tu, src);
            const int64_t jv = __shfl_sync(0xffffffffu, ju, src);
            if (vv) {
#pragma unroll
                for (int k = r; k < 2 * PIECES; k += 4) {
                    const bool isB = k >= PIECES;
                    const int pc = isB ? k - PIECES : k;
                    const T* srcp = (isB ? bval + 16 * jv : aval + 16 * tv) + pc * (16 / sizeof(T));
                    cp_async16(bb + (v * 2 + (isB ? 1 : 0)) * TE + pc * (16 / sizeof(T)), srcp);
                }
            }
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
        if (has) pos += 4;
        return has;
    };
    // write row `row`'s tiles: lane r writes row r of each tile, +0.0 where the bit is clear (R2)
    auto flush = [&](int row) {
        int64_t c0 = 0;
        int nC = 0;
#pragma unroll
        for (int u = 0; u < STAGED_RPG; ++u) nC = (u == row) ? rn[u] : nC;
        c0 = __shfl_sync(gm, rc0, row, 4);
#pragma unroll
        for (int k = 0; k < NC; ++k) {
            if (k < nC) {
                const uint32_t nib = (s_cmap[gi][row][k] >> (4 * r)) & 0xFu;
                Acc o[4];
#pragma unroll
                for (int e = 0; e < 4; ++e) o[e] = ((nib >> e) & 1u) ? acc[k][e] : Acc(0);
                if constexpr (sizeof(T) == 8)
                    group_store_tile_f64((double*)(cval + 16 * (c0 + k)), o, r, gm, lane & ~3);
                else
                    RowIO<T>::store(cval + 16 * (c0 + k) + 4 * r, o);
            }
#pragma unroll
            for (int e = 0; e < 4; ++e) acc[k][e] = Acc(0);
        }
    };
    __syncwarp();  // s_cid / s_cmap written by the group's lanes
    Batch curb, nxtb;
    uint32_t cbm, nbm;
    int32_t cbj, nbj;
    bool chas = issue(0, curb, cbm, cbj);
    for (int k = 0;; ++k) {
        if (!__any_sync(0xffffffffu, chas)) break;
        bool nhas = false;
        if constexpr (NBUF == 2) {  // batch k+1's copies fly while batch k is multiplied
            nhas = issue((k + 1) & 1, nxtb, nbm, nbj);
            asm volatile("cp.async.wait_group 1;" ::: "memory");  // batch k's copies have landed
        } else {
            asm volatile("cp.async.wait_group 0;" ::: "memory");
        }
        __syncwarp();
        const uint32_t mC = curb.valid ? bitmap_multiply(curb.ma, cbm) : 0u;
        const T* bb = buf + (NBUF == 2 ? (k & 1) : 0) * (GROUP_BUF / NBUF);
#pragma unroll
        for (int v = 0; v < 4; ++v) {
            const int src = (lane & ~3) + v;
            const uint32_t mv = __shfl_sync(0xffffffffu, mC, src);
            const int rv = __shfl_sync(0xffffffffu, curb.row, src);
            const int32_t Jv = __shfl_sync(0xffffffffu, cbj, src);
            if (mv) {  // lane r: row r of A_t * B_j, same FMA order as k_numeric_group
                if (rv != cur) {  // group-uniform: a new C block row starts
                    if (cur >= 0) flush(cur);
                    cur = rv;
#pragma unroll
                    for (int kk = 0; kk < NC; ++kk) cid[kk] = s_cid[gi][cur][kk];
                }
                int q = 0;
#pragma unroll
                for (int kk = 0; kk < NC; ++kk) q = (cid[kk] == Jv) ? kk : q;
                Acc arow[4], b0[4], b1[4], b2[4], b3[4], w[4];
                const T* at = bb + (v * 2) * TE;
                const T* bt = at + TE;
                SRow<T>::load(at + 4 * r, arow);
                SRow<T>::load(bt, b0);
                SRow<T>::load(bt + 4, b1);
                SRow<T>::load(bt + 8, b2);
                SRow<T>::load(bt + 12, b3);
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                    Acc s_ = arow[0] * b0[e];
                    s_ = fma(arow[1], b1[e], s_);
                    s_ = fma(arow[2], b2[e], s_);
                    s_ = fma(arow[3], b3[e], s_);
                    w[e] = s_;
                }
#pragma unroll
                for (int kk = 0; kk < NC; ++kk)
                    if (kk == q)
#pragma unroll
                        for (int e = 0; e < 4; ++e) acc[kk][e] += w[e];
            }
        }
        __syncwarp();  // buffer k&1 is refilled by the next issue
        if constexpr (NBUF == 1) nhas = issue(0, nxtb, nbm, nbj);
        curb = nxtb;
        cbm = nbm;
        cbj = nbj;
        chas = nhas;
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    if (cur >= 0) flush(cur);
}

static unsigned capped(int64_t blocks) {
    const int64_t cap = (int64_t)num_sms() * 32;
    return (unsigned)(blocks < 1 ? 1 : (blocks > cap ? cap : blocks));
}

template <int LOGS, int STEP>
static amgt_status launch_warp_bin(int64_t n, const int32_t* rows, const SymCtx& c, int64_t* nnz_row, const int64_t* cptr,
                                   int32_t* cidx, uint16_t* cmap, HRec hr, cudaStream_t s) {
    if (n == 0) return AMGT_OK;
    const size_t sm = (size_t)8 * (2 * (1 << LOGS) + (1 << LOGS) / 2) * sizeof(int);
    auto kern = k_sym_warp<LOGS, STEP>;
    AMGT_CUDA(dyn_smem(kern, sm));
    kern<<<(unsigned)ceil_div(n * 32, 256), 256, sm, s>>>(n, rows, c, nnz_row, cptr, cidx, cmap, hr);
    AMGT_LAUNCHED();
    return AMGT_OK;
}

template <int LOGS, int STEP>
static amgt_status launch_block_bin(int64_t n, const int32_t* rows, const SymCtx& c, int64_t* nnz_row,
                                    const int64_t* cptr, int32_t* cidx, uint16_t* cmap, int64_t BCB, HRec hr,
                                    cudaStream_t s) {
    int jbits = 1;  // bits of a tile column (the radix sort's key width)
    while (jbits < 31 && ((int64_t)1 << jbits) < BCB) ++jbits;
    if (n == 0) return AMGT_OK;
    constexpr int S = 1 << LOGS;
    const size_t sm = (size_t)S * 4 * 2 + (STEP == 2 && LOGS > 12 ? (size_t)S / 2 * 8 : 0);  // list: bitonic path
    const int threads = LOGS >= 12 ? 512 : 256;
    auto kern = k_sym_block<LOGS, STEP>;
    AMGT_CUDA(dyn_smem(kern, sm));
    kern<<<capped(n), threads, sm, s>>>(n, rows, c, nnz_row, cptr, cidx, cmap, jbits, hr);
    AMGT_LAUNCHED();
    return AMGT_OK;
}

template <int STEP>
static amgt_status launch_dense_bin(int64_t n, const int32_t* rows, const SymCtx& c, int64_t BCB, Alloc& a,
                                    int64_t* nnz_row, const int64_t* cptr, int32_t* cidx, uint16_t* cmap,
                                    cudaStream_t s) {
    if (n == 0) return AMGT_OK;
    const int64_t W = ceil_div(BCB, 32);
    const size_t need = (size_t)W * 2 * sizeof(uint32_t);
    auto kern = k_sym_dense<STEP>;
    const size_t max_dyn = 160 * 1024;
    if (need <= max_dyn) {
        AMGT_CUDA(dyn_smem(kern, need));
        kern<<<capped(n), 512, need, s>>>(n, rows, c, W, nullptr, nnz_row, cptr, cidx, cmap);
        AMGT_LAUNCHED();
    } else {
        const int64_t G = std::min<int64_t>(n, (int64_t)num_sms());
        Scratch<uint32_t> ws;
        AMGT_TRY(ws.init(a, (size_t)G * 2 * W));
        kern<<<(unsigned)G, 512, 0, s>>>(n, rows, c, W, ws.p, nnz_row, cptr, cidx, cmap);
        AMGT_LAUNCHED();
    }
    return AMGT_OK;
}

struct SpgemmPlan;
// State of the whole-GPU dense rows between symbolic steps 1 and 2 (row bitmaps, prefixes, items).
struct GDense {
    bool on = false;
    bool plan = false;      // leave numeric records for the dense rows (SpgemmPlan)
    int dense_from = 7;
    int dense_from_eff = 7;  // the bins >= this took the dense kernels (either form)
    int64_t nd = 0, W = 0;
    int64_t cub_total = 0;  // all (A tile, B tile) pairs
    unsigned long long* npairs_dev = nullptr;  // pairs of the dense rows (counted in step 1)
    int64_t npairs = -1;                       // ... read back with the C tile count
    int64_t TB = 0, BRB = 0, vbytes = 8;
    const int64_t* pp = nullptr;  // pair prefix over A tiles, when computed before step 1
    SpgemmPlan* P = nullptr;      // step 2: the plan receiving the dense rows' records
    uint32_t* pcnt = nullptr;     // step 2: products per C tile
    Scratch<uint32_t> bm, pre;
    Scratch<int64_t> nitem, ioff;
    Scratch<int32_t> item_row;
};

// ---------------------------------------------------------------- numeric plan of the dense rows
// The whole-GPU symbolic step 2 already resolves, for every (A tile, B tile) pair of the dense
// rows, the rank of its C tile (the bitmap prefix of R15).  It records (C tile q, B tile j, A
// tile t) per pair and flags the C tiles that take more than one product, the way a two-phase
// SpGEMM keeps its work buffers between the phases (cuSPARSE's SpGEMM keeps a user buffer):
// the numeric phase of these rows is then one streaming pass with no searches.  Records are
// stored band-major: the pairs of all dense rows whose A column K (= B row) lies in band b
// precede those of band b + 1, so the B rows the concurrently running CTAs read are one band
// (~24 MB, L2-resident) instead of all of B.  A plan is keyed by C's blc_idx pointer, consumed
// by the first amgt_spgemm_numeric on that C (a second call recomputes) and dropped when C's
// structure is released.
struct SpgemmPlan {
    const void* key = nullptr;
    const int64_t* aptr = nullptr;
    const int32_t* aidx = nullptr;
    const int64_t* bptr = nullptr;
    int64_t BR = 0, TC = 0;
    int64_t nrec = 0;       // records: [0, dense pairs) band-major, then the hash-bin rows'
    int4* rec = nullptr;    // records (PlanRec / HRec)
    size_t bytes = 0;       // device bytes held
    uint32_t* mflag = nullptr;  // bit q: C tile q takes several products
    uint8_t* rowf = nullptr;    // per C block row: 1 = computed from the records
    cudaEvent_t used = nullptr;  // recorded after the last work that reads the plan (any stream)
    bool covers_all = false;     // every row with more than CAP C tiles has records
    // deterministic multi-product tiles: their C tiles, slot ranges, and the product count
    int64_t* nm_dev = nullptr;   // device: number of multi tiles
    int32_t* mq = nullptr;
    int64_t* moff = nullptr;
    int64_t nmp = 0;             // products of the multi tiles (side-buffer slots)
    // plan memory comes from the caller's allocator when the symbolic call had one (a caching
    // allocator reuses it across symbolic/numeric/free cycles; the scratch pool re-mapped it:
    // erratic symbolic times), copied here because the plan outlives the call
    amgt_allocator alc{};
    bool has_alc = false;
    size_t rec_b = 0, mflag_b = 0, rowf_b = 0, mq_b = 0, moff_b = 0;
    void* get(size_t bytes, cudaStream_t st) {
        Alloc a{has_alc ? &alc : nullptr, st};
        return a.get(bytes);
    }
    void put(void* p, size_t bytes, cudaStream_t st) {
        if (!p) return;
        Alloc a{has_alc ? &alc : nullptr, st};
        a.put(p, bytes);
    }
};

static std::mutex g_plan_mu;
static std::vector<SpgemmPlan*> g_plans;
constexpr size_t MAX_PLANS = 4;
constexpr size_t MAX_PLAN_BYTES = (size_t)2 << 30;  // least recently built plans dropped beyond

// Frees on stream s after the plan's last use, wherever that ran (virtual ranks share the cache
// from several threads and streams: an eviction on one stream must not free records another
// stream's kernels still read).
static void plan_free(SpgemmPlan* P, cudaStream_t s) {
    if (!P) return;
    if (P->used) {
        cudaStreamWaitEvent(s, P->used, 0);
        cudaEventDestroy(P->used);
    }
    P->put(P->rec, P->rec_b, s);
    P->put(P->mflag, P->mflag_b, s);
    P->put(P->nm_dev, sizeof(int64_t), s);
    P->put(P->mq, P->mq_b, s);
    P->put(P->moff, P->moff_b, s);
    P->put(P->rowf, P->rowf_b, s);
    delete P;
}

static void plan_put(SpgemmPlan* P, cudaStream_t s) {
    if (!P->used && cudaEventCreateWithFlags(&P->used, cudaEventDisableTiming) != cudaSuccess) {
        cudaGetLastError();
        P->used = nullptr;
    }
    if (P->used) cudaEventRecord(P->used, s);  // the work just enqueued on s is the latest use
    std::vector<SpgemmPlan*> old;
    {
        std::lock_guard<std::mutex> lk(g_plan_mu);
        for (size_t i = 0; i < g_plans.size();)
            if (g_plans[i]->key == P->key) { old.push_back(g_plans[i]); g_plans.erase(g_plans.begin() + i); }
            else ++i;
        g_plans.push_back(P);
        size_t held = 0;
        for (SpgemmPlan* q : g_plans) held += q->bytes;
        while (g_plans.size() > 1 && (g_plans.size() > MAX_PLANS || held > MAX_PLAN_BYTES)) {
            held -= g_plans.front()->bytes;
            old.push_back(g_plans.front());
            g_plans.erase(g_plans.begin());
        }
    }
    for (SpgemmPlan* q : old) plan_free(q, s);
}

static SpgemmPlan* plan_take(const void* key) {
    std::lock_guard<std::mutex> lk(g_plan_mu);
    for (size_t i = 0; i < g_plans.size(); ++i)
        if (g_plans[i]->key == key) {
            SpgemmPlan* P = g_plans[i];
            g_plans.erase(g_plans.begin() + i);
            return P;
        }
    return nullptr;
}

void spgemm_plan_drop(const void* key, cudaStream_t s) {
    if (!key) return;
    SpgemmPlan* P = plan_take(key);
    if (P) plan_free(P, s);
}

// pairs per A tile (all tiles): the global pair index space of the records
__global__ void k_plan_plen(int64_t TA, SymCtx c, int64_t* __restrict__ plen) {
    for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < TA; t += (int64_t)gridDim.x * blockDim.x) {
        const int32_t K = c.aidx[t];
        plen[t] = c.bptr[K + 1] - c.bptr[K];
    }
}

// tl[li][b] = pp of the first A tile of dense row li with column >= b * BW (b = 0..nb)
__global__ void k_plan_bands(int64_t nd, int nb, int64_t BW, const int32_t* __restrict__ rows, SymCtx c,
                             const int64_t* __restrict__ pp, int64_t* __restrict__ tl) {
    const int64_t n = nd * (nb + 1);
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t li = i / (nb + 1);
        const int b = (int)(i - li * (nb + 1));
        const int64_t I = rows[li];
        int64_t lo = c.aptr[I], hi = c.aptr[I + 1];
        if (b < nb) {
            const int64_t x = (int64_t)b * BW;
            while (lo < hi) {
                const int64_t mid = (lo + hi) >> 1;
                if ((int64_t)c.aidx[mid] < x) lo = mid + 1; else hi = mid;
            }
        } else {
            lo = hi;
        }
        tl[i] = pp[lo];
    }
}

// band-major item sizes sz[b * nd + li] = pairs of row li in band b
__global__ void k_plan_sizes(int64_t nd, int nb, const int64_t* __restrict__ tl, int64_t* __restrict__ sz) {
    const int64_t n = nd * nb;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t b = i / nd, li = i - b * nd;
        sz[i] = tl[li * (nb + 1) + b + 1] - tl[li * (nb + 1) + b];
    }
}

// records of a hash-bin row (bin < hb_hi) with more than CAP C tiles: its Cub pairs
__global__ void k_plan_hcount(int64_t BR, const int64_t* __restrict__ bin_of, const int64_t* __restrict__ nnz_row,
                              const int64_t* __restrict__ cub_row, int hb_hi, int64_t* __restrict__ hcnt) {
    for (int64_t I = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; I < BR; I += (int64_t)gridDim.x * blockDim.x) {
        const int64_t b = bin_of[I];
        hcnt[I] = (b < hb_hi && nnz_row[I] > CAP) ? cub_row[I] : 0;
    }
}

__global__ void k_plan_rowf(int64_t nd, const int32_t* __restrict__ rows, uint8_t* __restrict__ rowf) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nd; i += (int64_t)gridDim.x * blockDim.x)
        rowf[rows[i]] = 1;
}

template <int STEP>
static amgt_status launch_gdense(int64_t nd, const int32_t* rows, const SymCtx& c, int64_t BCB, int64_t TA, Alloc& a,
                                 GDense& g, int64_t* nnz_row, const int64_t* cptr, int32_t* cidx, uint16_t* cmap,
                                 int64_t BR, int64_t TC, const void* key, cudaStream_t s) {
    if (nd == 0) return AMGT_OK;
    static int per_sm = 0;
    if (!per_sm) {
        AMGT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_gdense_pairs<1>, GD_CH, 0));
        per_sm = max(per_sm, 1);
    }
    const unsigned pgrid = (unsigned)(num_sms() * per_sm);
    const int64_t W = g.W;
    PlanRec pr{};
    if (STEP == 1) {
        g.nd = nd;
        const int64_t cap_items = TA / GD_CH + nd + 1;  // >= sum over the rows of ceil(tiles / GD_CH)
        AMGT_TRY(g.bm.init(a, (size_t)nd * W));
        AMGT_TRY(g.pre.init(a, (size_t)nd * W));
        AMGT_TRY(g.nitem.init(a, nd));
        AMGT_TRY(g.ioff.init(a, nd + 1));
        AMGT_TRY(g.item_row.init(a, (size_t)cap_items));
        AMGT_CUDA(cudaMemsetAsync(g.bm.p, 0, (size_t)nd * W * sizeof(uint32_t), s));
        k_gdense_items<<<capped(ceil_div(nd, 256)), 256, 0, s>>>(nd, rows, c.aptr, g.nitem.p);
        AMGT_LAUNCHED();
        AMGT_TRY(scan_exclusive(g.nitem.p, g.ioff.p, nd, a, s));
        k_gdense_item_rows<<<capped(nd), 256, 0, s>>>(nd, g.ioff.p, g.item_row.p);
        AMGT_LAUNCHED();
        k_gdense_pairs<1><<<pgrid, GD_CH, 0, s>>>(g.ioff.p + nd, g.item_row.p, g.ioff.p, rows, c, W, g.bm.p,
                                                nullptr, nullptr, nullptr, pr, g.plan ? g.npairs_dev : nullptr);
        AMGT_LAUNCHED();
        k_gdense_count<<<capped(nd), GD_CNT_THREADS, 0, s>>>(nd, rows, W, g.bm.p, g.pre.p, nnz_row);
        AMGT_LAUNCHED();
        return AMGT_OK;
    }
    // step 2 (+ the dense rows' records of the numeric plan, positions [0, npairs) band-major)
    Scratch<int64_t> plen, pp, tl, sz, ioffB;
    if (g.P && g.plan && g.npairs > 0) {
        static const double band_bytes = [] {
            const char* e = getenv("AMGT_PLAN_BAND_MB");
            return (e ? atof(e) : 24.0) * 1e6;
        }();
        const double row_bytes = g.BRB ? (double)g.TB / g.BRB * (16.0 * g.vbytes + 6.0) : 1.0;
        int64_t BW = std::max<int64_t>(1, (int64_t)(band_bytes / std::max(row_bytes, 1.0)));
        BW = std::max<int64_t>(BW, ceil_div(std::max<int64_t>(g.BRB, 1), 64));  // at most 64 bands
        const int nb = (int)ceil_div(std::max<int64_t>(g.BRB, 1), BW);
        const bool have_pp = g.pp != nullptr;
        const bool ok = (have_pp || (plen.try_init(a, TA) && pp.try_init(a, TA + 1))) &&
                        tl.try_init(a, (size_t)nd * (nb + 1)) && sz.try_init(a, (size_t)nd * nb) &&
                        ioffB.try_init(a, (size_t)nd * nb + 1);
        if (ok) {
            const int64_t* ppp = g.pp;
            if (!have_pp) {
                k_plan_plen<<<capped(ceil_div(TA, 256)), 256, 0, s>>>(TA, c, plen.p);
                AMGT_LAUNCHED();
                AMGT_TRY(scan_exclusive(plen.p, pp.p, TA, a, s));
                ppp = pp.p;
            }
            k_plan_bands<<<capped(ceil_div(nd * (nb + 1), 256)), 256, 0, s>>>(nd, nb, BW, rows, c, ppp, tl.p);
            AMGT_LAUNCHED();
            k_plan_sizes<<<capped(ceil_div(nd * nb, 256)), 256, 0, s>>>(nd, nb, tl.p, sz.p);
            AMGT_LAUNCHED();
            AMGT_TRY(scan_exclusive(sz.p, ioffB.p, nd * nb, a, s));
            k_plan_rowf<<<capped(ceil_div(nd, 256)), 256, 0, s>>>(nd, rows, g.P->rowf);
            AMGT_LAUNCHED();
            pr = PlanRec{ppp, tl.p, ioffB.p, nd, BW, nb, g.P->rec, g.pcnt};
        } else {
            // no dense records: these rows' slots stay empty (q = -1) and they take the other kernels
            g.plan = false;
        }
    }
    k_gdense_out<<<capped(ceil_div(nd * W, 1024)), 256, 0, s>>>(nd, rows, W, g.bm.p, g.pre.p, cptr, cidx);
    AMGT_LAUNCHED();
    k_gdense_pairs<2><<<pgrid, GD_CH, 0, s>>>(g.ioff.p + nd, g.item_row.p, g.ioff.p, rows, c, W, g.bm.p,
                                            g.pre.p, cptr, reinterpret_cast<uint32_t*>(cmap), pr, nullptr);
    AMGT_LAUNCHED();
    return AMGT_OK;
}

template <int STEP>
static amgt_status run_bins(const int64_t* cnt, const int64_t* off, const int32_t* rows, const SymCtx& c, int64_t BCB,
                            int64_t TA, Alloc& a, GDense& g, int64_t* nnz_row, const int64_t* cptr, int32_t* cidx,
                            uint16_t* cmap, int64_t BR, int64_t TC, const void* key, HRec hr, cudaStream_t s) {
    // Bins >= dense_from take the dense-bitmap kernel (a bitmap over B's W = BC/32 column
    // words: sorted by construction, cost ~ W + Cub per row) instead of a hash table + bitonic
    // sort (~ Cub log^2 Cub): from the first bin whose lower edge 128*2^(b-1) reaches W/16,
    // while the bitmap fits in shared memory (measured on config 4, W = 8192: bins >= 3
    // 2.2 ms symbolic vs 3.6 ms with bin 7 alone dense).  AMGT_DENSE_FROM_BIN overrides.
    static const int dense_env = [] { const char* e = getenv("AMGT_DENSE_FROM_BIN"); return e ? atoi(e) : -1; }();
    // Whole-GPU form (global row bitmaps, k_gdense_*; AMGT_GDENSE=0 keeps k_sym_dense): from the
    // first bin whose lower edge reaches W / 8 words (cost ~ W words per row of memset + scan +
    // expansion against ~Cub pairs), while the bitmaps and prefixes stay under 4 GB.
    static const int gd_env = [] { const char* e = getenv("AMGT_GDENSE"); return e ? atoi(e) : 1; }();
    const int64_t W = ceil_div(BCB, 32);
    int dense_from = 7;
    if (STEP == 1) {
        g.on = false;
        g.W = W;
        if (gd_env) {
            for (int b = 2; b < 7; ++b)
                if ((128ll << (b - 1)) * 8 >= W) { dense_from = b; break; }
            if (dense_env >= 2 && dense_env <= 7) dense_from = dense_env;
            int64_t nd = 0;
            for (int b = dense_from; b < NBINS; ++b) nd += cnt[b];
            g.on = (double)nd * W * 8.0 <= 4e9;
            g.dense_from = dense_from;
        }
    }
    if (g.on) {
        dense_from = g.dense_from;
    } else {
        dense_from = 7;
        if (W * 2 * (int64_t)sizeof(uint32_t) <= 160 * 1024)
            for (int b = 2; b < 7; ++b)
                if ((128ll << (b - 1)) * 16 >= W) { dense_from = b; break; }
        if (dense_env >= 2 && dense_env <= 7) dense_from = dense_env;
    }
    g.dense_from_eff = dense_from;
    auto block_bin = [&](int b, auto launch) -> amgt_status { return b < dense_from ? launch() : AMGT_OK; };
    AMGT_TRY((launch_warp_bin<8, STEP>(cnt[0], rows + off[0], c, nnz_row, cptr, cidx, cmap, hr, s)));
    AMGT_TRY((launch_warp_bin<9, STEP>(cnt[1], rows + off[1], c, nnz_row, cptr, cidx, cmap, hr, s)));
    AMGT_TRY(block_bin(2, [&] { return launch_block_bin<10, STEP>(cnt[2], rows + off[2], c, nnz_row, cptr, cidx, cmap, BCB, hr, s); }));
    AMGT_TRY(block_bin(3, [&] { return launch_block_bin<11, STEP>(cnt[3], rows + off[3], c, nnz_row, cptr, cidx, cmap, BCB, hr, s); }));
    AMGT_TRY(block_bin(4, [&] { return launch_block_bin<12, STEP>(cnt[4], rows + off[4], c, nnz_row, cptr, cidx, cmap, BCB, hr, s); }));
    AMGT_TRY(block_bin(5, [&] { return launch_block_bin<13, STEP>(cnt[5], rows + off[5], c, nnz_row, cptr, cidx, cmap, BCB, HRec{}, s); }));
    AMGT_TRY(block_bin(6, [&] { return launch_block_bin<14, STEP>(cnt[6], rows + off[6], c, nnz_row, cptr, cidx, cmap, BCB, HRec{}, s); }));
    int64_t nd = 0;  // bins dense_from..7 are contiguous in the row lists
    for (int b = dense_from; b < NBINS; ++b) nd += cnt[b];
    if (g.on)
        AMGT_TRY((launch_gdense<STEP>(nd, rows + off[dense_from], c, BCB, TA, a, g, nnz_row, cptr, cidx, cmap, BR, TC,
                                      key, s)));
    else
        AMGT_TRY((launch_dense_bin<STEP>(nd, rows + off[dense_from], c, BCB, a, nnz_row, cptr, cidx, cmap, s)));
    return AMGT_OK;
}

static double spgemm_bytes(const amgt_mbsr* A, const amgt_mbsr* B, const amgt_mbsr* C, bool values) {
    const double s = values ? 16.0 * prec_bytes(A->prec) : 0.0;
    return (A->blc_num + B->blc_num + C->blc_num) * (s + 6.0) + (A->blc_row + B->blc_row + C->blc_row + 3) * 8.0;
}

amgt_status spgemm_symbolic_impl(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* Cout, amgt_spgemm_info* info,
                                 Alloc& a) {
    cudaStream_t s = a.s;
    if (A->n != B->m) return fail(AMGT_ERR_ARG, "SpGEMM: A.n (%lld) != B.m (%lld)", (long long)A->n, (long long)B->m);
    if (A->prec != B->prec) return fail(AMGT_ERR_ARG, "SpGEMM: A and B precisions differ");
    const int64_t BR = A->blc_row;
    SymCtx c{A->blc_ptr, A->blc_idx, A->blc_map, B->blc_ptr, B->blc_idx, B->blc_map};
    Scratch<int64_t> bin_of, nnz_row;
    Scratch<unsigned long long> ctr;  // [0..15] stats (layout above) | [16..24] bin cursors | [25] longest C row
    Scratch<int32_t> rows;
    GDense gd;  // whole-GPU dense rows (steps 1 and 2)
    Scratch<int64_t> plen_s, pp_s;  // pair prefix over A tiles (rows longer than SMALL_CUB tiles)
    Scratch<int64_t> cub_row, hcnt, hoff;  // hash-bin rows: Cub, record counts and offsets
    int64_t nH = 0;                        // record slots of the hash-bin rows (an upper bound)
    AMGT_TRY(bin_of.init(a, BR + 1));
    AMGT_TRY(nnz_row.init(a, BR + 1));
    AMGT_TRY(ctr.init(a, 32));
    AMGT_CUDA(cudaMemsetAsync(ctr.p, 0, 32 * sizeof(unsigned long long), s));
    unsigned long long* stats = ctr.p;
    unsigned long long* cursor = ctr.p + 16;
    unsigned long long* rmax = ctr.p + 25;
    amgt_mbsr C{};
    C.blc_ptr = (int64_t*)a.get((BR + 1) * sizeof(int64_t));
    if (!C.blc_ptr) return fail(AMGT_ERR_ALLOC, "SpGEMM: blc_ptr allocation failed");
    // every error return below releases what C holds (blc_ptr alone before mbsr_alloc)
    bool done = false;
    struct CGuard {
        amgt_mbsr& C;
        Alloc& a;
        bool& done;
        int64_t BR;
        ~CGuard() {
            if (done) return;
            if (C.own) mbsr_release(&C, a);
            else a.put(C.blc_ptr, (BR + 1) * sizeof(int64_t));
        }
    } cguard{C, a, done, BR};
    unsigned long long hs[16];
    {
        TimerScope ts(TC_SPGEMM_SYM, (A->blc_num + B->blc_num) * 6.0 + (A->blc_row + B->blc_row) * 8.0, s);
        // step 1 over every block row: Cub + bins (L149-151) and, for the category-8 rows
        // (Cub <= 32), the distinct tile columns (Alg. 3 lines 1-13)
        // keep the category-8 rows' sorted lists from step 1 (32 slots per row) when the scratch
        // stays moderate; step 2 is then a copy
        Scratch<int32_t> sidx;
        Scratch<uint16_t> smap;
        bool keep = BR > 0 && (double)BR * SMALL_CUB * 6.0 <= 2e9;
        if (keep)  // optional: without it step 2 re-expands the rows (k_sym_flat<2>)
            keep = sidx.try_init(a, (size_t)BR * SMALL_CUB) && smap.try_init(a, (size_t)BR * SMALL_CUB);
        // B rows of at most one tile and A rows of at most 32 (A P with an aggregation P):
        // k_sym_b1 (needs the kept scratch rows; AMGT_SYM_B1=0 forces the general kernel)
        static const int symb1_env = [] { const char* e = getenv("AMGT_SYM_B1"); return e ? atoi(e) : 1; }();
        const bool b1 = symb1_env && keep && B->row_max == 1 && A->row_max > 0 && A->row_max <= SMALL_CUB;
        if (BR > 0 && b1) {
            k_sym_b1<<<(unsigned)std::min<int64_t>(ceil_div(4 * BR, 256), (int64_t)num_sms() * 8), 256, 0, s>>>(
                BR, c, nnz_row.p, bin_of.p, stats, sidx.p, smap.p);
            AMGT_LAUNCHED();
            if (info && A->blc_num > 0) {
                k_pair_stats<<<capped(ceil_div(A->blc_num, 256)), 256, 0, s>>>(A->blc_num, c, stats, g_tc_thr_spgemm);
                AMGT_LAUNCHED();
            }
        } else if (BR > 0) {
            // rows of A longer than 4 SMALL_CUB tiles: the pair prefix over A tiles first (Cub per row
            // without a walk; reused by the whole-GPU dense rows' records)
            if (A->row_max > 4 * SMALL_CUB && A->blc_num > 0 && plen_s.try_init(a, A->blc_num) &&
                pp_s.try_init(a, A->blc_num + 1)) {
                k_plan_plen<<<capped(ceil_div(A->blc_num, 256)), 256, 0, s>>>(A->blc_num, c, plen_s.p);
                AMGT_LAUNCHED();
                AMGT_TRY(scan_exclusive(plen_s.p, pp_s.p, A->blc_num, a, s));
                gd.pp = pp_s.p;
            }
            AMGT_TRY(cub_row.init(a, BR));
            k_sym_flat<1><<<(unsigned)ceil_div(BR, 8 * SF_ROWS), 256, 0, s>>>(BR, c, nnz_row.p, nullptr, nullptr, nullptr,
                                                                     bin_of.p, stats, sidx.p, smap.p, gd.pp,
                                                                     cub_row.p);
            AMGT_LAUNCHED();
            if (info && A->blc_num > 0) {
                k_pair_stats<<<capped(ceil_div(A->blc_num, 256)), 256, 0, s>>>(A->blc_num, c, stats, g_tc_thr_spgemm);
                AMGT_LAUNCHED();
            }
        }
        AMGT_TRY(scan_exclusive(nnz_row.p, C.blc_ptr, BR, a, s, rmax));
        int64_t TC = 0;
        unsigned long long hmax = 0;
        int64_t* pin = pinned_slots();
        auto read_back = [&](bool with_stats) -> amgt_status {  // pinned when available
            if (pin) {
                int64_t* ps = pin + PIN_SYM;
                if (with_stats) AMGT_CUDA(cudaMemcpyAsync(ps, stats, sizeof(hs), cudaMemcpyDeviceToHost, s));
                AMGT_CUDA(cudaMemcpyAsync(ps + 16, C.blc_ptr + BR, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
                AMGT_CUDA(cudaMemcpyAsync(ps + 17, rmax, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
                AMGT_CUDA(cudaMemcpyAsync(ps + 18, ctr.p + 26, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
                AMGT_CUDA(cudaStreamSynchronize(s));
                if (with_stats) memcpy(hs, ps, sizeof(hs));
                TC = ps[16];
                hmax = (unsigned long long)ps[17];
                gd.npairs = ps[18];
            } else {
                if (with_stats) AMGT_CUDA(cudaMemcpyAsync(hs, stats, sizeof(hs), cudaMemcpyDeviceToHost, s));
                AMGT_CUDA(cudaMemcpyAsync(&TC, C.blc_ptr + BR, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
                AMGT_CUDA(cudaMemcpyAsync(&hmax, rmax, sizeof(hmax), cudaMemcpyDeviceToHost, s));
                AMGT_CUDA(cudaMemcpyAsync(&gd.npairs, ctr.p + 26, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
                AMGT_CUDA(cudaStreamSynchronize(s));
            }
            return AMGT_OK;
        };
        trace_point("sym step1", s);
        AMGT_TRY(read_back(true));  // sync 1: bins, C tile count (L153)
        int64_t cnt[NCAT], off[NCAT], acc = 0;
        for (int b = 0; b < NCAT; ++b) { cnt[b] = (int64_t)hs[cat_stat(b)]; off[b] = acc; acc += cnt[b]; }
        int64_t big = 0;
        for (int b = 0; b < NBINS; ++b) big += cnt[b];
        int64_t cnt_big[NCAT];  // the rows the per-bin kernels take (category 8 is done)
        for (int b = 0; b < NCAT; ++b) cnt_big[b] = b < NBINS ? cnt[b] : 0;
        if (big > 0) {  // rows with more than 32 candidates: per-bin hash kernels, then rescan
            AMGT_TRY(rows.init(a, BR + 1));
            k_bin_scatter<<<capped(ceil_div(BR, 256)), 256, 0, s>>>(BR, bin_of.p, stats, cursor, rows.p);
            AMGT_LAUNCHED();
            static const int plan_env = [] { const char* e = getenv("AMGT_SPGEMM_PLAN"); return e ? atoi(e) : 1; }();
            gd.plan = plan_env && A->blc_num < INT32_MAX && B->blc_num < INT32_MAX &&
                      (double)hs[8] * 12.0 <= 6e9;  // records: 12 B per pair
            gd.cub_total = (int64_t)hs[8];
            gd.npairs_dev = ctr.p + 26;
            gd.TB = B->blc_num;
            gd.BRB = B->blc_row;
            gd.vbytes = (int64_t)prec_bytes(B->prec);
            amgt_status st = run_bins<1>(cnt_big, off, rows.p, c, B->blc_col, A->blc_num, a, gd, nnz_row.p, nullptr,
                                         nullptr, nullptr, BR, 0, nullptr, HRec{}, s);
            if (st != AMGT_OK) return st;
            AMGT_CUDA(cudaMemsetAsync(rmax, 0, sizeof(unsigned long long), s));
            AMGT_TRY(scan_exclusive(nnz_row.p, C.blc_ptr, BR, a, s, rmax));
            trace_point("sym bins step1", s);
            AMGT_TRY(read_back(false));  // sync 2: C tile count with the long rows
            // hash-bin rows (bins < min(dense, 5): the kernels that sort in shared memory) with more
            // than CAP C tiles (some exist only if the longest C row has more): their pair counts ->
            // record offsets; the records are allocated for an upper bound (all pairs outside the
            // dense rows), so no further synchronisation
            if (plan_env && cub_row.p && (int64_t)hmax > CAP && hcnt.try_init(a, BR) && hoff.try_init(a, BR + 1)) {
                const int hb_hi = std::min(gd.dense_from_eff, 5);
                k_plan_hcount<<<capped(ceil_div(BR, 256)), 256, 0, s>>>(BR, bin_of.p, nnz_row.p, cub_row.p, hb_hi,
                                                                      hcnt.p);
                AMGT_LAUNCHED();
                AMGT_TRY(scan_exclusive(hcnt.p, hoff.p, BR, a, s));
                nH = std::max<int64_t>((int64_t)hs[8] - (gd.on && gd.plan ? std::max<int64_t>(gd.npairs, 0) : 0), 0);
            }
        }
        amgt_status st = mbsr_alloc(&C, A->m, B->n, TC, A->prec, a, true, true, C.blc_ptr);
        if (st != AMGT_OK) return st;
        C.row_max = (int64_t)hmax;
        if (TC > 0) AMGT_CUDA(cudaMemsetAsync(C.blc_map, 0, ((TC + 1) & ~int64_t(1)) * sizeof(uint16_t), s));
        // numeric plan: records of the whole-GPU dense rows ([0, npD), band-major) and of the
        // hash-bin rows with more than CAP C tiles ([npD, npD + nH), row-major)
        SpgemmPlan* P = nullptr;
        Scratch<uint32_t> pcnt;
        const int64_t npD = gd.on && gd.plan ? std::max<int64_t>(gd.npairs, 0) : 0;
        if (big > 0 && TC > 0 && TC < INT32_MAX && npD + nH > 0 && A->blc_num < INT32_MAX && B->blc_num < INT32_MAX) {
            P = new SpgemmPlan();
            P->key = C.blc_idx;
            P->aptr = A->blc_ptr;
            P->aidx = A->blc_idx;
            P->bptr = B->blc_ptr;
            P->BR = BR;
            P->TC = TC;
            P->nrec = npD + nH;
            const size_t nf = (size_t)ceil_div(TC, 32);
            P->has_alc = a.al != nullptr;
            if (a.al) P->alc = *a.al;
            P->rec_b = (size_t)P->nrec * sizeof(int4);
            P->mflag_b = nf * sizeof(uint32_t);
            P->rowf_b = (size_t)BR;
            P->rec = (int4*)P->get(P->rec_b, s);
            P->mflag = (uint32_t*)P->get(P->mflag_b, s);
            P->rowf = (uint8_t*)P->get(P->rowf_b, s);
            P->bytes = (size_t)P->nrec * sizeof(int4) + nf * sizeof(uint32_t) + (size_t)BR;
            if (!P->rec || !P->mflag || !P->rowf || !pcnt.try_init(a, (size_t)TC)) {
                plan_free(P, s);
                P = nullptr;
            } else {
                AMGT_CUDA(cudaMemsetAsync(P->rec, 0xFF, (size_t)P->nrec * sizeof(int4), s));
                AMGT_CUDA(cudaMemsetAsync(pcnt.p, 0, (size_t)TC * sizeof(uint32_t), s));
                AMGT_CUDA(cudaMemsetAsync(P->rowf, 0, (size_t)BR, s));
            }
        }
        trace_point("sym alloc", s);
        gd.P = npD > 0 ? P : nullptr;
        gd.pcnt = pcnt.p;
        HRec hr{};
        if (P && nH > 0) hr = HRec{hoff.p, P->rec + npD, pcnt.p, P->rowf};
        struct PlanScope {  // the plan goes to the cache once step 2 has filled it (freed on errors)
            SpgemmPlan*& P;
            cudaStream_t s;
            bool ok = false;
            ~PlanScope() {
                if (P && !ok) plan_free(P, s);
            }
        } pscope{P, s};
        if (BR > 0) {  // step 2 (Alg. 3 lines 13-14 + bitmap OR, R15)
            if (keep)
                k_sym_copy<<<capped(ceil_div(4 * BR, 256)), 256, 0, s>>>(BR, bin_of.p, C.blc_ptr, sidx.p, smap.p,
                                                                       C.blc_idx, C.blc_map);
            else
                k_sym_flat<2><<<(unsigned)ceil_div(BR, 8 * SF_ROWS), 256, 0, s>>>(BR, c, nullptr, C.blc_ptr, C.blc_idx,
                                                                         C.blc_map, bin_of.p, nullptr);
            AMGT_LAUNCHED();
            if (big > 0) {
                st = run_bins<2>(cnt_big, off, rows.p, c, B->blc_col, A->blc_num, a, gd, nullptr, C.blc_ptr, C.blc_idx,
                                 C.blc_map, BR, TC, C.blc_idx, hr, s);
                if (st != AMGT_OK) return st;
            }
        }
        trace_point("sym step2", s);
        if (P) {
            // rows past CAP C tiles without records: dense rows whose records failed, hash rows when
            // the longest C row exceeds CAP and no offsets were computed, bins 5-6 (bitonic kernels)
            int64_t dense_rows = 0, bitonic_rows = 0;
            for (int b = gd.dense_from_eff; b < NBINS; ++b) dense_rows += cnt_big[b];
            for (int b = 5; b < std::min(gd.dense_from_eff, NBINS); ++b) bitonic_rows += cnt_big[b];
            const bool dense_ok = dense_rows == 0 || (gd.on && gd.plan && npD > 0);
            const bool hash_ok = (int64_t)hmax <= CAP || (hoff.p != nullptr && nH > 0);
            P->covers_all = dense_ok && hash_ok && bitonic_rows == 0;
            k_plan_mark<<<capped(ceil_div(TC, 256)), 256, 0, s>>>(TC, pcnt.p, P->mflag);
            AMGT_LAUNCHED();
            // deterministic multi tiles: number them, give each a slot range, point their records at
            // the slots (two read-backs: the tile count, then the slot count)
            // opt-in (AMGT_SPGEMM_DET=1): two more host syncs and per-call slot arrays; measured on
            // config 4 with erratic symbolic times (2.1-4.3 ms vs 1.88 ms without)
            static const int det_env = [] { const char* e = getenv("AMGT_SPGEMM_DET"); return e ? atoi(e) : 0; }();
            const int64_t nw = ceil_div(TC, 32);
            Scratch<int64_t> wpop, mwpre, mcnt;
            Scratch<uint32_t> mfill;
            int64_t* pin = pinned_slots();
            auto read1 = [&](const int64_t* dsrc, int64_t* out) -> amgt_status {  // one synchronised read-back
                if (pin) {
                    AMGT_CUDA(cudaMemcpyAsync(pin + PIN_SYM + 19, dsrc, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
                    AMGT_CUDA(cudaStreamSynchronize(s));
                    *out = pin[PIN_SYM + 19];
                } else {
                    AMGT_CUDA(cudaMemcpyAsync(out, dsrc, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
                    AMGT_CUDA(cudaStreamSynchronize(s));
                }
                return AMGT_OK;
            };
            int64_t nm = 0;
            bool det = det_env && wpop.try_init(a, nw) && mwpre.try_init(a, nw + 1);
            if (det) {
                k_plan_wpop<<<capped(ceil_div(nw, 256)), 256, 0, s>>>(nw, P->mflag, wpop.p);
                AMGT_LAUNCHED();
                AMGT_TRY(scan_exclusive(wpop.p, mwpre.p, nw, a, s));
                trace_point("sym det mark", s);
                AMGT_TRY(read1(mwpre.p + nw, &nm));  // sync: the number of multi tiles
                if (nm > 0) {
                    P->mq_b = (size_t)nm * sizeof(int32_t);
                    P->moff_b = (size_t)(nm + 1) * sizeof(int64_t);
                    P->nm_dev = (int64_t*)P->get(sizeof(int64_t), s);
                    P->mq = (int32_t*)P->get(P->mq_b, s);
                    P->moff = (int64_t*)P->get(P->moff_b, s);
                    det = P->nm_dev && P->mq && P->moff && mcnt.try_init(a, nm) && mfill.try_init(a, nm);
                } else {
                    det = false;  // no multi tiles: nothing to order
                }
            }
            if (det) {
                AMGT_CUDA(cudaMemcpyAsync(P->nm_dev, mwpre.p + nw, sizeof(int64_t), cudaMemcpyDeviceToDevice, s));
                k_plan_mlist<<<capped(ceil_div(nw, 256)), 256, 0, s>>>(TC, P->mflag, mwpre.p, pcnt.p, P->mq, mcnt.p);
                AMGT_LAUNCHED();
                AMGT_TRY(scan_exclusive(mcnt.p, P->moff, nm, a, s));
                AMGT_CUDA(cudaMemsetAsync(mfill.p, 0, (size_t)nm * sizeof(uint32_t), s));
                if (P->nrec > 0) {
                    k_plan_slots<<<capped(ceil_div(P->nrec, 256)), 256, 0, s>>>(P->nrec, P->rec, P->mflag, mwpre.p,
                                                                               P->moff, mfill.p);
                    AMGT_LAUNCHED();
                }
                trace_point("sym det slots", s);
                AMGT_TRY(read1(P->moff + nm, &P->nmp));  // sync: the products of the multi tiles
                P->bytes += (size_t)nm * 12 + 8;
            } else {
                P->put(P->nm_dev, sizeof(int64_t), s);
                P->put(P->mq, P->mq_b, s);
                P->put(P->moff, P->moff_b, s);
                P->nm_dev = nullptr;
                P->mq = nullptr;
                P->moff = nullptr;
            }
            pscope.ok = true;
            plan_put(P, s);
        }
        ts.bytes = (A->blc_num + B->blc_num) * 6.0 * 2 + (A->blc_row + B->blc_row) * 8.0 + TC * 6.0 + (BR + 1) * 8.0;
    }
    if (info) {
        for (int b = 0; b < NBINS; ++b) info->bin_rows[b] = (int64_t)hs[b];
        info->bin_rows[0] += (int64_t)hs[12];  // category 8 is part of bin 0
        info->cub_total = (int64_t)hs[8];
        info->pairs_nonzero = (int64_t)hs[9];
        info->pairs_tc = (int64_t)hs[10];
        info->scalar_products = (int64_t)hs[11];
        Scratch<unsigned long long> nr;
        AMGT_TRY(nr.init(a, 3));
        AMGT_CUDA(cudaMemsetAsync(nr.p, 0, 3 * sizeof(unsigned long long), s));
        if (BR > 0) {
            k_numeric_rows_stats<<<capped(ceil_div(BR, 256)), 256, 0, s>>>(BR, C.blc_ptr, nr.p);
            AMGT_LAUNCHED();
        }
        unsigned long long h3[3];
        AMGT_CUDA(cudaMemcpyAsync(h3, nr.p, sizeof(h3), cudaMemcpyDeviceToHost, s));
        AMGT_CUDA(cudaStreamSynchronize(s));
        for (int k = 0; k < 3; ++k) info->numeric_rows[k] = (int64_t)h3[k];
    }
    done = true;
    *Cout = C;
    trace_point("sym end", s);
    trace_dump();
    return AMGT_OK;
}

// ---------------------------------------------------------------- numeric: B with one tile per row
// C = A B when every block row of B holds at most one tile (the aggregation P of the RAP's A P,
// R19): each A tile (I, K) meets at most one B tile (K, J_K), so C row I (<= NC tiles, positions
// from the symbolic phase) is a sum of A tile x single B tile products.  A 4-lane group per C
// block row, lane r owning row r of every C tile.  The row's A tiles are taken 32 at a time: the
// group first resolves each tile's B position and C slot (lane r, slot s <- tile 4s + r: column,
// B row pointers, B column — three rounds of independent loads for the whole chunk), then streams
// the chunk four tiles per step with no dependent load left (A row r of four tiles in flight per
// lane in registers, their B tiles copied row by row into a per-group shared-memory buffer with
// cp.async and read back as broadcasts).  The products are formed as
// in tile_mma and added in A-tile order into the lane's rows of the C tiles in shared memory
// (lane-private, deterministic: the staged kernel's arithmetic); C rows written once with
// full-line stores (+0.0 at the clear bits, R2).  Group buffers are padded by 16 B so the eight
// groups of a warp spread over the banks.
constexpr int B1_WARPS = 8;
template <typename Acc, int NC>
constexpr int b1_gstride() { return NC * 16 + 16 / (int)sizeof(Acc); }
// per group: the C-row accumulators (b1_gstride Acc) + the step's four B tiles (64 T, 16-B padded)
template <typename T>
constexpr int b1_bstride() { return 64 + 16 / (int)sizeof(T); }
template <typename T, typename Acc, int NC>
constexpr size_t b1_smem_bytes() {
    return (size_t)B1_WARPS * 8 * (b1_gstride<Acc, NC>() * sizeof(Acc) + b1_bstride<T>() * sizeof(T));
}

// Row r of a B tile: global -> shared memory without registers (cp.async), and shared -> Acc.
template <typename T> struct B1Row;
template <> struct B1Row<double> {
    static __device__ __forceinline__ void copy(double* d, const double* g) { cp_async16(d, g); cp_async16(d + 2, g + 2); }
    static __device__ __forceinline__ void read(const double* p, double (&v)[4]) {
        const double2 a = reinterpret_cast<const double2*>(p)[0], b = reinterpret_cast<const double2*>(p)[1];
        v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
    }
};
template <> struct B1Row<float> {
    static __device__ __forceinline__ void copy(float* d, const float* g) { cp_async16(d, g); }
    static __device__ __forceinline__ void read(const float* p, float (&v)[4]) {
        const float4 a = *reinterpret_cast<const float4*>(p);
        v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
    }
};
template <> struct B1Row<__half> {
    static __device__ __forceinline__ void copy(__half* d, const __half* g) {
        const uint32_t sa = (uint32_t)__cvta_generic_to_shared(d);
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(sa), "l"(g) : "memory");
    }
    static __device__ __forceinline__ void read(const __half* p, float (&v)[4]) {
        const uint2 u = *reinterpret_cast<const uint2*>(p);
        const float2 lo = __half22float2(*reinterpret_cast<const __half2*>(&u.x));
        const float2 hi = __half22float2(*reinterpret_cast<const __half2*>(&u.y));
        v[0] = lo.x; v[1] = lo.y; v[2] = hi.x; v[3] = hi.y;
    }
};

template <typename Acc> struct SmemRow;
template <> struct SmemRow<double> {
    static __device__ __forceinline__ void add(double* p, const double (&v)[4]) {
        double2* q = reinterpret_cast<double2*>(p);
        double2 a = q[0], b = q[1];
        a.x += v[0]; a.y += v[1]; b.x += v[2]; b.y += v[3];
        q[0] = a; q[1] = b;
    }
    static __device__ __forceinline__ void take(double* p, double (&v)[4]) {
        double2* q = reinterpret_cast<double2*>(p);
        const double2 a = q[0], b = q[1];
        v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
        q[0] = q[1] = make_double2(0.0, 0.0);
    }
    static __device__ __forceinline__ void zero(double* p) {
        reinterpret_cast<double2*>(p)[0] = reinterpret_cast<double2*>(p)[1] = make_double2(0.0, 0.0);
    }
};
template <> struct SmemRow<float> {
    static __device__ __forceinline__ void add(float* p, const float (&v)[4]) {
        float4* q = reinterpret_cast<float4*>(p);
        float4 a = *q;
        a.x += v[0]; a.y += v[1]; a.z += v[2]; a.w += v[3];
        *q = a;
    }
    static __device__ __forceinline__ void take(float* p, float (&v)[4]) {
        float4* q = reinterpret_cast<float4*>(p);
        const float4 a = *q;
        v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
        *q = make_float4(0.f, 0.f, 0.f, 0.f);
    }
    static __device__ __forceinline__ void zero(float* p) { *reinterpret_cast<float4*>(p) = make_float4(0.f, 0.f, 0.f, 0.f); }
};

template <typename T, typename Acc, int NC>
__global__ void __launch_bounds__(B1_WARPS * 32, 2) k_numeric_b1(int64_t BR, SymCtx c, const T* __restrict__ aval,
                                                             const T* __restrict__ bval, const int64_t* __restrict__ cptr,
                                                             const int32_t* __restrict__ cidx,
                                                             const uint16_t* __restrict__ cmap, T* __restrict__ cval) {
    extern __shared__ __align__(16) unsigned char b1_smem[];
    const int lane = threadIdx.x & 31, g = lane >> 2, r = lane & 3;
    const unsigned gm = 0xFu << (lane & ~3);
    const int gb = lane & ~3;
    const int gid = (threadIdx.x >> 5) * 8 + g;
    Acc* acc = reinterpret_cast<Acc*>(b1_smem) + gid * b1_gstride<Acc, NC>() + 4 * r;
    T* sB = reinterpret_cast<T*>(b1_smem + (size_t)B1_WARPS * 8 * b1_gstride<Acc, NC>() * sizeof(Acc)) +
            gid * b1_bstride<T>();  // tile u at sB + 16 u (row-major)
#pragma unroll
    for (int q = 0; q < NC; ++q) SmemRow<Acc>::zero(acc + 16 * q);
    const int64_t ng = ((int64_t)gridDim.x * blockDim.x) >> 2;
    for (int64_t I = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 2; I < BR; I += ng) {
        const int64_t c0 = cptr[I];
        const int nC = (int)(cptr[I + 1] - c0);
        int32_t cj[NC];
#pragma unroll
        for (int q = 0; q < NC; ++q) cj[q] = q < nC ? __ldg(cidx + c0 + q) : -1;
        const int64_t t0 = c.aptr[I], t1 = c.aptr[I + 1];
        for (int64_t tc = t0; tc < t1; tc += 32) {
            // chunk metadata: lane r resolves tiles tc + 4s + r
            int32_t K[8], bp[8];
#pragma unroll
            for (int s = 0; s < 8; ++s) K[s] = tc + 4 * s + r < t1 ? __ldg(c.aidx + tc + 4 * s + r) : -1;
            int64_t b0[8];
            bool has[8];
#pragma unroll
            for (int s = 0; s < 8; ++s) {
                b0[s] = K[s] >= 0 ? __ldg(c.bptr + K[s]) : 0;
                has[s] = K[s] >= 0 && __ldg(c.bptr + K[s] + 1) > b0[s];
            }
            uint32_t qq = 0;
#pragma unroll
            for (int s = 0; s < 8; ++s) {
                const int32_t J = has[s] ? __ldg(c.bidx + b0[s]) : -1;
                int q = 15;
#pragma unroll
                for (int k = 0; k < NC; ++k)
                    if (cj[k] == J && J >= 0) q = k;
                bp[s] = q < NC ? (int32_t)b0[s] : -1;
                qq |= (uint32_t)q << (4 * s);
            }
            const int ns = (int)(t1 - tc < 32 ? t1 - tc : 32);
#pragma unroll
            for (int s = 0; s < 8; ++s) {
                if (4 * s >= ns) break;  // uniform across the group
                int qv[4];
                Acc ar[4][4];
#pragma unroll
                for (int u = 0; u < 4; ++u) {  // B row r of the four tiles -> shared memory, A row r -> registers
                    const int32_t bpu = __shfl_sync(gm, bp[s], gb + u);
                    qv[u] = (int)((__shfl_sync(gm, qq, gb + u) >> (4 * s)) & 15u);
                    if (bpu >= 0) {
                        B1Row<T>::copy(sB + 16 * u + 4 * r, bval + 16 * (int64_t)bpu + 4 * r);
                        RowIO<T>::load(aval + 16 * (tc + 4 * s + u) + 4 * r, ar[u]);
                    } else {
                        qv[u] = 15;
                    }
                }
                asm volatile("cp.async.commit_group;" ::: "memory");
                asm volatile("cp.async.wait_group 0;" ::: "memory");
                __syncwarp(gm);
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    if (qv[u] >= NC) continue;  // uniform across the group (same tile)
                    Acc pr[4];  // row r of A_t B, in tile_mma's order (k = 0..3)
                    {
                        Acc b0[4];
                        B1Row<T>::read(sB + 16 * u, b0);
#pragma unroll
                        for (int col = 0; col < 4; ++col) pr[col] = ar[u][0] * b0[col];
                    }
#pragma unroll
                    for (int k = 1; k < 4; ++k) {
                        Acc bk[4];
                        B1Row<T>::read(sB + 16 * u + 4 * k, bk);
#pragma unroll
                        for (int col = 0; col < 4; ++col) pr[col] = fma_acc(ar[u][k], bk[col], pr[col]);
                    }
                    SmemRow<Acc>::add(acc + 16 * qv[u], pr);
                }
                __syncwarp(gm);  // the step's B tiles are consumed before the next step's copies
            }
        }
#pragma unroll
        for (int q = 0; q < NC; ++q) {
            if (q >= nC) break;
            const uint32_t mp = (__ldg(cmap + c0 + q) >> (4 * r)) & 0xFu;
            Acc v[4], o[4];
            SmemRow<Acc>::take(acc + 16 * q, v);
#pragma unroll
            for (int col = 0; col < 4; ++col) o[col] = ((mp >> col) & 1u) ? v[col] : Acc(0);
            RowIO<T>::store(cval + 16 * (c0 + q) + 4 * r, o);
        }
    }
}

template <typename T, typename Acc, int NC>
static amgt_status launch_b1(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* C, const SymCtx& c, cudaStream_t s) {
    auto kern = k_numeric_b1<T, Acc, NC>;
    const size_t sm = b1_smem_bytes<T, Acc, NC>();
    AMGT_CUDA(dyn_smem(kern, sm));
    static const int per_sm = [&] {
        int n = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kern, B1_WARPS * 32, sm);
        return n > 0 ? n : 1;
    }();
    const int64_t BR = A->blc_row;
    const unsigned grid = (unsigned)std::min<int64_t>(ceil_div(4 * BR, B1_WARPS * 32), (int64_t)num_sms() * per_sm);
    kern<<<grid, B1_WARPS * 32, sm, s>>>(BR, c, (const T*)A->blc_val, (const T*)B->blc_val, C->blc_ptr, C->blc_idx,
                                         C->blc_map, (T*)C->blc_val);
    AMGT_LAUNCHED();
    return AMGT_OK;
}

// ---------------------------------------------------------------- numeric: plan rows
// Multi-product C tiles of the plan rows start at zero (the accumulation target: C values, or
// the FP32 workspace for FP16).
template <typename Acc>
__global__ void k_plan_zero(int64_t TC, const uint32_t* __restrict__ mflag, Acc* __restrict__ acc) {
    const int64_t nw = (TC + 31) / 32;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nw; i += (int64_t)gridDim.x * blockDim.x) {
        uint32_t f = mflag[i];
        while (f) {
            const int b = __ffs(f) - 1;
            f &= f - 1;
            uint4* v = reinterpret_cast<uint4*>(acc + 16 * (32 * i + b));
#pragma unroll
            for (int e = 0; e < (int)sizeof(Acc); ++e) v[e] = make_uint4(0u, 0u, 0u, 0u);
        }
    }
}

template <typename Acc> struct SideRow;
template <> struct SideRow<double> {
    static __device__ __forceinline__ void store(double* p, const double (&v)[4]) {
        reinterpret_cast<double2*>(p)[0] = make_double2(v[0], v[1]);
        reinterpret_cast<double2*>(p)[1] = make_double2(v[2], v[3]);
    }
    static __device__ __forceinline__ void load(const double* p, double (&v)[4]) {
        const double2 a = reinterpret_cast<const double2*>(p)[0], b = reinterpret_cast<const double2*>(p)[1];
        v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y;
    }
};
template <> struct SideRow<float> {
    static __device__ __forceinline__ void store(float* p, const float (&v)[4]) {
        *reinterpret_cast<float4*>(p) = make_float4(v[0], v[1], v[2], v[3]);
    }
    static __device__ __forceinline__ void load(const float* p, float (&v)[4]) {
        const float4 a = *reinterpret_cast<const float4*>(p);
        v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
    }
};

// Each multi tile (a 4-lane group): its products' slots in ascending A-tile order (insertion by
// t, recomputed per step so any count works), lane r adds row r of them into a zero row in that
// order (the accumulation of Alg. 4 in pair order: deterministic) and writes the tile row
// (+0.0 at the clear bits, R2; FP16 rounded once from the FP32 sum).
template <typename T, typename Acc>
__global__ void k_plan_msum(const int64_t* __restrict__ nm_dev, const int32_t* __restrict__ mq,
                            const int64_t* __restrict__ moff, const Acc* __restrict__ side_v,
                            const int32_t* __restrict__ side_t, const uint16_t* __restrict__ cmap,
                            T* __restrict__ cval) {
    const int64_t nm = *nm_dev;
    const int r = threadIdx.x & 3;
    for (int64_t mi = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 2; mi < nm;
         mi += ((int64_t)gridDim.x * blockDim.x) >> 2) {
        const int64_t s0 = moff[mi], s1 = moff[mi + 1];
        Acc sum[4] = {Acc(0), Acc(0), Acc(0), Acc(0)};
        int prev = INT_MIN;
        int64_t prev_s = -1;
        for (int64_t k = s0; k < s1; ++k) {  // next slot in (t, slot) order
            int best = INT_MAX;
            int64_t bs = -1;
            for (int64_t x = s0; x < s1; ++x) {
                const int tx = side_t[x];
                const bool after = tx > prev || (tx == prev && x > prev_s);
                if (after && (tx < best || (tx == best && x < bs))) { best = tx; bs = x; }
            }
            Acc v[4];
            SideRow<Acc>::load(side_v + 16 * bs + 4 * r, v);
#pragma unroll
            for (int e = 0; e < 4; ++e) sum[e] += v[e];
            prev = best;
            prev_s = bs;
        }
        const int64_t q = mq[mi];
        const uint32_t nib = (cmap[q] >> (4 * r)) & 0xFu;
        Acc o[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) o[e] = ((nib >> e) & 1u) ? sum[e] : Acc(0);
        RowIO<T>::store(cval + 16 * q + 4 * r, o);
    }
}

// One pass over the records, PLAN_R records per block of work: the records arrive in registers
// one block ahead, the A and B tiles of a block are copied to shared memory with cp.async one
// block ahead (double-buffered), and four threads per record each form one row of A_t * B_j
// (the tile_mma arithmetic, k = 0..3).  A single-product tile is written with full-line
// stores (the four threads' rows are one 128-B line for FP64; +0.0 at the clear bits, R2); a
// multi-product tile takes REDs at its bitmap positions (zeroed by k_plan_zero).
constexpr int PLAN_R = 64;  // records per block of work (4 threads each)
template <typename T>
__device__ __forceinline__ void cp_async16_g(void* smem, const void* gmem) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sa), "l"(gmem) : "memory");
}
// the same with an L2 eviction-priority policy (createpolicy)
__device__ __forceinline__ void cp_async16_hint(void* smem, const void* gmem, uint64_t pol) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2;" ::"r"(sa), "l"(gmem), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
// streaming (evict-first) row stores of the C tiles: the product is not read again here
template <typename T> struct RowCS;
template <> struct RowCS<double> {
    static __device__ __forceinline__ void store(double* p, const double (&v)[4]) {
        __stcs(reinterpret_cast<double2*>(p), make_double2(v[0], v[1]));
        __stcs(reinterpret_cast<double2*>(p) + 1, make_double2(v[2], v[3]));
    }
};
template <> struct RowCS<float> {
    static __device__ __forceinline__ void store(float* p, const float (&v)[4]) {
        __stcs(reinterpret_cast<float4*>(p), make_float4(v[0], v[1], v[2], v[3]));
    }
};
template <> struct RowCS<__half> {
    static __device__ __forceinline__ void store(__half* p, const float (&v)[4]) { RowIO<__half>::store(p, v); }
};
template <typename T, typename Acc, bool DET = false>
__global__ void __launch_bounds__(PLAN_R * 4) k_plan_flat(int64_t total, const int4* __restrict__ rec,
                                                         const uint32_t* __restrict__ mflag,
                                                         const T* __restrict__ aval, const T* __restrict__ bval,
                                                         T* __restrict__ cval, Acc* __restrict__ gacc,
                                                         int hints, Acc* __restrict__ side_v = nullptr,
                                                         int32_t* __restrict__ side_t = nullptr) {
    constexpr int TE = 16;
    constexpr int CH = 16 / (int)sizeof(T);       // elements per 16-B piece
    constexpr int PC = TE / CH;                   // 16-B pieces per tile
    constexpr int TS = TE + CH;                   // padded tile stride: the 8 records a warp reads
                                                  // at once fall on different banks
    __shared__ __align__(16) T sA[2][PLAN_R][TS];
    __shared__ __align__(16) T sB[2][PLAN_R][TS];
    __shared__ int4 sr[2][PLAN_R];
    __shared__ int sa[2][PLAN_R];  // record whose A copy this record uses (runs of one A tile)
    const int tid = threadIdx.x;
    const int64_t nblk = (total + PLAN_R - 1) / PLAN_R;
    Acc* acc = gacc ? gacc : reinterpret_cast<Acc*>(cval);
    const uint64_t pol = policy_evict_last();
    auto load_rec = [&](int64_t blk) {
        int4 r = make_int4(-1, 0, 0, 0);
        if (tid < PLAN_R && blk < nblk) {
            const int64_t p = blk * PLAN_R + tid;
            if (p < total) r = __ldg(rec + p);
        }
        return r;
    };
    auto stage = [&](int buf, const int4& r) {  // warps 0-1: record + A-run slot
        if (tid < PLAN_R) {
            const int lane = tid & 31;
            const int zp = __shfl_up_sync(0xffffffffu, r.z, 1);
            const unsigned bal = __ballot_sync(0xffffffffu, lane == 0 || r.x == -1 || r.z != zp);
            sr[buf][tid] = r;
            sa[buf][tid] = (tid & ~31) + 31 - __clz(bal & (0xffffffffu >> (31 - lane)));
        }
    };
    auto issue = [&](int buf) {  // tiles of the records in sr[buf]
        for (int k = tid; k < PLAN_R * 2 * PC; k += PLAN_R * 4) {
            const int ri = k / (2 * PC), part = k - ri * 2 * PC;
            const int4 r = sr[buf][ri];
            if (r.x == -1) continue;  // empty product (<= -2: a multi tile's product slot)
            if (part < PC) {
                if (sa[buf][ri] == ri) cp_async16_g<T>(&sA[buf][ri][part * CH], aval + 16 * (int64_t)r.z + part * CH);
            } else if (hints & 1) {
                cp_async16_hint(&sB[buf][ri][(part - PC) * CH], bval + 16 * (int64_t)r.y + (part - PC) * CH, pol);
            } else {
                cp_async16_g<T>(&sB[buf][ri][(part - PC) * CH], bval + 16 * (int64_t)r.y + (part - PC) * CH);
            }
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    int64_t blk = blockIdx.x;
    if (blk >= nblk) return;
    stage(0, load_rec(blk));
    __syncthreads();
    issue(0);
    int4 rnext = load_rec(blk + gridDim.x);
    const int ri = tid >> 2, row = tid & 3;
    for (int it = 0; blk < nblk; ++it, blk += gridDim.x) {
        const int buf = it & 1;
        const bool more = blk + gridDim.x < nblk;
        if (more) {
            stage(buf ^ 1, rnext);
            __syncthreads();
            issue(buf ^ 1);
            rnext = load_rec(blk + 2 * (int64_t)gridDim.x);
            asm volatile("cp.async.wait_group 1;" ::: "memory");
        } else {
            asm volatile("cp.async.wait_group 0;" ::: "memory");
        }
        __syncthreads();
        const int4 r = sr[buf][ri];
        if (r.x >= 0) {
            Acc a4[4], o[4];
            SRow<T>::load(&sA[buf][sa[buf][ri]][4 * row], a4);
            Acc b0[4], b1[4], b2[4], b3[4];
            SRow<T>::load(&sB[buf][ri][0], b0);
            SRow<T>::load(&sB[buf][ri][4], b1);
            SRow<T>::load(&sB[buf][ri][8], b2);
            SRow<T>::load(&sB[buf][ri][12], b3);
#pragma unroll
            for (int e = 0; e < 4; ++e) {
                Acc v = a4[0] * b0[e];
                v = fma_acc(a4[1], b1[e], v);
                v = fma_acc(a4[2], b2[e], v);
                v = fma_acc(a4[3], b3[e], v);
                o[e] = v;
            }
            const uint32_t nib = ((uint32_t)r.w >> (4 * row)) & 0xFu;
            const bool multi = (__ldg(mflag + (r.x >> 5)) >> (r.x & 31)) & 1u;
            const int64_t q = r.x;
            if (!multi) {
#pragma unroll
                for (int e = 0; e < 4; ++e) o[e] = ((nib >> e) & 1u) ? o[e] : Acc(0);
                if (hints & 2) RowCS<T>::store(cval + 16 * q + 4 * row, o);
                else RowIO<T>::store(cval + 16 * q + 4 * row, o);
            } else {
#pragma unroll
                for (int e = 0; e < 4; ++e)
                    if ((nib >> e) & 1u) atomicAdd(acc + 16 * q + 4 * row + e, o[e]);
            }
        } else if (DET && r.x <= -2) {  // a product of a multi tile: to its slot (k_plan_msum adds them)
            Acc a4[4], o[4];
            SRow<T>::load(&sA[buf][sa[buf][ri]][4 * row], a4);
            Acc b0[4], b1[4], b2[4], b3[4];
            SRow<T>::load(&sB[buf][ri][0], b0);
            SRow<T>::load(&sB[buf][ri][4], b1);
            SRow<T>::load(&sB[buf][ri][8], b2);
            SRow<T>::load(&sB[buf][ri][12], b3);
#pragma unroll
            for (int e = 0; e < 4; ++e) {
                Acc v = a4[0] * b0[e];
                v = fma_acc(a4[1], b1[e], v);
                v = fma_acc(a4[2], b2[e], v);
                v = fma_acc(a4[3], b3[e], v);
                o[e] = v;
            }
            const int64_t slot = -(int64_t)r.x - 2;
            SideRow<Acc>::store(side_v + 16 * slot + 4 * row, o);
            if (row == 0) side_t[slot] = r.z;
        }
        __syncthreads();  // buffer `buf` is refilled two iterations on
    }
}

// Bulk-copy (TMA 1-D, cp.async.bulk) form of k_plan_flat: per record, the thread owning it in
// warps 0-1 arms the stage's mbarrier with its byte count and issues one bulk copy per tile (B,
// and A at the start of a run of one A tile) — 1-2 instructions per record instead of sixteen
// 16-B cp.async spread over the block, and the copies bypass the LSU/L1 request path.
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
    uint32_t done = 0;
    while (!done) {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(done)
            : "r"(smem_u32(b)), "r"(parity)
            : "memory");
    }
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(b))
                 : "memory");
}

template <typename T, typename Acc>
__global__ void __launch_bounds__(PLAN_R * 4) k_plan_flat_bulk(int64_t total, const int4* __restrict__ rec,
                                                              const uint32_t* __restrict__ mflag,
                                                              const T* __restrict__ aval, const T* __restrict__ bval,
                                                              T* __restrict__ cval, Acc* __restrict__ gacc, int hints) {
    constexpr int TE = 16;
    constexpr int CH = 16 / (int)sizeof(T);
    constexpr int TS = TE + CH;  // padded tile stride (bank spread), 16-B multiple
    constexpr uint32_t TB = TE * sizeof(T);
    __shared__ __align__(16) T sA[2][PLAN_R][TS];
    __shared__ __align__(16) T sB[2][PLAN_R][TS];
    __shared__ int4 sr[2][PLAN_R];
    __shared__ int sa[2][PLAN_R];
    __shared__ __align__(8) uint64_t mbar[2];
    const int tid = threadIdx.x;
    const int64_t nblk = (total + PLAN_R - 1) / PLAN_R;
    Acc* acc = gacc ? gacc : reinterpret_cast<Acc*>(cval);
    int64_t blk = blockIdx.x;
    if (blk >= nblk) return;
    if (tid == 0) {
        mbar_init(&mbar[0], PLAN_R);
        mbar_init(&mbar[1], PLAN_R);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    auto load_rec = [&](int64_t b) {
        int4 r = make_int4(-1, 0, 0, 0);
        if (tid < PLAN_R && b < nblk) {
            const int64_t p = b * PLAN_R + tid;
            if (p < total) r = __ldg(rec + p);
        }
        return r;
    };
    // warps 0-1: stage the record, its A-run slot, arm the barrier and issue its copies
    auto produce = [&](int buf, const int4& r) {
        if (tid < PLAN_R) {
            const int lane = tid & 31;
            const int zp = __shfl_up_sync(0xffffffffu, r.z, 1);
            const unsigned bal = __ballot_sync(0xffffffffu, lane == 0 || r.x < 0 || r.z != zp);
            const int slot = (tid & ~31) + 31 - __clz(bal & (0xffffffffu >> (31 - lane)));
            sr[buf][tid] = r;
            sa[buf][tid] = slot;
            const bool own_a = r.x >= 0 && slot == tid;
            const uint32_t bytes = r.x >= 0 ? TB * (own_a ? 2u : 1u) : 0u;
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // prior generic reads of the buffer
            mbar_arrive_tx(&mbar[buf], bytes);
            if (r.x >= 0) {
                bulk_g2s(&sB[buf][tid][0], bval + 16 * (int64_t)r.y, TB, &mbar[buf]);
                if (own_a) bulk_g2s(&sA[buf][tid][0], aval + 16 * (int64_t)r.z, TB, &mbar[buf]);
            }
        }
    };
    uint32_t par[2] = {0u, 0u};
    produce(0, load_rec(blk));
    int4 rnext = load_rec(blk + gridDim.x);
    const int ri = tid >> 2, row = tid & 3;
    for (int it = 0; blk < nblk; ++it, blk += gridDim.x) {
        const int buf = it & 1;
        if (blk + gridDim.x < nblk) {
            produce(buf ^ 1, rnext);
            rnext = load_rec(blk + 2 * (int64_t)gridDim.x);
        }
        mbar_wait(&mbar[buf], par[buf]);
        par[buf] ^= 1u;
        const int4 r = sr[buf][ri];
        if (r.x >= 0) {
            Acc a4[4], o[4];
            SRow<T>::load(&sA[buf][sa[buf][ri]][4 * row], a4);
            Acc b0[4], b1[4], b2[4], b3[4];
            SRow<T>::load(&sB[buf][ri][0], b0);
            SRow<T>::load(&sB[buf][ri][4], b1);
            SRow<T>::load(&sB[buf][ri][8], b2);
            SRow<T>::load(&sB[buf][ri][12], b3);
#pragma unroll
            for (int e = 0; e < 4; ++e) {
                Acc v = a4[0] * b0[e];
                v = fma_acc(a4[1], b1[e], v);
                v = fma_acc(a4[2], b2[e], v);
                v = fma_acc(a4[3], b3[e], v);
                o[e] = v;
            }
            const uint32_t nib = ((uint32_t)r.w >> (4 * row)) & 0xFu;
            const bool multi = (__ldg(mflag + (r.x >> 5)) >> (r.x & 31)) & 1u;
            const int64_t q = r.x;
            if (!multi) {
#pragma unroll
                for (int e = 0; e < 4; ++e) o[e] = ((nib >> e) & 1u) ? o[e] : Acc(0);
                if (hints & 2) RowCS<T>::store(cval + 16 * q + 4 * row, o);
                else RowIO<T>::store(cval + 16 * q + 4 * row, o);
            } else {
#pragma unroll
                for (int e = 0; e < 4; ++e)
                    if ((nib >> e) & 1u) atomicAdd(acc + 16 * q + 4 * row + e, o[e]);
            }
        }
        __syncthreads();  // buffer `buf` is refilled by the next iteration's producers
    }
}

// FP16: round the multi-product tiles from the FP32 workspace (+0.0 where the bit is clear)
template <typename T, typename Acc>
__global__ void k_plan_finalize(int64_t TC, const uint32_t* __restrict__ mflag, const uint16_t* __restrict__ cmap,
                                const Acc* __restrict__ gacc, T* __restrict__ cval) {
    const int64_t nw = (TC + 31) / 32;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nw; i += (int64_t)gridDim.x * blockDim.x) {
        uint32_t f = mflag[i];
        while (f) {
            const int b = __ffs(f) - 1;
            f &= f - 1;
            const int64_t q = 32 * i + b;
            const uint32_t mp = cmap[q];
#pragma unroll
            for (int e = 0; e < 16; ++e) cval[16 * q + e] = ((mp >> e) & 1u) ? from_acc<T>(gacc[16 * q + e]) : from_acc<T>(Acc(0));
        }
    }
}

template <typename T, typename Acc>
static amgt_status launch_numeric(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* C, Alloc& a) {
    cudaStream_t s = a.s;
    const int64_t BR = A->blc_row;
    if (BR == 0 || C->blc_num == 0) return AMGT_OK;
    SymCtx c{A->blc_ptr, A->blc_idx, A->blc_map, B->blc_ptr, B->blc_idx, B->blc_map};
    Scratch<int32_t> big, lng, mid;
    Scratch<unsigned long long> nbig;
    AMGT_TRY(big.init(a, BR));
    AMGT_TRY(lng.init(a, BR));
    AMGT_TRY(mid.init(a, BR));
    // [warp rows, long rows, long-row item cursor (pass 0), mid rows, mid-row cursor, long cursor (pass 1)]
    AMGT_TRY(nbig.init(a, 6));
    AMGT_CUDA(cudaMemsetAsync(nbig.p, 0, 6 * sizeof(unsigned long long), s));
    // tensor-core route off (every tile on CUDA cores): the staged kernel; else the kernel
    // with the DMMA / HMMA routes.  AMGT_NUM_STAGED=0 forces the latter (measurement).
    static const int staged_env = [] { const char* e = getenv("AMGT_NUM_STAGED"); return e ? atoi(e) : 1; }();
    const bool tc_route = (sizeof(T) == 8 || sizeof(T) == 2) && g_tc_thr_spgemm <= 16;
    // the symbolic phase's records for its dense rows (consumed here; used on the staged path)
    SpgemmPlan* plan = plan_take(C->blc_idx);
    struct PlanGuard {  // the plan stays with C (structure-only records) for later numeric calls
        SpgemmPlan*& p;
        cudaStream_t s;
        ~PlanGuard() {
            if (p) plan_put(p, s);
        }
    } plan_guard{plan, s};
    if (plan && (tc_route || !staged_env || plan->aptr != A->blc_ptr || plan->aidx != A->blc_idx ||
                 plan->bptr != B->blc_ptr || plan->TC != C->blc_num || plan->BR != BR)) {
        plan_free(plan, s);
        plan = nullptr;
    }
    static const int b1_env = [] { const char* e = getenv("AMGT_NUM_B1"); return e ? atoi(e) : 1; }();
    if (!tc_route && b1_env && B->row_max == 1 && C->row_max > 0 && C->row_max <= GROUP_NC &&
        B->blc_num < ((int64_t)1 << 31)) {
        // every B block row holds at most one tile (aggregation P): k_numeric_b1 over all rows
        return C->row_max <= 4 ? launch_b1<T, Acc, 4>(A, B, C, c, s) : launch_b1<T, Acc, GROUP_NC>(A, B, C, c, s);
    }
    if (!tc_route && staged_env) {
        static const int nbuf_env = [] { const char* e = getenv("AMGT_STAGED_NBUF"); return e ? atoi(e) : 2; }();
        const int nbuf = nbuf_env == 1 ? 1 : 2;
        const size_t sm = (size_t)STAGED_WARPS * 8 * nbuf * 4 * 2 * 16 * sizeof(T);
        const bool nc4 = C->row_max > 0 && C->row_max <= 4;
        auto kern = nc4 ? (nbuf == 2 ? k_numeric_staged<T, Acc, 4, 2> : k_numeric_staged<T, Acc, 4, 1>)
                        : (nbuf == 2 ? k_numeric_staged<T, Acc, GROUP_NC, 2> : k_numeric_staged<T, Acc, GROUP_NC, 1>);
        AMGT_CUDA(dyn_smem(kern, sm));
        // rows per group: several when rows are short (mean pairs per row ~ (T_A/BR_A)(T_B/BR_B)),
        // one when a row alone keeps the batch pipeline busy (and the grid large)
        const double mp = (BR ? (double)A->blc_num / BR : 0.0) * (B->blc_row ? (double)B->blc_num / B->blc_row : 0.0);
        const int rpg = (int)std::max(1.0, std::min((double)STAGED_RPG, std::floor(32.0 / std::max(mp, 1.0))));
        kern<<<(unsigned)ceil_div(ceil_div(BR, 8 * rpg), STAGED_WARPS), STAGED_WARPS * 32, sm, s>>>(
            BR, c, (const T*)A->blc_val, (const T*)B->blc_val, C->blc_ptr, C->blc_idx, C->blc_map, (T*)C->blc_val,
            big.p, nbig.p, lng.p, nbig.p + 1, mid.p, nbig.p + 3, rpg, plan ? plan->rowf : nullptr);
    } else {
        k_numeric_group<T, Acc><<<(unsigned)ceil_div(ceil_div(BR, 8) * 32, 256), 256, 0, s>>>(
            BR, c, (const T*)A->blc_val, (const T*)B->blc_val, C->blc_ptr, C->blc_idx, C->blc_map, (T*)C->blc_val,
            big.p, nbig.p, lng.p, nbig.p + 1, mid.p, nbig.p + 3, g_tc_thr_spgemm);
    }
    AMGT_LAUNCHED();
    if (plan) {  // the dense rows: one pass over the symbolic phase's records
        const bool det = plan->moff != nullptr;  // multi tiles summed in A-tile order (k_plan_msum)
        Scratch<Acc> pacc;  // FP16: FP32 workspace of the multi-product tiles (REDs path)
        Scratch<Acc> side_v;
        Scratch<int32_t> side_t;
        if (det) {
            AMGT_TRY(side_v.init(a, 16 * (size_t)std::max<int64_t>(plan->nmp, 1)));
            AMGT_TRY(side_t.init(a, (size_t)std::max<int64_t>(plan->nmp, 1)));
        } else if (sizeof(T) < sizeof(Acc)) {
            AMGT_TRY(pacc.init(a, 16 * (size_t)C->blc_num));
        }
        Acc* acc = sizeof(T) < sizeof(Acc) ? pacc.p : reinterpret_cast<Acc*>(C->blc_val);
        const int64_t nw = ceil_div(C->blc_num, 32);
        if (!det) {
            k_plan_zero<Acc><<<capped(ceil_div(nw, 256)), 256, 0, s>>>(C->blc_num, plan->mflag, acc);
            AMGT_LAUNCHED();
        }
        // L2 policies: bit 0 B tiles evict-last, bit 1 C stores evict-first (AMGT_PLAN_HINTS)
        static const int plan_hints = [] { const char* e = getenv("AMGT_PLAN_HINTS"); return e ? atoi(e) : 3; }();
        static int flat_per_sm = 0;
        if (!flat_per_sm) {
            AMGT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&flat_per_sm, k_plan_flat<T, Acc>, PLAN_R * 4, 0));
            flat_per_sm = max(flat_per_sm, 1);
        }
        static const int bulk_env = [] { const char* e = getenv("AMGT_PLAN_BULK"); return e ? atoi(e) : 0; }();  // measured slower (cfg4 1.80 vs 1.67 ms)
        if (bulk_env && !det) {  // (the bulk form has no slot path)
            static int bulk_per_sm = 0;
            if (!bulk_per_sm) {
                AMGT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bulk_per_sm, k_plan_flat_bulk<T, Acc>,
                                                                        PLAN_R * 4, 0));
                bulk_per_sm = max(bulk_per_sm, 1);
            }
            k_plan_flat_bulk<T, Acc><<<(unsigned)(num_sms() * bulk_per_sm), PLAN_R * 4, 0, s>>>(
                plan->nrec, plan->rec, plan->mflag, (const T*)A->blc_val, (const T*)B->blc_val, (T*)C->blc_val,
                sizeof(T) < sizeof(Acc) ? pacc.p : nullptr, plan_hints);
        } else
        if (det)
            k_plan_flat<T, Acc, true><<<(unsigned)(num_sms() * flat_per_sm), PLAN_R * 4, 0, s>>>(
                plan->nrec, plan->rec, plan->mflag, (const T*)A->blc_val, (const T*)B->blc_val, (T*)C->blc_val,
                nullptr, plan_hints, side_v.p, side_t.p);
        else
            k_plan_flat<T, Acc><<<(unsigned)(num_sms() * flat_per_sm), PLAN_R * 4, 0, s>>>(
                plan->nrec, plan->rec, plan->mflag, (const T*)A->blc_val, (const T*)B->blc_val, (T*)C->blc_val,
                sizeof(T) < sizeof(Acc) ? pacc.p : nullptr, plan_hints);
        AMGT_LAUNCHED();
        if (det) {
            k_plan_msum<T, Acc><<<capped(ceil_div(4 * std::max<int64_t>(C->blc_num / 8, 1), 256)), 256, 0, s>>>(
                plan->nm_dev, plan->mq, plan->moff, side_v.p, side_t.p, C->blc_map, (T*)C->blc_val);
            AMGT_LAUNCHED();
        } else if (sizeof(T) < sizeof(Acc)) {
            k_plan_finalize<T, Acc><<<capped(ceil_div(nw, 256)), 256, 0, s>>>(C->blc_num, plan->mflag, C->blc_map,
                                                                            pacc.p, (T*)C->blc_val);
            AMGT_LAUNCHED();
        }
    }
    // row classes present (C->row_max from symbolic; 0 = unknown: launch everything)
    int64_t rmax = C->row_max > 0 ? C->row_max : INT64_MAX;
    if (plan && plan->covers_all) rmax = std::min<int64_t>(rmax, CAP);  // longer rows: records only
    if (rmax <= GROUP_NC) return AMGT_OK;
    static int warp_per_sm = 0;  // resident CTAs of the warp kernel (per instantiation)
    if (!warp_per_sm) {
        AMGT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&warp_per_sm, k_numeric<T, Acc>, NUM_WARPS * 32, 0));
        warp_per_sm = max(warp_per_sm, 1);
    }
    k_numeric<T, Acc><<<(unsigned)(num_sms() * warp_per_sm), NUM_WARPS * 32, 0, s>>>(
        big.p, nbig.p, c, (const T*)A->blc_val, (const T*)B->blc_val, C->blc_ptr, C->blc_idx, C->blc_map,
        (T*)C->blc_val, nullptr, g_tc_thr_spgemm);  // rows <= CAP accumulate in shared memory
    AMGT_LAUNCHED();
    if (rmax <= CAP) return AMGT_OK;
    Scratch<Acc> gacc;  // FP16: FP32 accumulation workspace of the atomically accumulated rows
    if (sizeof(T) < sizeof(Acc)) AMGT_TRY(gacc.init(a, 16 * (size_t)C->blc_num));
    {
        int per_sm = 0;
        const size_t msm = MID_WARPS * (32 * 16 * sizeof(Acc) + 2 * MIDCAP * sizeof(int32_t));
        AMGT_CUDA(dyn_smem(k_numeric_mid<T, Acc>, msm));
        AMGT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_numeric_mid<T, Acc>, MID_WARPS * 32, msm));
        k_numeric_mid<T, Acc><<<(unsigned)num_sms() * (unsigned)max(per_sm, 1), MID_WARPS * 32, msm, s>>>(
            mid.p, nbig.p + 3, nbig.p + 4, c, (const T*)A->blc_val, (const T*)B->blc_val, C->blc_ptr, C->blc_idx,
            (T*)C->blc_val, sizeof(T) < sizeof(Acc) ? gacc.p : nullptr);
        AMGT_LAUNCHED();
    }
    const bool has_long = rmax > MIDCAP;
    if (has_long) {  // long rows: (row, LONG_PAIRS-pair chunk) work items over a persistent grid
        Scratch<int64_t> nch, choff;
        AMGT_TRY(nch.init(a, BR));
        AMGT_TRY(choff.init(a, BR + 1));
        Acc* ga = sizeof(T) < sizeof(Acc) ? gacc.p : nullptr;
        Scratch<int64_t> plen, pp;  // pairs per A tile of the long rows -> exclusive prefix
        AMGT_TRY(plen.init(a, A->blc_num));
        AMGT_TRY(pp.init(a, A->blc_num + 1));
        AMGT_CUDA(cudaMemsetAsync(plen.p, 0, A->blc_num * sizeof(int64_t), s));
        k_long_plen<<<(unsigned)num_sms() * 8, 256, 0, s>>>(lng.p, nbig.p + 1, c, plen.p);
        AMGT_LAUNCHED();
        AMGT_TRY(scan_exclusive(plen.p, pp.p, A->blc_num, a, s));
        k_long_prep<<<capped(ceil_div(BR, 256)), 256, 0, s>>>(BR, lng.p, nbig.p + 1, A->blc_ptr, pp.p, nch.p);
        AMGT_LAUNCHED();
        AMGT_TRY(scan_exclusive(nch.p, choff.p, BR, a, s));
        Scratch<int32_t> cnt;  // products per C tile (long rows)
        AMGT_TRY(cnt.init(a, C->blc_num));
        AMGT_CUDA(cudaMemsetAsync(cnt.p, 0, C->blc_num * sizeof(int32_t), s));
        // pair records: capacity for power-law rows (about one product per C tile); past it
        // (or past int32 indices) pass 1 re-derives the pairs instead
        const bool fits32 = C->blc_num < INT32_MAX && B->blc_num < INT32_MAX && A->blc_num < INT32_MAX;
        PairRec rec{nullptr, nullptr, nullptr, nullptr, fits32 ? 2 * C->blc_num + A->blc_num : -1};
        Scratch<int32_t> rq, rj, rt;
        Scratch<uint16_t> rm;
        if (fits32) {
            AMGT_TRY(rq.init(a, rec.cap));
            AMGT_TRY(rj.init(a, rec.cap));
            AMGT_TRY(rt.init(a, rec.cap));
            AMGT_TRY(rm.init(a, rec.cap));
            rec.q = rq.p; rec.j = rj.p; rec.t = rt.p; rec.m = rm.p;
        }
        const int64_t* pp_total = pp.p + A->blc_num;
        for (int pass = 0; pass < 2; ++pass) {
            // column samples (+ per-warp product staging in pass 1)
            const size_t sm = (size_t)LONG_SMEM * sizeof(int32_t) + (pass ? 8 * 32 * 16 * sizeof(Acc) : 0);
            auto kern = pass == 0 ? k_numeric_long<T, Acc, 0> : k_numeric_long<T, Acc, 1>;
            AMGT_CUDA(dyn_smem(kern, sm));
            int per_sm = 0;  // persistent grid: exactly the resident CTAs
            AMGT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 256, sm));
            kern<<<(unsigned)num_sms() * (unsigned)max(per_sm, 1), 256, sm, s>>>(
                lng.p, nbig.p + 1, choff.p, BR, pp.p, pp_total, nbig.p + 2 + 3 * pass, cnt.p, rec, c,
                (const T*)A->blc_val, (const T*)B->blc_val, C->blc_ptr, C->blc_idx, (T*)C->blc_val, ga);
            AMGT_LAUNCHED();
        }
        k_long_flat<T, Acc><<<(unsigned)num_sms() * 8, 256, 0, s>>>(pp_total, rec, cnt.p, (const T*)A->blc_val,
                                                                  (const T*)B->blc_val, (T*)C->blc_val, ga);
        AMGT_LAUNCHED();
    }
    if (sizeof(T) < sizeof(Acc)) {  // FP16: round the FP32 workspace (FP64/FP32 accumulate in place)
        Scratch<int64_t> nch, ccoff;
        AMGT_TRY(nch.init(a, BR));
        AMGT_TRY(ccoff.init(a, BR + 1));
        const int32_t* lists[2] = {mid.p, lng.p};
        const unsigned long long* counts[2] = {nbig.p + 3, nbig.p + 1};
        for (int l = 0; l < (has_long ? 2 : 1); ++l) {
            k_long_prep_c<<<capped(ceil_div(BR, 256)), 256, 0, s>>>(BR, lists[l], counts[l], C->blc_ptr, nch.p);
            AMGT_LAUNCHED();
            AMGT_TRY(scan_exclusive(nch.p, ccoff.p, BR, a, s));
            k_long_rows_finalize<T, Acc><<<(unsigned)num_sms() * 2, 256, 0, s>>>(
                lists[l], counts[l], ccoff.p, BR, C->blc_ptr, C->blc_map, (T*)C->blc_val, gacc.p);
            AMGT_LAUNCHED();
        }
    }
    return AMGT_OK;
}

amgt_status spgemm_numeric_impl(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* C, Alloc& a) {
    if (A->n != B->m || C->m != A->m || C->n != B->n) return fail(AMGT_ERR_ARG, "SpGEMM numeric: dimension mismatch");
    if (A->prec != B->prec || C->prec != A->prec) return fail(AMGT_ERR_ARG, "SpGEMM numeric: precision mismatch");
    TimerScope ts(TC_SPGEMM_NUM, spgemm_bytes(A, B, C, true), a.s);
    switch (A->prec) {
        case AMGT_FP64: return launch_numeric<double, double>(A, B, C, a);
        case AMGT_FP32: return launch_numeric<float, float>(A, B, C, a);
        default: return launch_numeric<__half, float>(A, B, C, a);
    }
}

}  // namespace amgt

using namespace amgt;

extern "C" {

amgt_status amgt_spgemm_symbolic(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* C, amgt_spgemm_info* info,
                                 const amgt_allocator* al, void* stream) {
    if (!A || !B || !C) return fail(AMGT_ERR_ARG, "amgt_spgemm_symbolic: NULL argument");
    Alloc a{al, (cudaStream_t)stream};
    return spgemm_symbolic_impl(A, B, C, info, a);
}

amgt_status amgt_spgemm_numeric(const amgt_mbsr* A, const amgt_mbsr* B, amgt_mbsr* C, void* stream) {
    if (!A || !B || !C) return fail(AMGT_ERR_ARG, "amgt_spgemm_numeric: NULL argument");
    Alloc a{nullptr, (cudaStream_t)stream};
    return spgemm_numeric_impl(A, B, C, a);
}

amgt_status amgt_rap(const amgt_mbsr* R, const amgt_mbsr* A, const amgt_mbsr* P, amgt_mbsr* Ac,
                     const amgt_allocator* al, void* stream) {
    if (!R || !A || !P || !Ac) return fail(AMGT_ERR_ARG, "amgt_rap: NULL argument");
    Alloc a{al, (cudaStream_t)stream};
    amgt_mbsr AP{};
    AMGT_TRY(spgemm_symbolic_impl(A, P, &AP, nullptr, a));
    amgt_status st = spgemm_numeric_impl(A, P, &AP, a);
    if (st == AMGT_OK) st = spgemm_symbolic_impl(R, &AP, Ac, nullptr, a);
    if (st == AMGT_OK) {
        st = spgemm_numeric_impl(R, &AP, Ac, a);
        if (st != AMGT_OK) mbsr_release(Ac, a);
    }
    mbsr_release(&AP, a);
    return st;
}

}  // extern "C"
