// tsg_step1.cu -- SURVEY §8(a) rows a0 (helper indices) and a1 (step 1 of Section 3.3).
//
// Step 1 of the paper computes the tile layout of C by a structural SpGEMM C' = A'B'
// and step 2 then intersects tile index sets per C tile (Alg 2 l.4-18).  Here both
// come out of one exact per-tile-row pass: each A tile enumerates its candidate B
// tiles (whole B tile row, or the B row list of its single column), a CTA per tile row sorts the
// row's candidates by tile column J (stable, so pairs stay in ascending K), and the heads of
// equal-J runs are the non-empty C tiles.  Pairs without products (colOcc(A)&rowOcc(B) == 0) are
// dropped (reading B3), so C never stores an empty tile (reading A6).
#include <algorithm>

#include "tsg_device.cuh"

namespace tsg {
namespace {

constexpr unsigned FULL = 0xffffffffu;
enum RowClass : uint8_t { ROW_EMPTY = 0, ROW_SMALL = 1, ROW_BIG = 2, ROW_MERGE = 3 };

__device__ __forceinline__ int bits_for(uint64_t v) {  // bits needed to represent v (>= 1)
    return v ? 64 - __clzll((long long)v) : 1;
}

// ------------------------------------------------------------------------------------------
// a0: occupancy words.  rowOcc bit r = row r non-empty; colOcc = OR of the 16 row masks.
// A pair (A_IK, B_KJ) has a product iff colOcc(A_IK) & rowOcc(B_KJ) != 0.
// ------------------------------------------------------------------------------------------
__global__ void k_occupancy(const uint16_t *__restrict__ mask, int64_t nt, uint16_t *__restrict__ row_occ,
                            uint16_t *__restrict__ col_occ, uint64_t *__restrict__ zero, int zero_words) { TSG_GRID_WAIT();
    if (blockIdx.x == 0)  // the call's device counters start at zero (saves a memset launch)
        for (int i = threadIdx.x; i < zero_words; i += blockDim.x) zero[i] = 0;
    int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= nt) return;
    const uint4 *p = reinterpret_cast<const uint4 *>(mask + t * TILE);
    uint4 a = __ldg(p), b = __ldg(p + 1);
    uint32_t w[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
    uint32_t ro = 0, co = 0;
#pragma unroll
    for (int k = 0; k < 8; k++) {
        uint32_t lo = w[k] & 0xffffu, hi = w[k] >> 16;
        ro |= (lo ? 1u : 0u) << (2 * k);
        ro |= (hi ? 1u : 0u) << (2 * k + 1);
        co |= lo | hi;
    }
    if (row_occ) row_occ[t] = (uint16_t)ro;
    if (col_occ) col_occ[t] = (uint16_t)co;
}

// per-tile records of a hypersparse operand (TileRec, tsg_kernels.cuh)
template <typename TI>
__global__ void k_tile_records(int64_t nt, const int32_t *__restrict__ tile_col, const int64_t *__restrict__ tile_nnz,
                               const uint16_t *__restrict__ mask, const uint8_t *__restrict__ idx,
                               const TI *__restrict__ val, TileRec *__restrict__ rec) { TSG_GRID_WAIT();
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= nt) return;
    const uint4 *p = reinterpret_cast<const uint4 *>(mask + t * TILE);
    const uint4 a = __ldg(p), b = __ldg(p + 1);
    const uint32_t w8[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
    uint32_t ro = 0;
#pragma unroll
    for (int k = 0; k < 8; k++) ro |= ((w8[k] & 0xffffu) ? 1u : 0u) << (2 * k) | ((w8[k] >> 16) ? 1u : 0u) << (2 * k + 1);
    const int64_t z0 = tile_nnz[t], z1 = tile_nnz[t + 1];
    TileRec r;
    r.col = tile_col[t];
    if (z1 - z0 == 1) {
        uint64_t bits = 0;
        const TI x = val[z0];
        memcpy(&bits, &x, sizeof(TI));
        r.v = bits;
        r.w = ro | (uint32_t)idx[z0] << 16 | 1u << 24;
    } else {
        r.v = (uint64_t)z0;
        r.w = ro;
    }
    rec[t] = r;
}

// B row lists ("mode ii"): for each global row k of B, the B tiles of tile row k/16 whose row
// k%16 is non-empty, ascending tile column.  One warp = two B tile rows, lane r = row r.
__global__ void __launch_bounds__(256) k_rowlist(int64_t tmB, const int64_t *__restrict__ tpB,
                                                 const uint16_t *__restrict__ maskB, const int64_t *__restrict__ lptr,
                                                 int32_t *__restrict__ lcnt, uint32_t *__restrict__ list,
                                                 const int32_t *__restrict__ tcB, int32_t *__restrict__ listJ) { TSG_GRID_WAIT();
    const int lane = threadIdx.x & 31, r = lane & 15;
    const int64_t K = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 2 + (lane >> 4);
    if (K >= tmB) return;
    const int64_t t0 = tpB[K], t1 = tpB[K + 1];
    if (!list) {
        int c = 0;
        for (int64_t t = t0; t < t1; t++) c += maskB[t * TILE + r] != 0;
        lcnt[K * TILE + r] = c;
    } else {
        // the entries' tile columns alongside (step 1 reads them without a dependent lookup)
        int64_t pos = lptr[K * TILE + r];
        for (int64_t t = t0; t < t1; t++)
            if (maskB[t * TILE + r]) {
                list[pos] = (uint32_t)t;
                listJ[pos++] = tcB[t];
            }
    }
}

// stats only: nnz of every global row of B, then products per A tile
__global__ void __launch_bounds__(256) k_brow_nnz(int64_t tmB, const int64_t *__restrict__ tpB,
                                                  const uint16_t *__restrict__ maskB, int32_t *__restrict__ rnnz) { TSG_GRID_WAIT();
    const int lane = threadIdx.x & 31, r = lane & 15;
    const int64_t K = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 2 + (lane >> 4);
    if (K >= tmB) return;
    int c = 0;
    for (int64_t t = tpB[K]; t < tpB[K + 1]; t++) c += __popc(maskB[t * TILE + r]);
    rnnz[K * TILE + r] = c;
}

__global__ void k_products(int64_t ntA, const int32_t *__restrict__ tcA, const uint16_t *__restrict__ maskA,
                           const int32_t *__restrict__ rnnz, DevCounters *cnt) { TSG_GRID_WAIT();
    int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    u64c p = 0;
    if (t < ntA) {
        int64_t K = tcA[t];
        for (int r = 0; r < TILE; r++) {
            uint32_t m = maskA[t * TILE + r];
            while (m) {
                int c = __ffs(m) - 1;
                m &= m - 1;
                p += rnnz[K * TILE + c];
            }
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) p += __shfl_xor_sync(FULL, p, o);
    if ((threadIdx.x & 31) == 0 && p) atomicAdd(&cnt->products, p);
}

// ------------------------------------------------------------------------------------------
// diagnostic (TSG_STATS_STRUCTURAL): |C'| of the paper's step 1, the structural tile product A'B'
// with its empty tiles: per tile row, the distinct tile columns J over
// every B tile of every B tile row K with A_IK stored, marked in a shared-memory bitmap.
// ------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_structural(const int64_t *__restrict__ tpA, const int32_t *__restrict__ tcA,
                                                   const int64_t *__restrict__ tpB, const int32_t *__restrict__ tcB,
                                                   int words, DevCounters *cnt) { TSG_GRID_WAIT();
    extern __shared__ uint32_t bm[];
    const int64_t I = blockIdx.x;
    for (int w = threadIdx.x; w < words; w += blockDim.x) bm[w] = 0;
    __syncthreads();
    for (int64_t a = tpA[I]; a < tpA[I + 1]; a++) {
        const int64_t K = tcA[a];
        for (int64_t b = tpB[K] + threadIdx.x; b < tpB[K + 1]; b += blockDim.x) {
            const uint32_t J = (uint32_t)tcB[b];
            atomicOr(&bm[J >> 5], 1u << (J & 31));
        }
    }
    __syncthreads();
    u64c c = 0;
    for (int w = threadIdx.x; w < words; w += blockDim.x) c += __popc(bm[w]);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) c += __shfl_xor_sync(FULL, c, o);
    if ((threadIdx.x & 31) == 0 && c) atomicAdd(&cnt->structural, c);
}

// ------------------------------------------------------------------------------------------
// multi-GPU partition: intermediate products per tile row of A*B -- a warp per
// tile row, lane = one A tile, sum over its nonzeros (r,c) of nnz(B row 16K + c) -- and the cuts
// at equal shares of their prefix sum (searchsorted-left of g*total/parts, monotone)
// ------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_row_products(int64_t tmA, const int64_t *__restrict__ tpA,
                                                     const int32_t *__restrict__ tcA, const uint16_t *__restrict__ maskA,
                                                     const int32_t *__restrict__ rnnz, int64_t *__restrict__ w) { TSG_GRID_WAIT();
    const int lane = threadIdx.x & 31;
    const int64_t I = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (I >= tmA) return;
    int64_t p = 0;
    for (int64_t t = tpA[I] + lane; t < tpA[I + 1]; t += 32) {
        const int64_t K = tcA[t];
        for (int r = 0; r < TILE; r++) {
            uint32_t m = maskA[t * TILE + r];
            while (m) {
                const int c = __ffs(m) - 1;
                m &= m - 1;
                p += rnnz[K * TILE + c];
            }
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) p += __shfl_xor_sync(FULL, p, o);
    if (lane == 0) w[I] = p;
}

__global__ void k_cuts(const int64_t *__restrict__ pre, int64_t tm, int64_t parts, int64_t *__restrict__ cuts) { TSG_GRID_WAIT();
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const int64_t total = pre[tm];
    int64_t prev = 0;
    cuts[0] = 0;
    for (int64_t g = 1; g < parts; g++) {
        // first i with pre[i] >= g * total / parts, i.e. pre[i] * parts >= g * total (exact)
        int64_t lo = 0, hi = tm;
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if ((__int128)pre[mid] * parts >= (__int128)g * total) hi = mid;
            else lo = mid + 1;
        }
        prev = max(prev, lo);
        cuts[g] = prev;
    }
    cuts[parts] = tm;
}

// ------------------------------------------------------------------------------------------
// a1 (plan): per A tile, how its candidate B tiles are enumerated.
//   scan mode: every tile of B tile row K (filtered later by occupancy);
//   list mode: when A_IK touches a single column c, exactly the B row list of k = 16K + c
//              (all of them contribute, no filter, no duplicates).
// cost = number of candidates; start encodes the mode (list: -(start+1)).
// ------------------------------------------------------------------------------------------
__global__ void k_atile_plan(int64_t ntA, const int32_t *__restrict__ tcA, const uint16_t *__restrict__ colOccA,
                             const int64_t *__restrict__ tpB, const int32_t *__restrict__ tcB,
                             const int64_t *__restrict__ lptr, const uint32_t *__restrict__ list,
                             const int32_t *__restrict__ listJ, bool scan_only,
                             int64_t *__restrict__ cost, int64_t *__restrict__ start, int32_t *__restrict__ jlo,
                             int32_t *__restrict__ jhi, DevCounters *cnt) { TSG_GRID_WAIT();
    int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    bool is_list = false;
    if (t < ntA) {
        const int64_t K = tcA[t];
        const uint32_t co = colOccA[t];
        int64_t b0 = tpB[K], len = tpB[K + 1] - b0, st = b0;
        if (!scan_only && lptr && __popc(co) == 1) {
            int64_t k = K * TILE + (__ffs(co) - 1);
            int64_t l0 = lptr[k], ll = lptr[k + 1] - l0;
            if (ll < len) {
                is_list = true;
                len = ll;
                st = l0;
            }
        }
        cost[t] = len;
        start[t] = is_list ? -(st + 1) : st;
        if (len > 0) {
            jlo[t] = is_list ? listJ[st] : tcB[st];
            jhi[t] = is_list ? listJ[st + len - 1] : tcB[st + len - 1];
        } else {
            jlo[t] = 0x7fffffff;
            jhi[t] = -1;
        }
    }
    unsigned b = __ballot_sync(FULL, is_list);
    if ((threadIdx.x & 31) == 0 && b) atomicAdd(&cnt->list_tiles, (u64c)__popc(b));
}

// a1 (row plan): candidate window and class of every tile row (one warp per row)
__global__ void k_row_plan(int64_t tmA, const int64_t *__restrict__ tpA, const int64_t *__restrict__ costOff,
                           const int32_t *__restrict__ jloA, const int32_t *__restrict__ jhiA, bool merge,
                           int32_t *__restrict__ rowJlo, int32_t *__restrict__ rowJhi, uint8_t *__restrict__ rowClass,
                           int64_t *__restrict__ nC, int32_t *__restrict__ bigList, int64_t *__restrict__ bigOff,
                           int32_t *__restrict__ smallList, DevCounters *cnt) { TSG_GRID_WAIT();
    const int lane = threadIdx.x & 31;
    const int64_t I = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (I >= tmA) return;
    const int64_t a0 = tpA[I], a1 = tpA[I + 1];
    int lo = 0x7fffffff, hi = -1;
    for (int64_t t = a0 + lane; t < a1; t += 32) {
        lo = min(lo, jloA[t]);
        hi = max(hi, jhiA[t]);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        lo = min(lo, __shfl_xor_sync(FULL, lo, o));
        hi = max(hi, __shfl_xor_sync(FULL, hi, o));
    }
    if (lane) return;
    const int64_t U = costOff[a1] - costOff[a0];
    rowJlo[I] = lo;
    rowJhi[I] = hi;
    if (U == 0 || hi < lo) {
        rowClass[I] = ROW_EMPTY;
        nC[I] = 0;
        return;
    }
    if (merge && a1 - a0 <= MERGE_MAX_A) {
        rowClass[I] = ROW_MERGE;
        atomicAdd(&cnt->nmerge, 1ULL);
        return;
    }
    const int wb = bits_for((uint64_t)(hi - lo + 1));  // valid 0..hi-lo, sentinel hi-lo+1
    const int ub = bits_for((uint64_t)(U > 1 ? U - 1 : 1));
    if (U <= ROW_CAP && wb + ub <= 32 && (a1 - a0) < 65536) {
        rowClass[I] = ROW_SMALL;
        atomicMax(&cnt->max_u_small, (u64c)U);
        smallList[atomicAdd(&cnt->nsmall, 1ULL)] = (int32_t)I;
    } else {
        rowClass[I] = ROW_BIG;
        u64c k = atomicAdd(&cnt->nbig, 1ULL);
        bigList[k] = (int32_t)I;
        bigOff[I] = (int64_t)atomicAdd(&cnt->big_u, (u64c)U);
    }
}

__device__ __forceinline__ int block_scan_int(int v, int *total, int *sm /* ROW_NW+1 ints */) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int incl = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        int o = __shfl_up_sync(FULL, incl, d);
        if (lane >= d) incl += o;
    }
    if (lane == 31) sm[w] = incl;
    __syncthreads();
    if (threadIdx.x == 0) {
        int s = 0;
        for (int k = 0; k < ROW_NW; k++) {
            int x = sm[k];
            sm[k] = s;
            s += x;
        }
        sm[ROW_NW] = s;
    }
    __syncthreads();
    int res = sm[w] + incl - v;
    *total = sm[ROW_NW];
    __syncthreads();
    return res;
}

// in-place exclusive scan of hist[0..L) (L <= 256*ROW_NW) by the CTA
__device__ void block_scan_array(uint32_t *hist, int L, int *sm) {
    const int per = (L + ROW_T - 1) / ROW_T;
    const int b = threadIdx.x * per, e = min(L, b + per);
    int s = 0;
    for (int i = b; i < e; i++) s += hist[i];
    int tot;
    int pre = block_scan_int(s, &tot, sm);
    for (int i = b; i < e; i++) {
        int x = hist[i];
        hist[i] = pre;
        pre += x;
    }
    __syncthreads();
}

// stable LSD radix sort of a[0..n) on bits [lo, lo+nbits); returns the buffer holding the result
template <typename K>
__device__ K *block_radix_sort(K *a, K *b, int64_t n, int lo, int nbits, uint32_t *hist, int *sm) {
    if (nbits <= 0 || n <= 1) return a;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int passes = (nbits + 7) / 8;
    const int dbits = (nbits + passes - 1) / passes;
    const int64_t per = (((n + ROW_NW - 1) / ROW_NW) + 31) & ~(int64_t)31;
    const int64_t w0 = min(n, (int64_t)w * per), w1 = min(n, w0 + per);
    const unsigned lt = (1u << lane) - 1u;
    for (int p = 0; p < passes; p++) {
        const int shift = lo + p * dbits;
        const int bits = min(dbits, nbits - p * dbits);
        const uint32_t B = 1u << bits, dm = B - 1u;
        for (uint32_t i = threadIdx.x; i < B * ROW_NW; i += ROW_T) hist[i] = 0;
        __syncthreads();
        for (int64_t base = w0; base < w1; base += 32) {
            const int64_t i = base + lane;
            const bool v = i < w1;
            const uint32_t d = v ? (uint32_t)((a[i] >> shift) & dm) : B;
            const unsigned peers = __match_any_sync(FULL, d);
            if (v && lane == __ffs(peers) - 1) hist[d * ROW_NW + w] += __popc(peers);
            __syncwarp();
        }
        __syncthreads();
        block_scan_array(hist, (int)(B * ROW_NW), sm);
        for (int64_t base = w0; base < w1; base += 32) {
            const int64_t i = base + lane;
            const bool v = i < w1;
            K key = v ? a[i] : (K)0;
            const uint32_t d = v ? (uint32_t)((key >> shift) & dm) : B;
            const unsigned peers = __match_any_sync(FULL, d);
            if (v) b[hist[d * ROW_NW + w] + __popc(peers & lt)] = key;
            __syncwarp();
            if (v && lane == __ffs(peers) - 1) hist[d * ROW_NW + w] += __popc(peers);
            __syncwarp();
        }
        __syncthreads();
        K *t = a;
        a = b;
        b = t;
    }
    return a;
}

template <typename K, typename KP>
__device__ void row_sort_body(const S1Params &P, int64_t I, K *keysA, K *keysB, uint32_t *posB_s, KP *kpos_s,
                              uint32_t *hist, int *sm, int ub) {
    const int64_t a0 = P.tpA[I], a1 = P.tpA[I + 1];
    const int nA = (int)(a1 - a0);
    const int64_t base = P.costOff[a0];
    const int64_t U = P.costOff[a1] - base;
    const int jlo = P.rowJlo[I];
    const uint32_t W = (uint32_t)(P.rowJhi[I] - jlo + 1);  // sentinel value for invalid candidates
    const int wb = bits_for(W);
    const K umask = (K)(((uint64_t)1 << ub) - 1);

    // expansion (load-balanced over the row's candidates)
    int nv = 0;
    for (int64_t u = threadIdx.x; u < U; u += ROW_T) {
        const int64_t target = base + u;
        int lo = 0, hi = nA - 1;
        while (lo < hi) {
            int mid = (lo + hi + 1) >> 1;
            if (P.costOff[a0 + mid] <= target) lo = mid;
            else hi = mid - 1;
        }
        const int64_t t = a0 + lo;
        const int64_t s = target - P.costOff[t];
        const int64_t st = P.startA[t];
        uint32_t posB;
        bool valid;
        if (st < 0) {
            posB = P.list[-st - 1 + s];
            valid = true;
        } else {
            posB = (uint32_t)(st + s);
            valid = (P.rowOccB[posB] & P.colOccA[t]) != 0;
        }
        const uint32_t jr = valid ? (uint32_t)(P.tcB[posB] - jlo) : W;
        keysA[u] = ((K)jr << ub) | (K)u;
        posB_s[u] = posB;
        kpos_s[u] = (KP)lo;
        nv += valid;
    }
    int nvalid;
    block_scan_int(nv, &nvalid, sm);

    K *R = block_radix_sort<K>(keysA, keysB, U, ub, wb, hist, sm);

    // heads: blocked ownership so ranks follow from one CTA scan
    const int64_t ipt = (nvalid + ROW_T - 1) / ROW_T;
    const int64_t i0 = min((int64_t)nvalid, (int64_t)threadIdx.x * ipt), i1 = min((int64_t)nvalid, i0 + ipt);
    int h = 0;
    {
        int64_t prev = (i0 > 0) ? (int64_t)(R[i0 - 1] >> ub) : -1;
        for (int64_t i = i0; i < i1; i++) {
            int64_t jr = (int64_t)(R[i] >> ub);
            h += (jr != prev);
            prev = jr;
        }
    }
    int nCrow;
    int rank = block_scan_int(h, &nCrow, sm);
    {
        int64_t prev = (i0 > 0) ? (int64_t)(R[i0 - 1] >> ub) : -1;
        for (int64_t i = i0; i < i1; i++) {
            const K key = R[i];
            const int64_t jr = (int64_t)(key >> ub);
            const int64_t u = (int64_t)(key & umask);
            const uint64_t pA = (uint64_t)(a0 + (int64_t)kpos_s[u]);
            P.pairs[base + i] = (pA << 32) | (uint64_t)posB_s[u];
            if (jr != prev) {
                P.tJ[base + rank] = jlo + (int32_t)jr;
                P.tStart[base + rank] = (uint32_t)i;
                rank++;
            }
            prev = jr;
        }
    }
    __syncthreads();
    for (int r = threadIdx.x; r < nCrow; r += ROW_T) {
        const uint32_t b = P.tStart[base + r];
        const uint32_t e = (r + 1 < nCrow) ? P.tStart[base + r + 1] : (uint32_t)nvalid;
        P.tCnt[base + r] = e - b;
        // work estimate for step 2's class split: number of (pair, c) items, i.e. columns c of
        // A_IK whose B_KJ row c is non-empty
        uint32_t w = 0;
        for (uint32_t i = b; i < e; i++) {
            const int64_t u = (int64_t)(R[i] & umask);
            w += __popc((uint32_t)P.colOccA[a0 + (int64_t)kpos_s[u]] & (uint32_t)P.rowOccB[posB_s[u]]);
        }
        P.tWork[base + r] = w;
    }
    if (threadIdx.x == 0) {
        P.nC[I] = nCrow;
        atomicAdd(&P.cnt->pairs, (u64c)nvalid);
    }
}

// ------------------------------------------------------------------------------------------
// a1 (merge): tile rows with at most 32 A tiles.  Lane l owns A tile a0+l; its candidate B tiles
// (scan mode: B tile row K; list mode: the B row list) are already sorted by tile column J, so
// the row's C tiles are a k-way merge of <= 32 sorted lists: per step the warp takes the minimum
// head J (redux), the lanes holding J (ballot, lane order = ascending K) are that C tile's pairs,
// and they advance.  Candidates without products are skipped lane-locally (reading B3).  Same
// outputs, in the same candidate-space slots, as the expand/radix-sort path below; no shared
// memory, no barriers, one step per C tile.
// ------------------------------------------------------------------------------------------
// C tile records of a merge: lane (n & 31) keeps step n's record, flushed 32 at a time (coalesced)
struct MergeOut {
    uint32_t rJ = 0, rS = 0, rC = 0, rW = 0, np = 0, ntl = 0;
    __device__ __forceinline__ void emit(const S1Params &P, int64_t base, int lane, uint32_t J, unsigned hm,
                                         uint32_t ws) {
        if (lane == (int)(ntl & 31)) {
            rJ = J;
            rS = np;
            rC = (uint32_t)__popc(hm);
            rW = ws;
        }
        np += (uint32_t)__popc(hm);
        ntl++;
        if ((ntl & 31) == 0) flush(P, base, lane, 32);
    }
    __device__ __forceinline__ void flush(const S1Params &P, int64_t base, int lane, uint32_t n) {
        if (lane < (int)n) {
            const int64_t o = base + ((ntl - 1) & ~31u) + lane;
            P.tJ[o] = (int32_t)rJ;
            P.tStart[o] = rS;
            P.tCnt[o] = rC;
            P.tWork[o] = rW;
        }
    }
    __device__ __forceinline__ void finish(const S1Params &P, int64_t base, int lane, int64_t I) {
        if (ntl & 31) flush(P, base, lane, ntl & 31);
        if (lane == 0) {
            P.nC[I] = ntl;
            atomicAdd(&P.cnt->pairs, (u64c)np);
        }
    }
};

#ifndef TSG_MERGE_W
#define TSG_MERGE_W 4
#endif
constexpr int MERGE_W = TSG_MERGE_W;  // warps (tile rows) per merge CTA
#ifndef TSG_MERGE_CAP
#define TSG_MERGE_CAP 768
#endif
constexpr int MERGE_CAP = TSG_MERGE_CAP;  // candidates of a row staged in shared memory (6 B each)

// One tile row's merge by one warp (sJw / sKw: the warp's MERGE_CAP staging slots).  Writes the
// row's pairs and C tile records at its candidate-space slots; returns the row's C tile count
// (warp-uniform).
__device__ uint32_t merge_row(const S1Params &P, int64_t I, int lane, uint32_t *sJrow, uint16_t *sKrow) {
    constexpr uint32_t INF = 0xffffffffu;
    constexpr uint32_t JM = (1u << 27) - 1u;  // tile column bits (n < 2^31); bits 27..31: work
    const int64_t a0 = P.tpA[I], a1 = P.tpA[I + 1];
    const int64_t base = P.costOff[a0];
    const int64_t U = P.costOff[a1] - base;
    const int64_t t = a0 + lane;
    int64_t len = 0, st = 0, off = 0;
    bool isl = false;
    uint32_t co = 0;
    if (t < a1) {
        off = P.costOff[t] - base;
        len = P.costOff[t + 1] - base - off;
        st = P.startA[t];
        isl = st < 0;
        if (isl) st = -st - 1;
        co = P.colOccA[t];
    }
    const unsigned lt = (1u << lane) - 1u;
    MergeOut out;
    if (U <= MERGE_CAP && P.tnB < (int64_t)JM) {
        // stage: each lane walks its own candidate list (a B tile row, or a B row list: no search
        // for the owner) and keeps, in order, those with a product (reading B3): tile column +
        // work in the top bits, and the candidate's index k (16 bits; the B tile position is
        // st + k, or list[st + k] in list mode).  Four candidates per lane in flight.
        // (32-bit indices: the row's candidates fit the stage, B tile positions fit 31 bits)
        const int ioff = (int)off, ilen = (int)len;
        const uint32_t st32 = (uint32_t)st;
        const uint32_t *lst = isl ? P.list + st : nullptr;
        uint32_t *sJw = sJrow + ioff;
        uint16_t *sKw = sKrow + ioff;
        int cntv = 0;
#pragma unroll 4
        for (int k = 0; k < ilen; k++) {
            const uint32_t pos = isl ? lst[k] : st32 + (uint32_t)k;
            const uint32_t wk = isl ? 1u : (uint32_t)__popc(co & (uint32_t)P.rowOccB[pos]);
            if (wk) {
                sJw[cntv] = (uint32_t)(isl ? P.listJ[st + k] : P.tcB[pos]) | (wk << 27);
                sKw[cntv] = (uint16_t)k;
                cntv++;
            }
        }
        __syncwarp();
        const int vlen = cntv;
        const uint32_t *mj = sJw;
        int s = 0;
        uint32_t hv = vlen > 0 ? mj[0] : INF;
        auto adv = [&]() { hv = s < vlen ? mj[s] : INF; };
        uint64_t *pout = P.pairs + base;
        const uint64_t thi = (uint64_t)t << 32;
        for (;;) {
            const uint32_t J = __reduce_min_sync(FULL, hv & JM);
            if (J == JM) break;  // every lane exhausted (INF & JM == JM > any tile column)
            const bool hit = hv != INF && (hv & JM) == J;
            const unsigned hm = __ballot_sync(FULL, hit);
            const uint32_t ws = __reduce_add_sync(FULL, hit ? hv >> 27 : 0u);
            if (hit) {
                const uint32_t k = sKw[s];
                const uint32_t pos = isl ? lst[k] : st32 + k;
                pout[out.np + (uint32_t)__popc(hm & lt)] = thi | pos;
            }
            out.emit(P, base, lane, J, hm, ws);
            if (hit) {
                s++;
                adv();
            }
        }
        out.finish(P, base, lane, I);
        return out.ntl;
    }
    // rows with more candidates than the stage holds: each lane keeps four candidates in flight
    constexpr uint32_t JINF = 0x7fffffffu;
    int64_t s = 0;
    uint32_t bJ[4], bP[4], bO[4];
    int bn = 0;
    uint32_t head = JINF, hpos = 0, hocc = 0;
    auto advance = [&]() {
        for (;;) {
            if (bn == 0) {
                if (s >= len) {
                    head = JINF;
                    return;
                }
#pragma unroll
                for (int k = 0; k < 4; k++) {
                    const bool v = s + k < len;
                    uint32_t pos = 0;
                    if (v) pos = isl ? P.list[st + s + k] : (uint32_t)(st + s + k);
                    bP[k] = pos;
                    bJ[k] = v ? (uint32_t)P.tcB[pos] : JINF;
                    bO[k] = v ? (uint32_t)P.rowOccB[pos] : 0u;
                }
                bn = (int)min((int64_t)4, len - s);
                s += bn;
            }
            const uint32_t J = bJ[0], pos = bP[0], occ = bO[0];
            bJ[0] = bJ[1]; bJ[1] = bJ[2]; bJ[2] = bJ[3];
            bP[0] = bP[1]; bP[1] = bP[2]; bP[2] = bP[3];
            bO[0] = bO[1]; bO[1] = bO[2]; bO[2] = bO[3];
            bn--;
            if (isl || (occ & co)) {
                head = J;
                hpos = pos;
                hocc = occ;
                return;
            }
        }
    };
    advance();
    for (;;) {
        const uint32_t J = __reduce_min_sync(FULL, head);
        if (J == JINF) break;
        const bool hit = head == J;
        const unsigned hm = __ballot_sync(FULL, hit);
        const uint32_t ws = __reduce_add_sync(FULL, hit ? (isl ? 1u : (uint32_t)__popc(co & hocc)) : 0u);
        if (hit) P.pairs[base + out.np + __popc(hm & lt)] = ((uint64_t)t << 32) | hpos;
        out.emit(P, base, lane, J, hm, ws);
        if (hit) advance();
    }
    out.finish(P, base, lane, I);
    return out.ntl;
}

#ifndef TSG_MERGE_MINB
#define TSG_MERGE_MINB 1
#endif
__global__ void __launch_bounds__(MERGE_W * 32, TSG_MERGE_MINB) k_row_merge(S1Params P, int64_t tm) { TSG_GRID_WAIT();
    __shared__ uint32_t sJ[MERGE_W][MERGE_CAP];
    __shared__ uint16_t sK[MERGE_W][MERGE_CAP];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t I = (int64_t)blockIdx.x * MERGE_W + w;
    if (I >= tm || P.rowClass[I] != ROW_MERGE) return;  // warp-uniform
    if (*P.utot > P.capU) {  // (scratch_fits, per warp)
        if (lane == 0) P.cnt->overflow = 1;
        return;
    }
    merge_row(P, I, lane, sJ[w], sK[w]);
}

// ------------------------------------------------------------------------------------------
// a2 on the row path (every tile row has <= 32 A tiles).  One warp per tile row: with the row's A
// masks staged once in shared memory, each C tile's bit masks are OR-ed from its pairs (written by
// step 1 at the row's candidate-space slots; Alg 2 l.19-25: mask_C[r] |= mask_B[c]
// for every nonzero (r,c) of A_IK) by a half warp with lane r owning row r (no atomics), followed
// by the 16-entry row offsets and the tile nnz.  Results stay at the row's candidate-space slots
// (C is allocated once, after this kernel); the row's nnz total goes to rowNnz[I] for
// the row-offset scan, the count of dense C tiles to the call's counters.
// ------------------------------------------------------------------------------------------
constexpr int SYM_SMEM = 1024 + 2 * 576;  // per warp: A row masks [32][16], two half-warp batches
__global__ void __launch_bounds__(MERGE_W * 32) k_sym_rows(S1Params P, int64_t tm) { TSG_GRID_WAIT();
    __shared__ __align__(16) unsigned char sR[MERGE_W][SYM_SMEM];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int64_t I = (int64_t)blockIdx.x * MERGE_W + w;
    if (I >= tm) return;  // warp-uniform
    if (P.rowClass[I] != ROW_MERGE) {  // empty row (the row path runs only when no other class exists)
        if (lane == 0) P.rowNnz[I] = 0;
        return;
    }
    const uint32_t nC = (uint32_t)P.nC[I];  // step 1 (k_row_merge) wrote the row's C tiles and pairs
    const int64_t a0 = P.tpA[I];
    const int nA = (int)(P.tpA[I + 1] - a0);
    const int64_t base = P.costOff[a0];
    // staging area (reuses the merge's): A row masks [32][16], then per half warp the B masks,
    // B row occupancy and A slots of a batch of 16 pairs
    unsigned char *wsm = sR[w];
    uint16_t *sMA = reinterpret_cast<uint16_t *>(wsm);
    if (lane < nA) {
        const uint4 *g = reinterpret_cast<const uint4 *>(P.mA + (a0 + lane) * TILE);
        uint4 *d = reinterpret_cast<uint4 *>(sMA + lane * TILE);
        d[0] = g[0];
        d[1] = g[1];
    }
    const int r = lane & 15, half = lane >> 4;
    unsigned char *hs = wsm + 1024 + half * 576;
    uint16_t *sMB = reinterpret_cast<uint16_t *>(hs);        // [16][16]
    uint16_t *sOB = reinterpret_cast<uint16_t *>(hs + 512);  // [16]
    uint8_t *sS = hs + 544;                                  // [16]
    __syncwarp();
    int64_t rownnz = 0;
    uint32_t ndense = 0;
    for (uint32_t q0 = 0; q0 < nC; q0 += 2) {
        const uint32_t q = q0 + half;
        const bool hv = q < nC;
        uint32_t st = 0, cnt = 0;
        if (hv) {
            st = P.tStart[base + q];
            cnt = P.tCnt[base + q];
        }
        uint32_t acc = 0;
        const uint32_t nbat = (cnt + 15) / 16;
        const uint32_t nbw = max(nbat, __shfl_xor_sync(FULL, nbat, 16));
        for (uint32_t bt = 0; bt < nbw; bt++) {
            const uint32_t i = bt * 16 + r;
            if (i < cnt) {
                const uint64_t pr = P.pairs[base + st + i];
                const int64_t pB = (int64_t)(uint32_t)pr;
                cp16(sMB + r * TILE, P.mB + pB * TILE);
                cp16(sMB + r * TILE + 8, P.mB + pB * TILE + 8);
                sOB[r] = P.rowOccB[pB];
                sS[r] = (uint8_t)((int64_t)(pr >> 32) - a0);
            }
            cp_wait_all();
            __syncwarp();
            const uint32_t nb = cnt > bt * 16 ? min(16u, cnt - bt * 16) : 0u;
            for (uint32_t k = 0; k < nb; k++) {
                uint32_t ma = (uint32_t)sMA[sS[k] * TILE + r] & sOB[k];
                const uint16_t *mb = sMB + k * TILE;
                while (ma) {
                    const int c = __ffs(ma) - 1;
                    ma &= ma - 1;
                    acc |= mb[c];
                }
            }
            __syncwarp();
        }
        const int cn = __popc(acc);
        int incl = cn;
#pragma unroll
        for (int d = 1; d < 16; d <<= 1) {
            const int o = __shfl_up_sync(FULL, incl, d, 16);
            if (r >= d) incl += o;
        }
        const int tot = __shfl_sync(FULL, incl, 15, 16);
        if (hv) {
            P.sMaskC[(base + q) * TILE + r] = (uint16_t)acc;
            P.sRowPtrC[(base + q) * TILE + r] = (uint8_t)(incl - cn);
            if (r == 0) {
                P.tWork[base + q] = (uint32_t)tot;  // the tile's nnz (the row path has no step-2 class split)
                rownnz += tot;
                ndense += tot >= P.dense_threshold;
            }
        }
    }
    rownnz += __shfl_xor_sync(FULL, rownnz, 16);
    ndense += __shfl_xor_sync(FULL, ndense, 16);
    if (lane == 0) {
        P.rowNnz[I] = rownnz;
        if (ndense) {
            atomicAdd(&P.cnt->n2dense, (u64c)ndense);
            atomicMax(&P.cnt->max_a_dense, (u64c)nA);
        }
    }
}

// step 1's scratch was sized from the free part of the call's arena before the candidate total
// was known on the host: every step-1 kernel checks it on the device and, if it does not fit, flags
// the call (read with C's tile count) and does nothing -- the host grows the arena and redoes
__device__ __forceinline__ bool scratch_fits(const S1Params &P) {
    const bool ok = *P.utot <= P.capU && (int64_t)P.cnt->big_u <= P.capBig;
    if (!ok && threadIdx.x == 0) P.cnt->overflow = 1;
    return ok;
}

__global__ void __launch_bounds__(ROW_T) k_row_small(S1Params P, int cap) { TSG_GRID_WAIT();
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ uint32_t hist[256 * ROW_NW];
    __shared__ int sm[ROW_NW + 1];
    if (!scratch_fits(P)) return;
    uint32_t *keysA = reinterpret_cast<uint32_t *>(smem);
    uint32_t *keysB = keysA + cap;
    uint32_t *posB = keysB + cap;
    uint16_t *kpos = reinterpret_cast<uint16_t *>(posB + cap);
    const int64_t n = (int64_t)P.cnt->nsmall;
    __shared__ int64_t kk;
    for (;;) {  // persistent over the small rows, one at a time from a counter
        if (threadIdx.x == 0) kk = (int64_t)atomicAdd(&P.cnt->next_small, 1ULL);
        __syncthreads();
        const int64_t k = kk;
        __syncthreads();
        if (k >= n) break;
        const int64_t I = P.smallList[k];
        const int64_t U = P.costOff[P.tpA[I + 1]] - P.costOff[P.tpA[I]];
        const int ub = bits_for((uint64_t)(U > 1 ? U - 1 : 1));
        row_sort_body<uint32_t, uint16_t>(P, I, keysA, keysB, posB, kpos, hist, sm, ub);
        __syncthreads();
    }
}

__global__ void __launch_bounds__(ROW_T) k_row_big(S1Params P) { TSG_GRID_WAIT();
    __shared__ uint32_t hist[256 * ROW_NW];
    __shared__ int sm[ROW_NW + 1];
    if (!scratch_fits(P)) return;
    const int64_t n = (int64_t)P.cnt->nbig;
    __shared__ int64_t kk;
    for (;;) {
        if (threadIdx.x == 0) kk = (int64_t)atomicAdd(&P.cnt->next_big, 1ULL);
        __syncthreads();
        const int64_t k = kk;
        __syncthreads();
        if (k >= n) break;
        const int64_t I = P.bigList[k];
        const int64_t o = P.bigOff[I];
        row_sort_body<uint64_t, uint32_t>(P, I, P.bigKeysA + o, P.bigKeysB + o, P.bigPosB + o, P.bigKpos + o, hist,
                                          sm, 32);
        __syncthreads();
    }
}

// ------------------------------------------------------------------------------------------
// a1 (rank): tile rows too wide for the warp merge and the shared-memory sort (R-MAT hubs, up to
// ~10^6 candidates).  One CTA per row, no sort: the row's tile columns J that have a product are
// marked in a shared-memory bitmap over the row's J window; a C tile's rank in the row is the
// number of marked columns before it (per-word popcount prefix).  Pairs are counted per rank,
// offsets scanned, and scattered with per-tile cursors; each C tile's (short) pair list is then
// insertion-sorted by A tile position, i.e. ascending K (reading A8).  Three passes over the
// candidates (expand once into global scratch, count, scatter) instead of a multi-pass radix sort.
// ------------------------------------------------------------------------------------------
#ifndef TSG_RANK_T
#define TSG_RANK_T 1024
#endif
#ifndef TSG_RANK_CPS
#define TSG_RANK_CPS 2
#endif
constexpr int RANK_T = TSG_RANK_T;  // threads of a bitmap-rank CTA (one wide tile row at a time)
constexpr int RANK_NW = RANK_T / 32;

__device__ __forceinline__ int64_t block_excl_scan64(int64_t v, int64_t *total, int64_t *sm /* RANK_NW+1 */) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int64_t incl = v;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const int64_t o = __shfl_up_sync(FULL, incl, d);
        if (lane >= d) incl += o;
    }
    if (lane == 31) sm[w] = incl;
    __syncthreads();
    if (threadIdx.x == 0) {
        int64_t acc = 0;
        for (int k = 0; k < RANK_NW; k++) {
            const int64_t x = sm[k];
            sm[k] = acc;
            acc += x;
        }
        sm[RANK_NW] = acc;
    }
    __syncthreads();
    const int64_t res = sm[w] + incl - v;
    *total = sm[RANK_NW];
    __syncthreads();
    return res;
}

__device__ void rank_row_big(const S1Params &P, int64_t I, int wwords, uint32_t *bm, int64_t *sm);

__global__ void __launch_bounds__(RANK_T) k_row_rank(S1Params P, int wwords) { TSG_GRID_WAIT();
    extern __shared__ uint32_t bm[];  // [wwords] bitmap, then [wwords] exclusive popcount prefix
    __shared__ int64_t sm[RANK_NW + 1];
    if (!scratch_fits(P)) return;
    const int64_t n = (int64_t)P.cnt->nbig;
    __shared__ int64_t kk;
    for (;;) {  // persistent over the wide rows, one at a time from a counter (they differ widely)
        if (threadIdx.x == 0) kk = (int64_t)atomicAdd(&P.cnt->next_big, 1ULL);
        __syncthreads();
        const int64_t k = kk;
        __syncthreads();
        if (k >= n) break;
        rank_row_big(P, P.bigList[k], wwords, bm, sm);
        __syncthreads();
    }
}

__device__ void rank_row_big(const S1Params &P, int64_t I, int wwords, uint32_t *bm, int64_t *sm) {
    uint32_t *pre = bm + wwords;
    const int64_t a0 = P.tpA[I], a1 = P.tpA[I + 1];
    const int nA = (int)(a1 - a0);
    const int64_t base = P.costOff[a0];
    const int64_t U = P.costOff[a1] - base;
    const int32_t jlo = P.rowJlo[I];
    const int64_t o = P.bigOff[I];
    uint32_t *sJ = reinterpret_cast<uint32_t *>(P.bigKeysA + o);  // J - jlo, or ~0u without product
    uint32_t *sPos = P.bigPosB + o;
    uint32_t *sK = P.bigKpos + o;
    for (int w = threadIdx.x; w < wwords; w += RANK_T) bm[w] = 0;
    __syncthreads();
    // pass 1: expand, mark the bitmap -- a warp per A tile of the row, its lanes over that tile's
    // candidates (no search for a candidate's owner; R-MAT A tiles hold ~40 candidates each)
    const int wid = threadIdx.x >> 5, lid = threadIdx.x & 31;
    for (int k = wid; k < nA; k += RANK_NW) {
        const int64_t t = a0 + k;
        const int64_t u0 = P.costOff[t] - base, len = P.costOff[t + 1] - base - u0;
        const int64_t st = P.startA[t];
        const uint32_t co = P.colOccA[t];
        for (int64_t s = lid; s < len; s += 32) {
            const int64_t u = u0 + s;
            uint32_t posB, occ = 0;
            bool valid;
            if (st < 0) {
                posB = P.list[-st - 1 + s];
                valid = true;
            } else {
                posB = (uint32_t)(st + s);
                occ = P.rowOccB[posB];
                valid = (occ & co) != 0;
            }
            const uint32_t jr = valid ? (uint32_t)((st < 0 ? P.listJ[-st - 1 + s] : P.tcB[posB]) - jlo) : ~0u;
            // the candidate's (pair, c) items (step 2's work estimate) ride in the top 5 bits
            const uint32_t wk = st < 0 ? 1u : (uint32_t)__popc(occ & co);
            sJ[u] = valid ? jr | (wk << 27) : ~0u;
            sPos[u] = posB;
            sK[u] = (uint32_t)k;
            if (valid) atomicOr(&bm[jr >> 5], 1u << (jr & 31));
        }
    }
    __syncthreads();
    // ranks: exclusive popcount prefix over the bitmap words (blocked ownership)
    const int per = (wwords + RANK_T - 1) / RANK_T;
    const int w0 = min(wwords, (int)threadIdx.x * per), w1 = min(wwords, w0 + per);
    int64_t cntw = 0;
    for (int w = w0; w < w1; w++) cntw += __popc(bm[w]);
    int64_t nC;
    int64_t run = block_excl_scan64(cntw, &nC, sm);
    for (int w = w0; w < w1; w++) {
        pre[w] = (uint32_t)run;
        run += __popc(bm[w]);
    }
    // the C tiles' tile columns, straight from the bitmap (each thread its words)
    for (int w = w0; w < w1; w++) {
        uint32_t m = bm[w];
        uint32_t rk = pre[w];
        while (m) {
            const int b = __ffs(m) - 1;
            m &= m - 1;
            P.tJ[base + rk++] = jlo + (int32_t)(w * 32 + b);
        }
    }
    uint32_t *cursor = reinterpret_cast<uint32_t *>(P.bigKeysB + o);  // per C tile, pass 3
    for (int64_t r = threadIdx.x; r < nC; r += RANK_T) {
        P.tCnt[base + r] = 0;
        P.tWork[base + r] = 0;
        cursor[r] = 0;
    }
    __syncthreads();
    // pass 2: pairs and work per C tile (global counters: shared ones for rows of up to 12 K C
    // tiles halve the occupancy and measured slower on C4, 51 vs 39 ms)
    for (int64_t u = threadIdx.x; u < U; u += RANK_T) {
        const uint32_t jw = sJ[u];
        if (jw == ~0u) continue;
        const uint32_t jr = jw & 0x7ffffffu;
        const uint32_t rank = pre[jr >> 5] + __popc(bm[jr >> 5] & ((1u << (jr & 31)) - 1u));
        atomicAdd(&P.tCnt[base + rank], 1u);
        atomicAdd(&P.tWork[base + rank], jw >> 27);
    }
    __syncthreads();
    // pair offsets of the C tiles (row-relative), blocked scan over the nC counts
    const int64_t perC = (nC + RANK_T - 1) / RANK_T;
    const int64_t c0 = min(nC, (int64_t)threadIdx.x * perC), c1 = min(nC, c0 + perC);
    int64_t cs = 0;
    for (int64_t r = c0; r < c1; r++) cs += P.tCnt[base + r];
    int64_t npairs;
    int64_t runc = block_excl_scan64(cs, &npairs, sm);
    for (int64_t r = c0; r < c1; r++) {
        P.tStart[base + r] = (uint32_t)runc;
        runc += P.tCnt[base + r];
    }
    __syncthreads();
    // pass 3: scatter the pairs with per-tile cursors
    for (int64_t u = threadIdx.x; u < U; u += RANK_T) {
        const uint32_t jw = sJ[u];
        if (jw == ~0u) continue;
        const uint32_t jr = jw & 0x7ffffffu;
        const uint32_t rank = pre[jr >> 5] + __popc(bm[jr >> 5] & ((1u << (jr & 31)) - 1u));
        const uint32_t slot = P.tStart[base + rank] + atomicAdd(&cursor[rank], 1u);
        P.pairs[base + slot] = ((uint64_t)(a0 + sK[u]) << 32) | sPos[u];
    }
    __syncthreads();
    // pass 4: each C tile's pairs in ascending A tile position (= ascending K)
    for (int64_t r = threadIdx.x; r < nC; r += RANK_T) {
        uint64_t *pp = P.pairs + base + P.tStart[base + r];
        const uint32_t n = P.tCnt[base + r];
        for (uint32_t i = 1; i < n; i++) {
            const uint64_t x = pp[i];
            uint32_t k = i;
            while (k > 0 && pp[k - 1] > x) {
                pp[k] = pp[k - 1];
                k--;
            }
            pp[k] = x;
        }
    }
    if (threadIdx.x == 0) {
        P.nC[I] = nC;
        atomicAdd(&P.cnt->pairs, (u64c)npairs);
    }
}

// transposed tile masks: maskT[c] bit r <=> nonzero (r,c)  (used by the item-driven paths)
// 8x8 bit-matrix transpose in a 64-bit word (byte i = row i, bit j = column j), three masked
// delta swaps
__device__ __forceinline__ uint64_t transpose8(uint64_t x) {
    uint64_t t;
    t = (x ^ (x >> 7)) & 0x00AA00AA00AA00AAull;
    x = x ^ t ^ (t << 7);
    t = (x ^ (x >> 14)) & 0x0000CCCC0000CCCCull;
    x = x ^ t ^ (t << 14);
    t = (x ^ (x >> 28)) & 0x00000000F0F0F0F0ull;
    x = x ^ t ^ (t << 28);
    return x;
}

// transposed masks (maskT[c] bit r <=> mask[r] bit c): the 16x16 tile as four 8x8 blocks,
// gathered with byte permutes, transposed in 64-bit words and scattered back
__global__ void k_transpose(const uint16_t *__restrict__ mask, int64_t nt, uint16_t *__restrict__ maskT) { TSG_GRID_WAIT();
    int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= nt) return;
    const uint4 *p = reinterpret_cast<const uint4 *>(mask + t * TILE);
    const uint4 a = __ldg(p), b = __ldg(p + 1);
    const uint32_t w[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};  // w[k] = row 2k | row 2k+1 << 16
    uint64_t y[2][2];  // y[rb][cb] = transpose of rows 8rb..8rb+7 x columns 8cb..8cb+7
#pragma unroll
    for (int rb = 0; rb < 2; rb++)
#pragma unroll
        for (int cb = 0; cb < 2; cb++) {
            const uint32_t sel = cb | (2 + cb) << 4 | (4 + cb) << 8 | (6 + cb) << 12;
            const uint32_t lo = __byte_perm(w[4 * rb], w[4 * rb + 1], sel);
            const uint32_t hi = __byte_perm(w[4 * rb + 2], w[4 * rb + 3], sel);
            y[rb][cb] = transpose8((uint64_t)lo | (uint64_t)hi << 32);
        }
    uint32_t o[8];  // o[m] = column 2m | column 2m+1 << 16, column c = byte c%8 of y[0][c/8] | of y[1][c/8] << 8
#pragma unroll
    for (int m = 0; m < 8; m++) {
        const int c = 2 * m, cb = c >> 3, k = c & 7, kk = k & 3;
        const uint32_t h0 = k >= 4 ? (uint32_t)(y[0][cb] >> 32) : (uint32_t)y[0][cb];
        const uint32_t h1 = k >= 4 ? (uint32_t)(y[1][cb] >> 32) : (uint32_t)y[1][cb];
        o[m] = __byte_perm(h0, h1, kk | (4 + kk) << 4 | (kk + 1) << 8 | (5 + kk) << 12);
    }
    uint4 *q = reinterpret_cast<uint4 *>(maskT + t * TILE);
    q[0] = make_uint4(o[0], o[1], o[2], o[3]);
    q[1] = make_uint4(o[4], o[5], o[6], o[7]);
}

// ------------------------------------------------------------------------------------------
// compaction: per-C-tile arrays (tile column, pair range, work estimate) from the per-row step-1
// results, one warp per tile row
// ------------------------------------------------------------------------------------------
// (ROWCTA: a CTA per tile row, for rows of thousands of C tiles -- R-MAT -- where a warp per row
// serialises the long rows)
template <bool ROWCTA>
__global__ void __launch_bounds__(256) k_compact(CompactParams P) { TSG_GRID_WAIT();
    const int lane = ROWCTA ? (int)threadIdx.x : (int)(threadIdx.x & 31);
    const int step = ROWCTA ? 256 : 32;
    const int64_t I = ROWCTA ? (int64_t)blockIdx.x : (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (I >= P.tm) return;
    const int64_t base = P.costOff[P.tpA[I]];
    const int64_t t0 = P.tilePtrC[I], n = P.tilePtrC[I + 1] - t0;
#pragma unroll 4
    for (int64_t r = lane; r < n; r += step) {
        const int64_t slot = base + r, t = t0 + r;
        P.tile_col[t] = P.tJ[slot];
        P.pairBeg[t] = base + P.tStart[slot];
        P.pairCnt[t] = P.tCnt[slot];
        P.work[t] = P.tWork[slot];
    }
}

}  // namespace

// ------------------------------------------------------------------------------------------
// launchers
// ------------------------------------------------------------------------------------------
void launch_tile_records(int64_t nt, const int32_t *tile_col, const int64_t *tile_nnz, const uint16_t *mask,
                         const uint8_t *idx, const void *val, int32_t dtype, TileRec *rec, cudaStream_t s) {
    const unsigned g = grid_for(nt, 256);
    if (dtype == TSG_F64)
        TSG_LAUNCH(k_tile_records<double>, g, 256, 0, s, nt, tile_col, tile_nnz, mask, idx,
                   static_cast<const double *>(val), rec);
    else if (dtype == TSG_F32)
        TSG_LAUNCH(k_tile_records<float>, g, 256, 0, s, nt, tile_col, tile_nnz, mask, idx,
                   static_cast<const float *>(val), rec);
    else
        TSG_LAUNCH(k_tile_records<__half>, g, 256, 0, s, nt, tile_col, tile_nnz, mask, idx,
                   static_cast<const __half *>(val), rec);
}

void launch_occupancy(const uint16_t *mask, int64_t nt, uint16_t *row_occ, uint16_t *col_occ, cudaStream_t s,
                      void *zero, size_t zero_bytes) {
    TSG_LAUNCH(k_occupancy, std::max(1u, grid_for(nt, 256)), 256, 0, s, mask, nt, row_occ, col_occ,
               static_cast<uint64_t *>(zero), (int)(zero_bytes / 8));
}

void launch_rowlist(int64_t tmB, const int64_t *tpB, const uint16_t *maskB, const int64_t *lptr, int32_t *lcnt,
                    uint32_t *list, const int32_t *tcB, int32_t *listJ, cudaStream_t s) {
    TSG_LAUNCH(k_rowlist, grid_for(ceil_div(tmB, 2), 8), 256, 0, s, tmB, tpB, maskB, lptr, lcnt, list, tcB, listJ);
}

void launch_row_products(int64_t tmA, const int64_t *tpA, const int32_t *tcA, const uint16_t *maskA, int64_t tmB,
                         const int64_t *tpB, const uint16_t *maskB, int32_t *rnnz, int64_t *w, cudaStream_t s) {
    TSG_LAUNCH(k_brow_nnz, grid_for(ceil_div(tmB, 2), 8), 256, 0, s, tmB, tpB, maskB, rnnz);
    TSG_LAUNCH(k_row_products, grid_for(tmA, 8), 256, 0, s, tmA, tpA, tcA, maskA, (const int32_t *)rnnz, w);
}

void launch_cuts(const int64_t *pre, int64_t tm, int64_t parts, int64_t *cuts, cudaStream_t s) {
    TSG_LAUNCH(k_cuts, 1, 32, 0, s, pre, tm, parts, cuts);
}

void launch_products(int64_t tmB, const int64_t *tpB, const uint16_t *maskB, int64_t ntA, const int32_t *tcA,
                     const uint16_t *maskA, int32_t *rnnz, DevCounters *cnt, cudaStream_t s) {
    TSG_LAUNCH(k_brow_nnz, grid_for(ceil_div(tmB, 2), 8), 256, 0, s, tmB, tpB, maskB, rnnz);
    TSG_LAUNCH(k_products, grid_for(ntA, 256), 256, 0, s, ntA, tcA, maskA, (const int32_t *)rnnz, cnt);
}

void launch_atile_plan(int64_t ntA, const int32_t *tcA, const uint16_t *colOccA, const int64_t *tpB,
                       const int32_t *tcB, const int64_t *lptr, const uint32_t *list, const int32_t *listJ,
                       bool scan_only, int64_t *cost, int64_t *start, int32_t *jlo, int32_t *jhi, DevCounters *cnt,
                       cudaStream_t s) {
    TSG_LAUNCH(k_atile_plan, grid_for(ntA, 256), 256, 0, s, ntA, tcA, colOccA, tpB, tcB, lptr, list, listJ, scan_only,
               cost, start, jlo, jhi, cnt);
}

void launch_row_plan(int64_t tmA, const int64_t *tpA, const int64_t *costOff, const int32_t *jloA,
                     const int32_t *jhiA, bool merge, int32_t *rowJlo, int32_t *rowJhi, uint8_t *rowClass,
                     int64_t *nC, int32_t *bigList, int64_t *bigOff, int32_t *smallList, DevCounters *cnt,
                     cudaStream_t s) {
    TSG_LAUNCH(k_row_plan, grid_for(tmA, 8), 256, 0, s, tmA, tpA, costOff, jloA, jhiA, merge, rowJlo, rowJhi,
               rowClass, nC, bigList, bigOff, smallList, cnt);
}

void launch_transpose(const uint16_t *mask, int64_t nt, uint16_t *maskT, cudaStream_t s) {
    TSG_LAUNCH(k_transpose, grid_for(nt, 256), 256, 0, s, mask, nt, maskT);
}

void launch_compact(const CompactParams &P, int64_t ntC, cudaStream_t s) {
    if (ntC > 512 * P.tm) TSG_LAUNCH(k_compact<true>, (unsigned)P.tm, 256, 0, s, P);
    else TSG_LAUNCH(k_compact<false>, grid_for(P.tm, 8), 256, 0, s, P);
}

bool launch_structural(int64_t tmA, const int64_t *tpA, const int32_t *tcA, const int64_t *tpB, const int32_t *tcB,
                       int64_t tnB, DevCounters *cnt, cudaStream_t s) {
    const int64_t words = (tnB + 31) / 32;
    if (words * 4 > 200 * 1024) return false;  // B too wide for the shared-memory bitmap
    const size_t smem = (size_t)std::max<int64_t>(words, 1) * 4;
    TSG_CUDA(cudaFuncSetAttribute(k_structural, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    TSG_LAUNCH(k_structural, (unsigned)tmA, 256, smem, s, tpA, tcA, tpB, tcB, (int)words, cnt);
    return true;
}

void launch_sym_rows(const S1Params &P, int64_t tm, cudaStream_t s) {
    TSG_LAUNCH(k_sym_rows, grid_for(tm, MERGE_W), MERGE_W * 32, 0, s, P, tm);
}

void launch_row_sort(const S1Params &P, int64_t tm, cudaStream_t s) {
    // the row classes' sizes live on the device: the merge covers every row (others exit at once),
    // the shared-memory sort and the wide-row kernels run persistent grids over their row lists
    static int nsm = 0;
    if (!nsm) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
        nsm = std::max(nsm, 1);
    }
    if (!P.sort_only) TSG_LAUNCH(k_row_merge, grid_for(tm, MERGE_W), MERGE_W * 32, 0, s, P, tm);
    {
        const int cap = ROW_CAP;
        const size_t smem = (size_t)cap * (4 + 4 + 4 + 2);
        TSG_CUDA(cudaFuncSetAttribute(k_row_small, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        TSG_LAUNCH(k_row_small, (unsigned)std::min<int64_t>(tm, 3LL * nsm), ROW_T, smem, s, P, cap);
    }
    // bitmap over the J window (<= tile columns of B) in shared memory, else the global sort
    const int64_t wwords = (P.tnB + 31) / 32;
    const size_t smem = (size_t)wwords * 8;
    if (!P.sort_only && smem <= 200 * 1024) {
        TSG_CUDA(cudaFuncSetAttribute(k_row_rank, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        TSG_LAUNCH(k_row_rank, (unsigned)std::min<int64_t>(tm, (int64_t)TSG_RANK_CPS * nsm), RANK_T, smem, s, P, (int)wwords);
    } else {
        TSG_LAUNCH(k_row_big, (unsigned)std::min<int64_t>(tm, 8LL * nsm), ROW_T, 0, s, P);
    }
}


}  // namespace tsg
