// tsg_spgemm.cu -- the three steps of TileSpGEMM (Section 3.3) on sm_100a.
//
//   a0  helper indices: per-tile row/column occupancy of A and B (16-bit), optional B row lists
//   a1  step 1: the exact set of non-empty C tiles per tile row, and per C tile its contributing
//       (A_IK, B_KJ) pair list in ascending K  (paper: C' = A'B' via NSPARSE; pairs
//       by set intersection, Alg 2 l.4-18, P:1049-1087 -- see DESIGN.md §4 for why the build
//       emits pairs from a per-tile-row expansion instead)
//   a2  step 2: per C tile the 16 row masks by OR-ing B row masks selected by A's nonzeros
//       (Alg 2 l.19-25), popcounts, 16-entry row offsets, tile nnz
//   a3  device prefix sums + allocation of C
//   a4  step 3: values with the adaptive accumulator (Alg 3): dense 16x16
//       accumulator for tiles with nnz >= t_nnz = 192, sparse accumulator
//       addressed through mask_C otherwise
//
// Summation order (reading A8): for every C entry, products are added with FMA in ascending
// pair K and ascending c inside the pair, i.e. ascending global k -- identical to the oracle's
// Gustavson order, so results are deterministic and bitwise reproducible.
#include <algorithm>

#include "tsg_internal.cuh"

namespace tsg {
namespace {

constexpr unsigned FULL = 0xffffffffu;
constexpr int ROW_T = 256;                // threads of a step-1 row CTA
constexpr int ROW_NW = ROW_T / 32;
constexpr int ROW_CAP = 4096;             // max candidates of a row sorted in shared memory
constexpr int STEP2_T = 256;              // 16 half-warps
constexpr int STEP2_CH = 256;             // C tiles per step-2 CTA
constexpr int STEP3_T = 256;

typedef unsigned long long u64c;
struct DevCounters {
    u64c max_u_small;  // largest candidate count among shared-memory rows
    u64c nbig;         // rows sorted in global memory
    u64c big_u;        // their total candidate count
    u64c list_tiles;   // A tiles expanded through B row lists
    u64c pairs;        // contributing pairs
    u64c ndense;       // C tiles with nnz >= t_nnz
    u64c products;     // intermediate products (stats only)
    u64c pad;
};

enum RowClass : uint8_t { ROW_EMPTY = 0, ROW_SMALL = 1, ROW_BIG = 2 };

__device__ __forceinline__ int bits_for(uint64_t v) {  // bits needed to represent v (>= 1)
    return v ? 64 - __clzll((long long)v) : 1;
}

// ------------------------------------------------------------------------------------------
// a0: occupancy words.  rowOcc bit r = row r non-empty; colOcc = OR of the 16 row masks.
// A pair (A_IK, B_KJ) has a product iff colOcc(A_IK) & rowOcc(B_KJ) != 0.
// ------------------------------------------------------------------------------------------
__global__ void k_occupancy(const uint16_t *__restrict__ mask, int64_t nt, uint16_t *__restrict__ row_occ,
                            uint16_t *__restrict__ col_occ) {
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

// B row lists ("mode ii"): for each global row k of B, the B tiles of tile row k/16 whose row
// k%16 is non-empty, ascending tile column.  One warp = two B tile rows, lane r = row r.
__global__ void __launch_bounds__(256) k_rowlist(int64_t tmB, const int64_t *__restrict__ tpB,
                                                 const uint16_t *__restrict__ maskB, const int64_t *__restrict__ lptr,
                                                 int32_t *__restrict__ lcnt, uint32_t *__restrict__ list) {
    const int lane = threadIdx.x & 31, r = lane & 15;
    const int64_t K = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 2 + (lane >> 4);
    if (K >= tmB) return;
    const int64_t t0 = tpB[K], t1 = tpB[K + 1];
    if (!list) {
        int c = 0;
        for (int64_t t = t0; t < t1; t++) c += maskB[t * TILE + r] != 0;
        lcnt[K * TILE + r] = c;
    } else {
        int64_t pos = lptr[K * TILE + r];
        for (int64_t t = t0; t < t1; t++)
            if (maskB[t * TILE + r]) list[pos++] = (uint32_t)t;
    }
}

// stats only: nnz of every global row of B, then products per A tile
__global__ void __launch_bounds__(256) k_brow_nnz(int64_t tmB, const int64_t *__restrict__ tpB,
                                                  const uint16_t *__restrict__ maskB, int32_t *__restrict__ rnnz) {
    const int lane = threadIdx.x & 31, r = lane & 15;
    const int64_t K = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 2 + (lane >> 4);
    if (K >= tmB) return;
    int c = 0;
    for (int64_t t = tpB[K]; t < tpB[K + 1]; t++) c += __popc(maskB[t * TILE + r]);
    rnnz[K * TILE + r] = c;
}

__global__ void k_products(int64_t ntA, const int32_t *__restrict__ tcA, const uint16_t *__restrict__ maskA,
                           const int32_t *__restrict__ rnnz, DevCounters *cnt) {
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
// a1 (plan): per A tile, how its candidate B tiles are enumerated.
//   scan mode: every tile of B tile row K (filtered later by occupancy);
//   list mode: when A_IK touches a single column c, exactly the B row list of k = 16K + c
//              (all of them contribute, no filter, no duplicates).
// cost = number of candidates; start encodes the mode (list: -(start+1)).
// ------------------------------------------------------------------------------------------
__global__ void k_atile_plan(int64_t ntA, const int32_t *__restrict__ tcA, const uint16_t *__restrict__ colOccA,
                             const int64_t *__restrict__ tpB, const int32_t *__restrict__ tcB,
                             const int64_t *__restrict__ lptr, const uint32_t *__restrict__ list, bool scan_only,
                             int64_t *__restrict__ cost, int64_t *__restrict__ start, int32_t *__restrict__ jlo,
                             int32_t *__restrict__ jhi, DevCounters *cnt) {
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
            int64_t f = is_list ? (int64_t)list[st] : st, l = is_list ? (int64_t)list[st + len - 1] : st + len - 1;
            jlo[t] = tcB[f];
            jhi[t] = tcB[l];
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
                           const int32_t *__restrict__ jloA, const int32_t *__restrict__ jhiA,
                           int32_t *__restrict__ rowJlo, int32_t *__restrict__ rowJhi, uint8_t *__restrict__ rowClass,
                           int64_t *__restrict__ nC, int32_t *__restrict__ bigList, int64_t *__restrict__ bigOff,
                           DevCounters *cnt) {
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
    const int wb = bits_for((uint64_t)(hi - lo + 1));  // valid 0..hi-lo, sentinel hi-lo+1
    const int ub = bits_for((uint64_t)(U > 1 ? U - 1 : 1));
    if (U <= ROW_CAP && wb + ub <= 32 && (a1 - a0) < 65536) {
        rowClass[I] = ROW_SMALL;
        atomicMax(&cnt->max_u_small, (u64c)U);
    } else {
        rowClass[I] = ROW_BIG;
        u64c k = atomicAdd(&cnt->nbig, 1ULL);
        bigList[k] = (int32_t)I;
        bigOff[I] = (int64_t)atomicAdd(&cnt->big_u, (u64c)U);
    }
}

// ------------------------------------------------------------------------------------------
// a1 (row sort): expand a tile row's candidates, stable-sort them by tile column J, and emit the
// C tiles (ascending J) with their pair lists (ascending K).  Keys are (J - Jlo) << UB | u where
// u is the candidate's kpos-major position, so the LSD radix passes run only over the J bits
// and stability keeps ascending K inside every C tile.
// ------------------------------------------------------------------------------------------
struct S1Params {
    const int64_t *tpA;
    const uint16_t *colOccA;
    const int64_t *costOff;
    const int64_t *startA;
    const int32_t *tcB;
    const uint16_t *rowOccB;
    const uint32_t *list;
    const int32_t *rowJlo;
    const int32_t *rowJhi;
    const uint8_t *rowClass;
    uint64_t *pairs;   // [Utot]  (posA << 32) | posB, at costOff[a0] + i
    int32_t *tJ;       // [Utot]  C tile column of rank r, at costOff[a0] + r
    uint32_t *tStart;  // [Utot]  first pair (row-relative)
    uint32_t *tCnt;    // [Utot]  pair count
    int64_t *nC;       // [tm]    C tiles of the row
    const int32_t *bigList;
    const int64_t *bigOff;
    uint64_t *bigKeysA, *bigKeysB;
    uint32_t *bigPosB, *bigKpos;
    DevCounters *cnt;
};

// CTA-wide exclusive scan of one int per thread (ROW_T threads)
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
        uint32_t e = (r + 1 < nCrow) ? P.tStart[base + r + 1] : (uint32_t)nvalid;
        P.tCnt[base + r] = e - P.tStart[base + r];
    }
    if (threadIdx.x == 0) {
        P.nC[I] = nCrow;
        atomicAdd(&P.cnt->pairs, (u64c)nvalid);
    }
}

__global__ void __launch_bounds__(ROW_T) k_row_small(S1Params P, int64_t tm, int cap) {
    extern __shared__ __align__(16) unsigned char smem[];
    __shared__ uint32_t hist[256 * ROW_NW];
    __shared__ int sm[ROW_NW + 1];
    const int64_t I = blockIdx.x;
    if (I >= tm || P.rowClass[I] != ROW_SMALL) return;
    uint32_t *keysA = reinterpret_cast<uint32_t *>(smem);
    uint32_t *keysB = keysA + cap;
    uint32_t *posB = keysB + cap;
    uint16_t *kpos = reinterpret_cast<uint16_t *>(posB + cap);
    const int64_t U = P.costOff[P.tpA[I + 1]] - P.costOff[P.tpA[I]];
    const int ub = bits_for((uint64_t)(U > 1 ? U - 1 : 1));
    row_sort_body<uint32_t, uint16_t>(P, I, keysA, keysB, posB, kpos, hist, sm, ub);
}

__global__ void __launch_bounds__(ROW_T) k_row_big(S1Params P) {
    __shared__ uint32_t hist[256 * ROW_NW];
    __shared__ int sm[ROW_NW + 1];
    const int64_t I = P.bigList[blockIdx.x];
    const int64_t o = P.bigOff[I];
    row_sort_body<uint64_t, uint32_t>(P, I, P.bigKeysA + o, P.bigKeysB + o, P.bigPosB + o, P.bigKpos + o, hist, sm,
                                      32);
}

// number of step-2 chunks of every tile row
__global__ void k_chunks(int64_t tm, const int64_t *__restrict__ nC, int64_t *__restrict__ chunks) {
    int64_t I = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (I < tm) chunks[I] = (nC[I] + STEP2_CH - 1) / STEP2_CH;
}

// ------------------------------------------------------------------------------------------
// a2: step 2 (symbolic).  A CTA takes a chunk of <= 256 C tiles of one tile row; a 16-lane half
// warp takes one C tile, lane r = row r.  For each pair and each nonzero (r,c) of A_IK:
// mask_C[r] |= mask_B_KJ[c]  (Alg 2 l.19-25).  Row offsets by a 16-lane shuffle scan.
// Also writes the compacted tile column and pair range of the tile.
// ------------------------------------------------------------------------------------------
struct S2Params {
    const int64_t *chunkPtr;
    int64_t tm;
    const int64_t *tpA;
    const int64_t *costOff;
    const int64_t *tilePtrC;
    const int32_t *tJ;
    const uint32_t *tStart;
    const uint32_t *tCnt;
    const uint64_t *pairs;
    const uint16_t *maskA;
    const uint16_t *maskB;
    int32_t *tile_col;
    int64_t *tile_nnz;  // per-tile nnz here; scanned to offsets afterwards
    uint8_t *row_ptr;
    uint16_t *mask;
    int64_t *pairBeg;
    uint32_t *pairCnt;
    uint32_t *denseList;
    int dense_threshold;
    DevCounters *cnt;
};

__global__ void __launch_bounds__(STEP2_T) k_step2(S2Params P) {
    __shared__ int64_t sI;
    const int lane = threadIdx.x & 31, r = lane & 15, hw = threadIdx.x >> 4;
    if (threadIdx.x == 0) {
        // largest I with chunkPtr[I] <= blockIdx.x
        int64_t lo = 0, hi = P.tm - 1, b = blockIdx.x;
        while (lo < hi) {
            int64_t mid = (lo + hi + 1) >> 1;
            if (P.chunkPtr[mid] <= b) lo = mid;
            else hi = mid - 1;
        }
        sI = lo;
    }
    __syncthreads();
    const int64_t I = sI;
    const int64_t rank0 = ((int64_t)blockIdx.x - P.chunkPtr[I]) * STEP2_CH;
    const int64_t tbase = P.tilePtrC[I];
    const int64_t nCrow = P.tilePtrC[I + 1] - tbase;
    const int64_t rEnd = min(nCrow, rank0 + STEP2_CH);
    const int64_t base = P.costOff[P.tpA[I]];
    const int iters = (int)((rEnd - rank0 + 15) / 16);
    for (int it = 0; it < iters; it++) {
        const int64_t rk = rank0 + it * 16 + hw;
        const bool valid = rk < rEnd;
        uint32_t acc = 0;
        int64_t t = tbase + rk;
        if (valid) {
            const int64_t slot = base + rk;
            const uint32_t s0 = P.tStart[slot], np = P.tCnt[slot];
            if (r == 0) {
                P.tile_col[t] = P.tJ[slot];
                P.pairBeg[t] = base + s0;
                P.pairCnt[t] = np;
            }
            const uint64_t *pp = P.pairs + base + s0;
            for (uint32_t q = 0; q < np; q++) {
                const uint64_t pr = pp[q];
                const int64_t pA = (int64_t)(pr >> 32), pB = (int64_t)(uint32_t)pr;
                uint32_t mA = P.maskA[pA * TILE + r];
                const uint16_t *mB = P.maskB + pB * TILE;
                while (mA) {
                    const int c = __ffs(mA) - 1;
                    mA &= mA - 1;
                    acc |= mB[c];
                }
            }
        }
        const int cnt_r = __popc(acc);
        int incl = cnt_r;
#pragma unroll
        for (int d = 1; d < 16; d <<= 1) {
            int o = __shfl_up_sync(FULL, incl, d, 16);
            if (r >= d) incl += o;
        }
        const int tot = __shfl_sync(FULL, incl, 15, 16);
        if (valid) {
            P.mask[t * TILE + r] = (uint16_t)acc;
            P.row_ptr[t * TILE + r] = (uint8_t)(incl - cnt_r);
            if (r == 0) {
                P.tile_nnz[t] = tot;
                if (tot >= P.dense_threshold) {
                    u64c k = atomicAdd(&P.cnt->ndense, 1ULL);
                    P.denseList[k] = (uint32_t)t;
                }
            }
        }
    }
}

// ------------------------------------------------------------------------------------------
// a4: step 3, sparse accumulator (tiles with nnz < t_nnz).  A half warp per C tile, lane r owns
// C row r: its accumulator slots q = popc(mask_C[r] & ((1<<j)-1)) (the "position from the bit
// mask" of P:1824-1857) live in shared memory, slot-major so lanes never conflict.  No atomics:
// each entry is owned by one lane, products arrive in ascending k.
// ------------------------------------------------------------------------------------------
struct S3Params {
    int64_t ntC;
    const int64_t *tile_nnzC;
    const uint8_t *row_ptrC;
    const uint16_t *maskC;
    const int32_t *tile_colC;
    const int64_t *pairBeg;
    const uint32_t *pairCnt;
    const uint64_t *pairs;
    const int64_t *tile_nnzA;
    const uint8_t *row_ptrA;
    const uint16_t *maskA;
    const uint8_t *idxA;
    const double *valA;
    const int64_t *tile_nnzB;
    const uint8_t *row_ptrB;
    const uint16_t *maskB;
    const uint8_t *idxB;
    const double *valB;
    uint8_t *idxC;
    double *valC;
    const uint32_t *denseList;
    int dense_threshold;
};

__global__ void __launch_bounds__(STEP3_T) k_step3_sparse(S3Params P) {
    __shared__ double accs[TILE * STEP3_T];
    const int r = threadIdx.x & 15;
    double *acc = accs + threadIdx.x;
    const int64_t hw0 = (int64_t)blockIdx.x * (STEP3_T / 16) + (threadIdx.x >> 4);
    const int64_t stride = (int64_t)gridDim.x * (STEP3_T / 16);
    for (int64_t t = hw0; t < P.ntC; t += stride) {
        const int64_t z0 = P.tile_nnzC[t];
        if (P.tile_nnzC[t + 1] - z0 >= P.dense_threshold) continue;
        const uint32_t mC = P.maskC[t * TILE + r];
        const int nq = __popc(mC);
        if (nq == 0) continue;
        for (int q = 0; q < nq; q++) acc[q * STEP3_T] = 0.0;
        const int64_t pb = P.pairBeg[t];
        const uint32_t np = P.pairCnt[t];
        for (uint32_t p = 0; p < np; p++) {
            const uint64_t pr = P.pairs[pb + p];
            const int64_t pA = (int64_t)(pr >> 32), pB = (int64_t)(uint32_t)pr;
            uint32_t mA = P.maskA[pA * TILE + r];
            if (!mA) continue;
            const double *va = P.valA + P.tile_nnzA[pA] + P.row_ptrA[pA * TILE + r];
            const int64_t bz = P.tile_nnzB[pB];
            const uint16_t *mBt = P.maskB + pB * TILE;
            const uint8_t *rBt = P.row_ptrB + pB * TILE;
            int ia = 0;
            while (mA) {
                const int c = __ffs(mA) - 1;
                mA &= mA - 1;
                const double a = va[ia++];
                uint32_t mB = mBt[c];
                const double *vb = P.valB + bz + rBt[c];
                int ib = 0;
                while (mB) {
                    const int j = __ffs(mB) - 1;
                    mB &= mB - 1;
                    const int q = __popc(mC & ((1u << j) - 1u));
                    acc[q * STEP3_T] = fma(a, vb[ib++], acc[q * STEP3_T]);
                }
            }
        }
        const int64_t ob = z0 + P.row_ptrC[t * TILE + r];
        uint32_t m = mC;
        for (int q = 0; q < nq; q++) {
            const int j = __ffs(m) - 1;
            m &= m - 1;
            P.idxC[ob + q] = (uint8_t)((r << 4) | j);
            P.valC[ob + q] = acc[q * STEP3_T];
        }
    }
}

// a4: step 3, dense accumulator (tiles with nnz >= t_nnz): a warp per C tile, both tiles of a
// pair staged densely in shared memory, lane (r = lane/2, h = lane%2) owns C(r, 8h..8h+7) in
// registers; compaction through mask_C at the end.  Structurally absent A entries
// are skipped; absent B entries are staged as 0 so a finite a adds an exact +-0 (the value is
// unchanged); a non-finite a falls back to mask-predicated FMAs so Inf*0 never appears.
__global__ void __launch_bounds__(256) k_step3_dense(S3Params P, int64_t ndense) {
    constexpr int AP = 17;  // padded row pitch of the staged A tile (conflict-free column reads)
    __shared__ double As[8][TILE * AP];
    __shared__ __align__(16) double Bs[8][TILE * TILE];
    __shared__ uint16_t Bm[8][TILE];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int r = lane >> 1, h = lane & 1;
    const int64_t stride = (int64_t)gridDim.x * 8;
    double *Ad = As[w];
    double *Bd = Bs[w];
    for (int64_t k = (int64_t)blockIdx.x * 8 + w; k < ndense; k += stride) {
        const int64_t t = P.denseList[k];
        double acc[8];
#pragma unroll
        for (int j = 0; j < 8; j++) acc[j] = 0.0;
        const int64_t pb = P.pairBeg[t];
        const uint32_t np = P.pairCnt[t];
        for (uint32_t p = 0; p < np; p++) {
            const uint64_t pr = P.pairs[pb + p];
            const int64_t pA = (int64_t)(pr >> 32), pB = (int64_t)(uint32_t)pr;
            for (int e = lane; e < TILE * AP; e += 32) Ad[e] = 0.0;
            for (int e = lane; e < TILE * TILE; e += 32) Bd[e] = 0.0;
            __syncwarp();
            bool nf = false;
            for (int64_t e = P.tile_nnzA[pA] + lane; e < P.tile_nnzA[pA + 1]; e += 32) {
                const uint32_t ix = P.idxA[e];
                const double v = P.valA[e];
                nf |= !isfinite(v);
                Ad[(ix >> 4) * AP + (ix & 15)] = v;
            }
            for (int64_t e = P.tile_nnzB[pB] + lane; e < P.tile_nnzB[pB + 1]; e += 32) {
                const uint32_t ix = P.idxB[e];
                Bd[(ix >> 4) * TILE + (ix & 15)] = P.valB[e];
            }
            if (lane < TILE) Bm[w][lane] = P.maskB[pB * TILE + lane];
            const uint32_t mA = P.maskA[pA * TILE + r];
            const bool anynf = __any_sync(FULL, nf);
            __syncwarp();
            if (!anynf) {
#pragma unroll
                for (int c = 0; c < TILE; c++) {
                    if ((mA >> c) & 1u) {
                        const double a = Ad[r * AP + c];
                        const double2 *bp = reinterpret_cast<const double2 *>(Bd + c * TILE + 8 * h);
#pragma unroll
                        for (int jj = 0; jj < 4; jj++) {
                            const double2 b2 = bp[jj];
                            acc[2 * jj] = fma(a, b2.x, acc[2 * jj]);
                            acc[2 * jj + 1] = fma(a, b2.y, acc[2 * jj + 1]);
                        }
                    }
                }
            } else {
                for (int c = 0; c < TILE; c++) {
                    if ((mA >> c) & 1u) {
                        const double a = Ad[r * AP + c];
                        const uint32_t mb = (uint32_t)Bm[w][c] >> (8 * h);
#pragma unroll
                        for (int jj = 0; jj < 8; jj++)
                            if ((mb >> jj) & 1u) acc[jj] = fma(a, Bd[c * TILE + 8 * h + jj], acc[jj]);
                    }
                }
            }
            __syncwarp();
        }
        const uint32_t mC = P.maskC[t * TILE + r];
        const int64_t ob = P.tile_nnzC[t] + P.row_ptrC[t * TILE + r];
#pragma unroll
        for (int jj = 0; jj < 8; jj++) {
            const int j = 8 * h + jj;
            if ((mC >> j) & 1u) {
                const int q = __popc(mC & ((1u << j) - 1u));
                P.idxC[ob + q] = (uint8_t)((r << 4) | j);
                P.valC[ob + q] = acc[jj];
            }
        }
    }
}

}  // namespace

// ------------------------------------------------------------------------------------------
// host orchestration of one tsg_spgemm call
// ------------------------------------------------------------------------------------------
namespace {
struct Timer {
    bool on = false;
    cudaStream_t s{};
    cudaEvent_t ev[8]{};
    void init(bool enable, cudaStream_t st) {
        on = enable;
        s = st;
        if (on)
            for (auto &e : ev) TSG_CUDA(cudaEventCreate(&e));
    }
    void mark(int i) {
        if (on) TSG_CUDA(cudaEventRecord(ev[i], s));
    }
    float ms(int a, int b) {
        float x = 0.f;
        if (on) cudaEventElapsedTime(&x, ev[a], ev[b]);
        return x;
    }
    ~Timer() {
        if (on)
            for (auto &e : ev) cudaEventDestroy(e);
    }
};
}  // namespace

void run_spgemm(const tsg_tiles *A, const tsg_tiles *B, uint32_t flags, const Allocator &al, cudaStream_t s,
                tsg_tiles *C, tsg_stats *st) {
    reset_call_launches();
    TSG_REQUIRE(A->nt < ((int64_t)1 << 31) && B->nt < ((int64_t)1 << 31), TSG_ERR_OVERFLOW, "input has >= 2^31 tiles");
    TSG_REQUIRE(A->tn == B->tm, TSG_ERR_SHAPE, "tile shapes disagree");
    TSG_REQUIRE(((uintptr_t)A->mask & 15) == 0 && ((uintptr_t)B->mask & 15) == 0, TSG_ERR_INVALID_ARG,
                "mask arrays must be 16-byte aligned");
    int TH = (int)((flags >> TSG_DENSE_THRESHOLD_SHIFT) & 0x1ffu);
    if (TH == 0) TH = TSG_DENSE_NNZ;
    Timer tm_;
    tm_.init((flags & TSG_STATS_TIMING) && st, s);
    tm_.mark(0);

    Buffers tmp(al, s), out(al, s);
    const int64_t ntA = A->nt, tmA = A->tm, tmB = B->tm;
    int syncs = 0;
    DevCounters *cnt = tmp.get<DevCounters>(1);
    TSG_CUDA(cudaMemsetAsync(cnt, 0, sizeof(DevCounters), s));

    // ---------------- a0: occupancy words, optional B row lists, optional product count
    uint16_t *colOccA = tmp.get<uint16_t>(ntA);
    uint16_t *rowOccB = tmp.get<uint16_t>(B->nt);
    TSG_LAUNCH(k_occupancy, grid_for(ntA, 256), 256, 0, s, A->mask, ntA, (uint16_t *)nullptr, colOccA);
    TSG_LAUNCH(k_occupancy, grid_for(B->nt, 256), 256, 0, s, B->mask, B->nt, rowOccB, (uint16_t *)nullptr);
    const bool lists = !(flags & TSG_STEP1_SCAN_ONLY) &&
                       ((flags & TSG_STEP1_LIST_ALWAYS) || (B->nt > 0 && B->nnz < 2 * B->nt));
    int64_t *lptr = nullptr;
    uint32_t *list = nullptr;
    const unsigned gridB = grid_for(ceil_div(tmB, 2), 8);
    if (lists) {
        int32_t *lcnt = tmp.get<int32_t>(TILE * tmB);
        lptr = tmp.get<int64_t>(TILE * tmB + 1);
        list = tmp.get<uint32_t>(B->nnz);
        TSG_LAUNCH(k_rowlist, gridB, 256, 0, s, tmB, B->tile_ptr, B->mask, (const int64_t *)nullptr, lcnt,
                   (uint32_t *)nullptr);
        exclusive_scan<int32_t>(lcnt, lptr, TILE * tmB, s, tmp);
        TSG_LAUNCH(k_rowlist, gridB, 256, 0, s, tmB, B->tile_ptr, B->mask, (const int64_t *)lptr, lcnt, list);
    }
    if (st && (flags & TSG_STATS_PRODUCTS)) {
        int32_t *rnnz = tmp.get<int32_t>(TILE * tmB);
        TSG_LAUNCH(k_brow_nnz, gridB, 256, 0, s, tmB, B->tile_ptr, B->mask, rnnz);
        TSG_LAUNCH(k_products, grid_for(ntA, 256), 256, 0, s, ntA, A->tile_col, A->mask, (const int32_t *)rnnz, cnt);
    }
    tm_.mark(1);

    // ---------------- a1: step 1
    int64_t *cost = tmp.get<int64_t>(ntA);
    int64_t *startA = tmp.get<int64_t>(ntA);
    int32_t *jloA = tmp.get<int32_t>(ntA);
    int32_t *jhiA = tmp.get<int32_t>(ntA);
    TSG_LAUNCH(k_atile_plan, grid_for(ntA, 256), 256, 0, s, ntA, A->tile_col, colOccA, B->tile_ptr, B->tile_col,
               (const int64_t *)lptr, (const uint32_t *)list, (bool)(flags & TSG_STEP1_SCAN_ONLY), cost, startA, jloA,
               jhiA, cnt);
    int64_t *costOff = tmp.get<int64_t>(ntA + 1);
    exclusive_scan<int64_t>(cost, costOff, ntA, s, tmp);
    int32_t *rowJlo = tmp.get<int32_t>(tmA);
    int32_t *rowJhi = tmp.get<int32_t>(tmA);
    uint8_t *rowClass = tmp.get<uint8_t>(tmA);
    int64_t *nC = tmp.get<int64_t>(tmA + 1);
    int32_t *bigList = tmp.get<int32_t>(tmA);
    int64_t *bigOff = tmp.get<int64_t>(tmA);
    TSG_LAUNCH(k_row_plan, grid_for(tmA, 8), 256, 0, s, tmA, A->tile_ptr, (const int64_t *)costOff,
               (const int32_t *)jloA, (const int32_t *)jhiA, rowJlo, rowJhi, rowClass, nC, bigList, bigOff, cnt);
    // sync #0: candidate total and row classes
    DevCounters hc{};
    int64_t Utot = 0;
    TSG_CUDA(cudaMemcpyAsync(&Utot, costOff + ntA, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    TSG_CUDA(cudaMemcpyAsync(&hc, cnt, sizeof(DevCounters), cudaMemcpyDeviceToHost, s));
    TSG_CUDA(cudaStreamSynchronize(s));
    syncs++;
    TSG_REQUIRE(Utot < ((int64_t)1 << 40), TSG_ERR_OVERFLOW, "too many step-1 candidates");

    S1Params P1{};
    P1.tpA = A->tile_ptr;
    P1.colOccA = colOccA;
    P1.costOff = costOff;
    P1.startA = startA;
    P1.tcB = B->tile_col;
    P1.rowOccB = rowOccB;
    P1.list = list;
    P1.rowJlo = rowJlo;
    P1.rowJhi = rowJhi;
    P1.rowClass = rowClass;
    P1.pairs = tmp.get<uint64_t>(Utot);
    P1.tJ = tmp.get<int32_t>(Utot);
    P1.tStart = tmp.get<uint32_t>(Utot);
    P1.tCnt = tmp.get<uint32_t>(Utot);
    P1.nC = nC;
    P1.bigList = bigList;
    P1.bigOff = bigOff;
    P1.cnt = cnt;
    if (hc.nbig > 0) {
        P1.bigKeysA = tmp.get<uint64_t>(hc.big_u);
        P1.bigKeysB = tmp.get<uint64_t>(hc.big_u);
        P1.bigPosB = tmp.get<uint32_t>(hc.big_u);
        P1.bigKpos = tmp.get<uint32_t>(hc.big_u);
    }
    if (hc.max_u_small > 0) {
        const int cap = (int)((hc.max_u_small + 31) & ~31LL);
        const size_t smem = (size_t)cap * (4 + 4 + 4 + 2);
        TSG_CUDA(cudaFuncSetAttribute(k_row_small, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        TSG_LAUNCH(k_row_small, (unsigned)tmA, ROW_T, smem, s, P1, tmA, cap);
    }
    if (hc.nbig > 0) TSG_LAUNCH(k_row_big, (unsigned)hc.nbig, ROW_T, 0, s, P1);

    int64_t *tile_ptr = out.get<int64_t>(tmA + 1);
    exclusive_scan<int64_t>(nC, tile_ptr, tmA, s, tmp);
    int64_t *chunks = tmp.get<int64_t>(tmA);
    int64_t *chunkPtr = tmp.get<int64_t>(tmA + 1);
    TSG_LAUNCH(k_chunks, grid_for(tmA, 256), 256, 0, s, tmA, (const int64_t *)nC, chunks);
    exclusive_scan<int64_t>(chunks, chunkPtr, tmA, s, tmp);
    tm_.mark(2);
    // sync #1: number of C tiles
    int64_t ntC = 0, nchunks = 0;
    TSG_CUDA(cudaMemcpyAsync(&ntC, tile_ptr + tmA, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    TSG_CUDA(cudaMemcpyAsync(&nchunks, chunkPtr + tmA, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    TSG_CUDA(cudaStreamSynchronize(s));
    syncs++;
    TSG_REQUIRE(ntC < ((int64_t)1 << 32), TSG_ERR_OVERFLOW, "C has >= 2^32 tiles");

    // ---------------- a2: step 2
    int32_t *tile_col = out.get<int32_t>(ntC);
    int64_t *tile_nnz = out.get<int64_t>(ntC + 1);
    uint8_t *row_ptr = out.get<uint8_t>(TILE * ntC);
    uint16_t *mask = out.get<uint16_t>(TILE * ntC);
    int64_t *pairBeg = tmp.get<int64_t>(ntC);
    uint32_t *pairCnt = tmp.get<uint32_t>(ntC);
    uint32_t *denseList = tmp.get<uint32_t>(TH <= 256 ? ntC : 0);
    tm_.mark(3);
    S2Params P2{chunkPtr, tmA, A->tile_ptr, costOff, tile_ptr, P1.tJ, P1.tStart, P1.tCnt, P1.pairs, A->mask, B->mask,
                tile_col, tile_nnz, row_ptr, mask, pairBeg, pairCnt, denseList, TH, cnt};
    TSG_LAUNCH(k_step2, (unsigned)nchunks, STEP2_T, 0, s, P2);
    // ---------------- a3: offsets of C's nonzeros, allocation
    exclusive_scan<int64_t>(tile_nnz, tile_nnz, ntC, s, tmp);
    tm_.mark(4);
    int64_t nnzC = 0;
    TSG_CUDA(cudaMemcpyAsync(&nnzC, tile_nnz + ntC, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    TSG_CUDA(cudaMemcpyAsync(&hc, cnt, sizeof(DevCounters), cudaMemcpyDeviceToHost, s));
    TSG_CUDA(cudaStreamSynchronize(s));
    syncs++;
    uint8_t *idx = out.get<uint8_t>(nnzC);
    double *val = out.get<double>(nnzC);
    tm_.mark(5);

    // ---------------- a4: step 3
    S3Params P3{ntC, tile_nnz, row_ptr, mask, tile_col, pairBeg, pairCnt, P1.pairs,
                A->tile_nnz, A->row_ptr, A->mask, A->idx, A->val,
                B->tile_nnz, B->row_ptr, B->mask, B->idx, B->val, idx, val, denseList, TH};
    if (ntC > 0) {
        unsigned g = (unsigned)std::min<int64_t>(ceil_div(ntC, STEP3_T / 16), 148 * 64);
        TSG_LAUNCH(k_step3_sparse, g, STEP3_T, 0, s, P3);
    }
    if (hc.ndense > 0) {
        unsigned g = (unsigned)std::min<int64_t>(ceil_div(hc.ndense, 8), 148 * 16);
        TSG_LAUNCH(k_step3_dense, g, 256, 0, s, P3, (int64_t)hc.ndense);
    }
    tm_.mark(6);

    // ---------------- the result handle
    C->m = A->m;
    C->n = B->n;
    C->tm = tmA;
    C->tn = B->tn;
    C->nt = ntC;
    C->nnz = nnzC;
    C->tile_ptr = tile_ptr;
    C->tile_col = tile_col;
    C->tile_nnz = tile_nnz;
    C->row_ptr = row_ptr;
    C->mask = mask;
    C->idx = idx;
    C->val = val;
    void *arr[7] = {tile_ptr, tile_col, tile_nnz, row_ptr, mask, idx, val};
    for (int k = 0; k < 7; k++) {
        C->bytes[k] = out.take(arr[k]);
        C->owns[k] = true;
    }
    C->al = al;
    if (st) {
        DevCounters fin{};
        TSG_CUDA(cudaMemcpyAsync(&fin, cnt, sizeof(DevCounters), cudaMemcpyDeviceToHost, s));
        TSG_CUDA(cudaStreamSynchronize(s));
        memset(st, 0, sizeof(*st));
        st->products = (flags & TSG_STATS_PRODUCTS) ? (int64_t)fin.products : -1;
        st->tiles_structural = -1;
        st->tiles_c = ntC;
        st->nnz_c = nnzC;
        st->candidates = Utot;
        st->pairs = (int64_t)fin.pairs;
        st->tiles_dense = (int64_t)fin.ndense;
        st->tiles_sparse = ntC - (int64_t)fin.ndense;
        st->step1_list_tiles = (int32_t)fin.list_tiles;
        st->host_syncs = syncs;
        st->kernel_launches = call_launches();
        if (tm_.on) {
            st->ms_index = tm_.ms(0, 1);
            st->ms_step1 = tm_.ms(1, 2);
            st->ms_alloc = tm_.ms(2, 3) + tm_.ms(4, 5);
            st->ms_step2 = tm_.ms(3, 4);
            st->ms_step3 = tm_.ms(5, 6);
            st->ms_total = tm_.ms(0, 6);
        }
    }
}

}  // namespace tsg
