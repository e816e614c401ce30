// tsg_rows.cu -- SURVEY §8(a) row a4 (step 3, numeric with the adaptive accumulator) on the row
// path: every tile row of A has <= 32 tiles (stencil / FEM / banded inputs), so one warp owns a
// whole C tile row.  The row's A tiles (masks, row offsets, value offsets) are staged in shared
// memory once and serve all of the row's C tiles (C2: 27 A tiles for ~67 C tiles); the C tile
// records of the fused step 1+2 (k_sym_rows, at the row's candidate-space slots) are copied into
// C's final arrays here, so C is written once (one allocation, after step 2).
//
// Per C tile, by its nnz (Alg 3; the adaptive accumulator P:1808-1876, threshold
// reading A7):
//   small  (nnz <= SMALL_NNZ): one lane per C nonzero (r, j) -- the output-stationary form of the
//          sparse accumulator: the lane walks the tile's pairs in ascending K and, per pair, the
//          columns c of mask_A[r] & colmask_B[j] in ascending order;
//   medium: a half warp per tile, lane r owns C row r with a 16-slot dense-in-j accumulator in
//          shared memory; per batch of 16 pairs the B tiles' masks and row offsets are staged by
//          cp.async, and each lane streams its items (pair, c): a = A(r,c), row c of B;
//   dense  (nnz >= t_nnz): the whole warp, both tiles of a pair staged densely, lane (r, h)
//          holding C(r, 8h..8h+7) in registers.
// Every C entry has one owner and receives its products in ascending k = 16K + c, so the values
// are bitwise equal to the per-C-tile path and to the oracle's fma mode (readings A8, A16).
#include <algorithm>

#include "tsg_device.cuh"

namespace tsg {
namespace {

constexpr unsigned FULL = 0xffffffffu;
constexpr int RN_W = 4;  // warps (tile rows in flight) per CTA
constexpr int RN_T = RN_W * 32;
constexpr int MAX_A = 32;  // A tiles of a row (the row path's condition)
#ifndef TSG_RN_MINB
#define TSG_RN_MINB 6
#endif
constexpr int RN_MINB = TSG_RN_MINB;  // CTAs per SM the register budget is sized for

// per-warp shared memory layout (bytes)
constexpr int OFF_MA = 0;                       // u16 [2][32][16]  A masks of the two rows
constexpr int OFF_RA = OFF_MA + 2 * MAX_A * 32; // u8  [2][32][16]  A row offsets
constexpr int OFF_ZA = OFF_RA + 2 * MAX_A * 16; // i64 [2][32]      A value offsets
constexpr int OFF_WORK = OFF_ZA + 2 * MAX_A * 8; // 3584: per-class work area
struct MedStage {                               // per half warp: a batch of 16 pairs
    uint16_t mB[16][16];                        // B masks
    uint8_t rB[16][16];                         // B row offsets
    int64_t zB[16];                             // B value offsets
    uint16_t oB[16];                            // B row occupancy
    uint8_t s[16];                              // A slot in the row
};
constexpr int ACC_BYTES = 2 * 256 * 8;          // medium accumulators of the two half warps (fp64)
constexpr int MED_BYTES = ACC_BYTES + 2 * (int)sizeof(MedStage);
constexpr int DENSE_BYTES = 2176 + 2048;        // dense staging: A 16 x 17, B 16 x 16 (fp64)
constexpr int WORK_BYTES = MED_BYTES > DENSE_BYTES ? MED_BYTES : DENSE_BYTES;
constexpr int WARP_SMEM = (OFF_WORK + WORK_BYTES + 15) & ~15;
static_assert(sizeof(MedStage) % 16 == 0, "MedStage keeps 16-byte alignment");
static_assert(OFF_WORK % 16 == 0, "work area 16-byte aligned");

struct RowTileRec {  // a C tile left by k_num_rows to k_num_small / k_num_dense
    int64_t slot, off, pairs;
    uint32_t cnt, nz;
};

struct RowNumParams {
    int64_t tm, ntC;
    // A
    const int64_t *tpA, *tnzA;
    const uint8_t *rpA, *ixA;
    const uint16_t *mA;
    const void *vA;
    // B
    const int64_t *tnzB;
    const uint8_t *rpB, *ixB;
    const uint16_t *mB, *mTB, *rowOccB;
    const void *vB;
    // the fused step 1+2 results, at candidate-space slots costOff[a0(I)] + rank
    const int64_t *costOff;
    const uint64_t *pairs;
    const int32_t *tJ;
    const uint32_t *tStart, *tCnt, *tNnz;
    const uint16_t *sMaskC;
    const uint8_t *sRowPtrC;
    const int64_t *rowOff;  // [tm+1] exclusive scan of the rows' nnz
    // C
    const int64_t *tpC;
    int32_t *tcC;
    int64_t *tnzC;
    uint8_t *rpC, *ixC;
    uint16_t *mC;
    void *vC;
    int dense_threshold, small_max;
    int max_a_dense;     // most A tiles in a tile row that has dense C tiles (sizes k_num_dense_row's staging)
    const uint16_t *colOccA;  // column occupancy words of A's tiles
    RowTileRec *small;   // small C tiles, for k_num_small
    DevCounters *cnt;
};

// acc[16 j] += a * B(c, j) over B's row c in ascending j; the first three slots are distinct, so
// their loads, FMAs and stores are independent
template <typename TI, typename TO>
__device__ __forceinline__ void accumulate_row(TO a, TO b0, TO b1, TO b2, uint32_t mb, const TI *vb, TO *acc) {
    const int j0 = __ffs(mb) - 1;
    uint32_t m = mb & (mb - 1);
    const int j1 = __ffs(m) - 1;
    m &= m - 1;
    const int j2 = __ffs(m) - 1;
    m &= m - 1;
    TO *p0 = acc + j0 * 16;
    TO *p1 = acc + (j1 >= 0 ? j1 : j0) * 16;
    TO *p2 = acc + (j2 >= 0 ? j2 : j0) * 16;
    const TO c0 = *p0, c1 = *p1, c2 = *p2;
    *p0 = vfma(a, b0, c0);
    if (j1 >= 0) *p1 = vfma(a, b1, c1);
    if (j2 >= 0) *p2 = vfma(a, b2, c2);
    const TI *q = vb + 3;
    while (m) {
        const int j = __ffs(m) - 1;
        m &= m - 1;
        acc[j * 16] = vfma(a, vcvt<TO>(*q++), acc[j * 16]);
    }
}

// one medium tile by a half warp (hm: the half's lane mask), lane r owning C row r: pairs in
// ascending K, uniform across the half (two halves hold tile rows of the same structure on
// stencils, so the warp stays converged); lane r walks row r of A_IK (values in c order) and
// accumulates B's row c into its 16 slots -- every slot receives its products in ascending k
template <typename TI, typename TO>
__device__ __forceinline__ void medium_tile(const RowNumParams &P, bool hv, int64_t base, int64_t a0,
                                            int64_t slot, uint32_t st, uint32_t cnt, int64_t off,
                                            const uint16_t *sMA, const uint8_t *sRA, const int64_t *sZA,
                                            MedStage &S, TO *acc, int r) {
    const TI *vA = static_cast<const TI *>(P.vA), *vB = static_cast<const TI *>(P.vB);
    uint32_t mCr = 0;
    int64_t ob = 0;
    if (hv) {
        mCr = P.sMaskC[slot * TILE + r];
        ob = off + P.sRowPtrC[slot * TILE + r];
    } else {
        cnt = 0;
    }
    const uint32_t cmax = max(cnt, __shfl_xor_sync(FULL, cnt, 16));  // warp-uniform loop bounds
    for (uint32_t b0 = 0; b0 < cmax; b0 += 16) {
        // lane i stages pair b0 + i and finds the rows of its A tile that meet a non-empty row of
        // its B tile; a 16x16 bit transpose gives lane r the batch pairs that touch row r
        const uint32_t q = b0 + r;
        uint32_t rows = 0;
        if (q < cnt) {
            const uint64_t pr = P.pairs[base + st + q];
            const int64_t pB = (int64_t)(uint32_t)pr;
            cp16(&S.mB[r][0], P.mB + pB * TILE);
            cp16(&S.mB[r][8], P.mB + pB * TILE + 8);
            cp16(&S.rB[r][0], P.rpB + pB * TILE);
            S.zB[r] = P.tnzB[pB];
            const uint32_t ob = P.rowOccB[pB];
            const int s = (int)((int64_t)(pr >> 32) - a0);
            S.s[r] = (uint8_t)s;
            const uint4 *am = reinterpret_cast<const uint4 *>(sMA + s * TILE);
            rows = rows_meeting(am[0], am[1], ob);
        }
        uint32_t rel = bit_transpose16(rows, r);
        cp_wait_all();
        __syncwarp();
        // lane r's own item stream over the batch: pairs touching row r in ascending K, each pair's
        // columns c of row r in ascending order (values of A's row r in order), B's row c
        // accumulated into the row's slots -- every slot receives its products in ascending k
        uint32_t m = 0;
        int i = 0;
        const TI *pa = nullptr, *pb = nullptr;
        for (;;) {
            if (!m) {
                if (!rel) break;
                i = __ffs(rel) - 1;
                rel &= rel - 1;
                const int s = S.s[i];
                m = sMA[s * TILE + r];
                pa = vA + sZA[s] + sRA[s * TILE + r];
                pb = vB + S.zB[i];
            }
            const int c = __ffs(m) - 1;
            m &= m - 1;
            const TO a = vcvt<TO>(*pa++);
            const uint32_t mb = S.mB[i][c];
            if (!mb) continue;  // row c of B_KJ is empty
            const TI *vb = pb + S.rB[i][c];
            const int n = __popc(mb);
            const TO bb0 = vcvt<TO>(vb[0]);
            const TO bb1 = n > 1 ? vcvt<TO>(vb[1]) : (TO)0;
            const TO bb2 = n > 2 ? vcvt<TO>(vb[2]) : (TO)0;
            accumulate_row(a, bb0, bb1, bb2, mb, vb, acc);
        }
        __syncwarp();
    }
    // compaction through mask_C[r]; every touched slot is in mask_C[r] and is reset for the next tile
    if (mCr) {
        uint8_t *px = P.ixC + ob;
        TO *pv = static_cast<TO *>(P.vC) + ob;
        uint32_t m = mCr;
        while (m) {
            const int j = __ffs(m) - 1;
            m &= m - 1;
            TO *sl = acc + j * 16;
            *px++ = (uint8_t)((r << 4) | j);
            *pv++ = *sl;
            *sl = (TO)0;
        }
    }
    __syncwarp();
}

// One warp per two consecutive tile rows, half h owning row 2w + h, 16 lanes per row.  The loops
// over the rows' tiles and pairs are warp-uniform (bounds = the max of the two halves) with
// full-warp reconvergence after every pair: adjacent tile rows of a stencil have the same
// structure, so both halves run the same instruction stream on all 32 lanes.
template <typename TI, typename TO>
__global__ void __launch_bounds__(RN_T, RN_MINB) k_num_rows(RowNumParams P) { TSG_GRID_WAIT();
    __shared__ __align__(16) unsigned char smem[RN_W][WARP_SMEM];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, r = lane & 15, half = lane >> 4;
    const int64_t I0 = ((int64_t)blockIdx.x * RN_W + w) * 2;
    if (I0 >= P.tm) return;  // warp-uniform
    const int64_t I = I0 + half;
    const bool rv = I < P.tm;  // the second row of an odd tail does not exist
    unsigned char *ws = smem[w];
    uint16_t *sMA = reinterpret_cast<uint16_t *>(ws + OFF_MA) + half * MAX_A * TILE;
    uint8_t *sRA = ws + OFF_RA + half * MAX_A * TILE;
    int64_t *sZA = reinterpret_cast<int64_t *>(ws + OFF_ZA) + half * MAX_A;
    unsigned char *wr = ws + OFF_WORK;
    TO *acc = reinterpret_cast<TO *>(wr) + half * 256 + r;
    MedStage &S = reinterpret_cast<MedStage *>(wr + ACC_BYTES)[half];

    int64_t t0 = 0, nC = 0, a0 = 0, base = 0, zrow = 0;
    int nA = 0;
    if (rv) {
        t0 = P.tpC[I];
        nC = P.tpC[I + 1] - t0;
        if (I == P.tm - 1 && r == 0) P.tnzC[P.tpC[P.tm]] = P.rowOff[P.tm];  // C's last offset (= nnz(C))
        a0 = P.tpA[I];
        nA = (int)(P.tpA[I + 1] - a0);
        base = P.costOff[a0];
        zrow = P.rowOff[I];
    }
    // the row's A tiles: masks, row offsets, value offsets (lane r stages tiles a0 + r, a0 + r + 16)
    for (int k = r; k < nA; k += 16) {
        const uint4 *gm = reinterpret_cast<const uint4 *>(P.mA + (a0 + k) * TILE);
        reinterpret_cast<uint4 *>(sMA + k * TILE)[0] = gm[0];
        reinterpret_cast<uint4 *>(sMA + k * TILE)[1] = gm[1];
        reinterpret_cast<uint4 *>(sRA + k * TILE)[0] = *reinterpret_cast<const uint4 *>(P.rpA + (a0 + k) * TILE);
        sZA[k] = P.tnzA[a0 + k];
    }
    // the medium accumulators start cleared (each tile resets the slots it used)
#pragma unroll
    for (int j = 0; j < TILE; j++) acc[j * 16] = (TO)0;
    __syncwarp();
    u64c nmd = 0;
    const unsigned lt = (1u << r) - 1u;
    const int64_t nCmax = max(nC, __shfl_xor_sync(FULL, nC, 16));
    for (int64_t q0 = 0; q0 < nCmax; q0 += 16) {
        // ---- the chunk's C tile records -> C's final arrays; nnz offsets; classes
        const int64_t q = q0 + r;
        const bool v = q < nC;
        const int64_t slot = base + q, t = t0 + q;
        uint32_t nz = 0, st = 0, cn = 0;
        if (v) {
            nz = P.tNnz[slot];
            st = P.tStart[slot];
            cn = P.tCnt[slot];
        }
        uint32_t incl = nz;
#pragma unroll
        for (int d = 1; d < 16; d <<= 1) {
            const uint32_t o = __shfl_up_sync(FULL, incl, d, 16);
            if (r >= d) incl += o;
        }
        const int64_t off = zrow + (incl - nz);
        zrow += __shfl_sync(FULL, incl, 15, 16);
        if (v) {
            P.tcC[t] = P.tJ[slot];
            P.tnzC[t] = off;
            const uint4 *gm = reinterpret_cast<const uint4 *>(P.sMaskC + slot * TILE);
            uint4 *dm = reinterpret_cast<uint4 *>(P.mC + t * TILE);
            dm[0] = gm[0];
            dm[1] = gm[1];
            *reinterpret_cast<uint4 *>(P.rpC + t * TILE) = *reinterpret_cast<const uint4 *>(P.sRowPtrC + slot * TILE);
        }
        const bool isD = v && (int)nz >= P.dense_threshold;
        const bool isS = v && !isD && (int)nz <= P.small_max;
        const bool isM = v && !isD && !isS;
        const unsigned BM = __ballot_sync(FULL, isM), BS = __ballot_sync(FULL, isS);
        unsigned bM = (BM >> (16 * half)) & 0xffffu;
        const unsigned bS = (BS >> (16 * half)) & 0xffffu;
        nmd += __popc(bM);

        // ---- medium tiles: each half its next one, in step
        unsigned both = BM;
        while (both) {
            const int f = bM ? __ffs(bM) - 1 : 0;
            const bool hv = bM != 0;
            if (bM) bM &= bM - 1;
            const uint32_t mst = __shfl_sync(FULL, st, f + 16 * half), mcn = __shfl_sync(FULL, cn, f + 16 * half);
            const int64_t moff = __shfl_sync(FULL, off, f + 16 * half);
            medium_tile<TI, TO>(P, hv, base, a0, base + q0 + f, mst, mcn, moff, sMA, sRA, sZA, S, acc, r);
            both = __ballot_sync(FULL, bM != 0);
        }

        // ---- small tiles: recorded for k_num_small (a lane per C nonzero, its own kernel at full
        // occupancy: the per-entry work is a chain of dependent loads)
        if (BS) {
            uint32_t si = 0;
            if (r == 0 && bS) si = (uint32_t)atomicAdd(&P.cnt->n3small, (u64c)__popc(bS));
            si = __shfl_sync(FULL, si, 16 * half);
            if (isS) {
                RowTileRec &d = P.small[si + __popc(bS & lt)];
                d.slot = slot;
                d.off = off;
                d.pairs = base + st;
                d.cnt = cn;
                d.nz = nz;
            }
        }

        // ---- dense tiles: k_num_dense_row (a CTA per tile row, after this kernel) computes them
    }
    if (r == 0 && nmd) atomicAdd(&P.cnt->n3medium, nmd);
}

// small C tiles (nnz <= small_max) recorded by k_num_rows: one lane per C nonzero (the
// output-stationary form of the paper's sparse accumulator): entry q of a tile is
// (r, j), r = the last row with row_ptr_C[r] <= q, j = the (q - row_ptr_C[r])-th bit of
// mask_C[r]; the lane walks the tile's pairs in ascending K and, per pair, the columns c of
// mask_A[r] & colmask_B[j] in ascending order.  Warps take 32 records at a time.
constexpr int NS_T = 256;
template <typename TI, typename TO>
__global__ void __launch_bounds__(NS_T, 5) k_num_small(RowNumParams P) { TSG_GRID_WAIT();
    __shared__ uint8_t mapsm[NS_T / 32][32 * 16];
    const int lane = threadIdx.x & 31;
    uint8_t *map = mapsm[threadIdx.x >> 5];
    const TI *vA = static_cast<const TI *>(P.vA), *vB = static_cast<const TI *>(P.vB);
    TO *vC = static_cast<TO *>(P.vC);
    const int64_t n = (int64_t)P.cnt->n3small;
    const int64_t gw = (int64_t)blockIdx.x * (NS_T / 32) + (threadIdx.x >> 5), nw = (int64_t)gridDim.x * (NS_T / 32);
    for (int64_t g0 = gw * 32; g0 < n; g0 += nw * 32) {
        const int64_t k = g0 + lane;
        RowTileRec d{};
        if (k < n) d = P.small[k];
        const uint32_t mine = k < n ? d.nz : 0u;
        uint32_t incl = mine;
#pragma unroll
        for (int s = 1; s < 32; s <<= 1) {
            const uint32_t o = __shfl_up_sync(FULL, incl, s);
            if (lane >= s) incl += o;
        }
        const uint32_t excl = incl - mine, tot = __shfl_sync(FULL, incl, 31);
        for (uint32_t q = 0; q < mine; q++) map[excl + q] = (uint8_t)lane;
        __syncwarp();
        for (uint32_t e0 = 0; e0 < tot; e0 += 32) {
            const uint32_t e = e0 + lane;
            const bool act = e < tot;
            const int f = act ? map[e] : 0;
            const uint32_t q = e - __shfl_sync(FULL, excl, f);
            const int64_t fs = __shfl_sync(FULL, d.slot, f), foff = __shfl_sync(FULL, d.off, f);
            const int64_t fp = __shfl_sync(FULL, d.pairs, f);
            const uint32_t fcn = __shfl_sync(FULL, d.cnt, f);
            if (act) {
                const uint4 rp = *reinterpret_cast<const uint4 *>(P.sRowPtrC + fs * TILE);
                // r = #{r' in 1..15 : row_ptr[r'] <= q}  (bytewise compare; row_ptr[0] = 0)
                const uint32_t qq = q * 0x01010101u;
                const int rr = (__popc(__vcmpleu4(rp.x, qq)) + __popc(__vcmpleu4(rp.y, qq)) +
                                __popc(__vcmpleu4(rp.z, qq)) + __popc(__vcmpleu4(rp.w, qq))) / 8 - 1;
                const uint32_t rpw = rr < 4 ? rp.x : rr < 8 ? rp.y : rr < 12 ? rp.z : rp.w;
                const int kr = (int)q - (int)((rpw >> (8 * (rr & 3))) & 0xffu);
                const int j = (int)__fns((uint32_t)P.sMaskC[fs * TILE + rr], 0, kr + 1);
                const uint32_t lowj = (1u << j) - 1u;
                TO acc = (TO)0;
                // the next pair's masks and offsets are loaded while the current one multiplies
                uint64_t pr = P.pairs[fp];
                int64_t pA = (int64_t)(pr >> 32), pB = (int64_t)(uint32_t)pr;
                uint32_t mAr = P.mA[pA * TILE + rr], mTj = P.mTB[pB * TILE + j];
                int64_t zA = P.tnzA[pA] + P.rpA[pA * TILE + rr], zB = P.tnzB[pB];
                if (fcn > 1) pr = P.pairs[fp + 1];
                for (uint32_t p = 0; p < fcn; p++) {
                    const int64_t cB = pB, czA = zA, czB = zB;
                    uint32_t x = mAr & mTj;
                    const uint32_t cmA = mAr;
                    if (p + 1 < fcn) {
                        pA = (int64_t)(pr >> 32);
                        pB = (int64_t)(uint32_t)pr;
                        mAr = P.mA[pA * TILE + rr];
                        mTj = P.mTB[pB * TILE + j];
                        zA = P.tnzA[pA] + P.rpA[pA * TILE + rr];
                        zB = P.tnzB[pB];
                        if (p + 2 < fcn) pr = P.pairs[fp + p + 2];
                    }
                    while (x) {
                        const int c = __ffs(x) - 1;
                        x &= x - 1;
                        const TO a = vcvt<TO>(vA[czA + __popc(cmA & ((1u << c) - 1u))]);
                        const TO b = vcvt<TO>(vB[czB + P.rpB[cB * TILE + c] + __popc((uint32_t)P.mB[cB * TILE + c] & lowj)]);
                        acc = vfma(a, b, acc);
                    }
                }
                P.ixC[foff + q] = (uint8_t)((rr << 4) | j);
                vC[foff + q] = acc;
            }
        }
        __syncwarp();
    }
}

// dense C tiles (nnz >= t_nnz): a CTA per tile row (P:1862-1870 for the accumulator).  The row's
// A tiles are expanded once into shared memory (16 x 17 values each, absent entries 0), so every
// dense C tile of the row reuses them -- a pair then moves only its B tile.  Warp 0 walks the
// row's C tiles 32 at a time (their nnz and nonzero offsets, as k_num_rows computes them) and
// lists the dense ones; the warps take them in turn.  Per pair the warp expands B_KJ into a 16 x 16
// buffer (cleared, then scattered), and walks the columns c of colOcc(A_IK) & rowOcc(B_KJ) in
// ascending order in warp-uniform groups of four (no divergence, immediate-offset shared
// loads); lane (r, h) adds A(r, c) * B(c, 8h..8h+7) to its eight register accumulators.  The
// zeros are exact: a finite a times an absent B entry, or 0 times a finite B entry, adds +-0.  A
// pair with a non-finite value in A_IK or B_KJ instead takes mask-predicated FMAs over the true
// nonzeros (Inf * 0 never appears).  Every C entry receives its products in ascending k.
constexpr int DR_W = 4;  // warps per CTA
constexpr int DR_AP = 17;  // staged A row pitch (values): conflict-free column reads
template <typename TI, typename TO>
__global__ void __launch_bounds__(DR_W * 32) k_num_dense_row(RowNumParams P) { TSG_GRID_WAIT();
    extern __shared__ __align__(16) unsigned char dyn[];
    __shared__ int64_t dOff[32];
    __shared__ uint8_t dQ[32], sNF[MAX_A];
    __shared__ int dN;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, r = lane >> 1, h = lane & 1;
    const int64_t I = blockIdx.x;
    const int64_t t0 = P.tpC[I], nC = P.tpC[I + 1] - t0;
    if (nC == 0) return;  // CTA-uniform
    const int64_t a0 = P.tpA[I];
    const int nA = (int)(P.tpA[I + 1] - a0);
    const int64_t base = P.costOff[a0];
    TO *sA = reinterpret_cast<TO *>(dyn);                                 // [maxA][16 * 17]
    TO *Bd = sA + (int64_t)P.max_a_dense * TILE * DR_AP + w * TILE * TILE;  // this warp's B tile
    const TI *vA = static_cast<const TI *>(P.vA), *vB = static_cast<const TI *>(P.vB);
    int64_t zrow = P.rowOff[I];
    bool staged = false;
    u64c nden = 0;
    for (int64_t q0 = 0; q0 < nC; q0 += 32) {
        if (w == 0) {  // this chunk's dense tiles and their nonzero offsets
            const int64_t q = q0 + lane;
            const uint32_t nz = q < nC ? P.tNnz[base + q] : 0u;
            uint32_t incl = nz;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t o = __shfl_up_sync(FULL, incl, d);
                if (lane >= d) incl += o;
            }
            const bool isD = q < nC && (int)nz >= P.dense_threshold;
            const unsigned bd = __ballot_sync(FULL, isD);
            if (isD) {
                const int k = __popc(bd & ((1u << lane) - 1u));
                dQ[k] = (uint8_t)lane;
                dOff[k] = zrow + (incl - nz);
            }
            zrow += __shfl_sync(FULL, incl, 31);
            if (lane == 0) dN = __popc(bd);
        }
        __syncthreads();
        const int nd = dN;
        if (nd && !staged) {  // the row's A tiles, expanded (first chunk with a dense tile)
            for (int sI = w; sI < nA; sI += DR_W) {
                TO *As = sA + sI * TILE * DR_AP;
                for (int e = lane; e < TILE * DR_AP; e += 32) As[e] = (TO)0;
                __syncwarp();
                bool bad = false;
                for (int64_t e = P.tnzA[a0 + sI] + lane; e < P.tnzA[a0 + sI + 1]; e += 32) {
                    const uint32_t ix = P.ixA[e];
                    const TO v = vcvt<TO>(vA[e]);
                    bad |= !isfinite(v);
                    As[(ix >> 4) * DR_AP + (ix & 15)] = v;
                }
                const bool any = __any_sync(FULL, bad);
                if (lane == 0) sNF[sI] = any;
            }
            staged = true;
            __syncthreads();
        }
        nden += nd;
        for (int k = w; k < nd; k += DR_W) {
            const int64_t slot = base + q0 + dQ[k];
            const int64_t off = dOff[k];
            const uint64_t *pp = P.pairs + base + P.tStart[slot];
            const uint32_t cnt = P.tCnt[slot];
            TO acc[8];
#pragma unroll
            for (int jj = 0; jj < 8; jj++) acc[jj] = (TO)0;
            uint64_t prn = cnt ? pp[0] : 0;
            for (uint32_t p = 0; p < cnt; p++) {
                const uint64_t pr = prn;
                if (p + 1 < cnt) prn = pp[p + 1];
                const int sI = (int)((int64_t)(pr >> 32) - a0);
                const int64_t pB = (int64_t)(uint32_t)pr;
                const uint32_t u = (uint32_t)P.colOccA[a0 + sI] & (uint32_t)P.rowOccB[pB];
#pragma unroll
                for (int e = lane; e < TILE * TILE * (int)sizeof(TO) / 16; e += 32)
                    reinterpret_cast<uint4 *>(Bd)[e] = make_uint4(0u, 0u, 0u, 0u);
                __syncwarp();
                bool bad = false;
                for (int64_t e = P.tnzB[pB] + lane; e < P.tnzB[pB + 1]; e += 32) {
                    const uint32_t ix = P.ixB[e];
                    const TO v = vcvt<TO>(vB[e]);
                    bad |= !isfinite(v);
                    Bd[(ix >> 4) * TILE + (ix & 15)] = v;
                }
                const bool anybad = __any_sync(FULL, bad) || sNF[sI];
                __syncwarp();
                const TO *ar = sA + sI * TILE * DR_AP + r * DR_AP;
                const TO *bs = Bd + 8 * h;
                if (!anybad) {
#pragma unroll
                    for (int g = 0; g < TILE; g += 4) {
                        if ((u >> g) & 15u) {  // warp-uniform
#pragma unroll
                            for (int c = g; c < g + 4; c++) {
                                const TO a = ar[c];
                                TO b[8];
                                lds8(bs + c * TILE, b);
#pragma unroll
                                for (int jj = 0; jj < 8; jj++) acc[jj] = vfma(a, b[jj], acc[jj]);
                            }
                        }
                    }
                } else {
                    const uint32_t mAr = P.mA[(a0 + sI) * TILE + r];
                    for (int c = 0; c < TILE; c++) {
                        if ((u >> c) & (mAr >> c) & 1u) {
                            const TO a = ar[c];
                            const uint32_t mb = (uint32_t)P.mB[pB * TILE + c] >> (8 * h);
#pragma unroll
                            for (int jj = 0; jj < 8; jj++)
                                if ((mb >> jj) & 1u) acc[jj] = vfma(a, bs[c * TILE + jj], acc[jj]);
                        }
                    }
                }
                __syncwarp();  // the B buffer is rewritten by the next pair
            }
            const uint32_t mCr = P.sMaskC[slot * TILE + r];
            const int64_t ob = off + P.sRowPtrC[slot * TILE + r];
#pragma unroll
            for (int jj = 0; jj < 8; jj++) {
                const int j = 8 * h + jj;
                if ((mCr >> j) & 1u) {
                    const int q = __popc(mCr & ((1u << j) - 1u));
                    P.ixC[ob + q] = (uint8_t)((r << 4) | j);
                    static_cast<TO *>(P.vC)[ob + q] = acc[jj];
                }
            }
        }
        __syncthreads();  // warp 0 rewrites the list
    }
    if (threadIdx.x == 0 && nden) atomicAdd(&P.cnt->n3dense, nden);
}

template <typename TI, typename TO>
void launch_t(const RowNumParams &P, int64_t n_dense, cudaStream_t s, cudaStream_t sd) {
    TSG_LAUNCH((k_num_rows<TI, TO>), grid_for(ceil_div(P.tm, 2), RN_W), RN_T, 0, s, P);
    if (P.small) {  // persistent grid: the record count is read on the device
        static int occ = 0;
        int nsm = 148;
        if (!occ) {
            int dev = 0;
            cudaGetDevice(&dev);
            cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_num_small<TI, TO>, NS_T, 0);
            occ = std::max(occ, 1) * nsm;
        }
        // small C tiles <= C's tiles: no more CTAs than 32-tile groups of them
        const int64_t need = ceil_div(ceil_div(P.ntC, 32), NS_T / 32);
        TSG_LAUNCH((k_num_small<TI, TO>), (unsigned)std::max<int64_t>(1, std::min<int64_t>(occ, need)), NS_T, 0, s, P);
    }
    if (n_dense > 0) {
        const size_t smem = ((size_t)P.max_a_dense * TILE * DR_AP + (size_t)DR_W * TILE * TILE) * sizeof(TO);
        TSG_CUDA(cudaFuncSetAttribute(k_num_dense_row<TI, TO>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        TSG_LAUNCH((k_num_dense_row<TI, TO>), (unsigned)P.tm, DR_W * 32, smem, sd, P);
    }
}

}  // namespace

void launch_num_rows(const RowNumArgs &a, cudaStream_t s, cudaStream_t sd) {
    RowNumParams P{};
    P.tm = a.tm;
    P.ntC = a.ntC;
    P.tpA = a.A->tile_ptr;
    P.tnzA = a.A->tile_nnz;
    P.rpA = a.A->row_ptr;
    P.ixA = a.A->idx;
    P.mA = a.A->mask;
    P.vA = a.A->val;
    P.tnzB = a.B->tile_nnz;
    P.rpB = a.B->row_ptr;
    P.ixB = a.B->idx;
    P.mB = a.B->mask;
    P.mTB = a.mTB;
    P.rowOccB = a.rowOccB;
    P.vB = a.B->val;
    P.costOff = a.costOff;
    P.pairs = a.pairs;
    P.tJ = a.tJ;
    P.tStart = a.tStart;
    P.tCnt = a.tCnt;
    P.tNnz = a.tNnz;
    P.sMaskC = a.sMaskC;
    P.sRowPtrC = a.sRowPtrC;
    P.rowOff = a.rowOff;
    P.tpC = a.C->tile_ptr;
    P.tcC = a.C->tile_col;
    P.tnzC = a.C->tile_nnz;
    P.rpC = a.C->row_ptr;
    P.ixC = a.C->idx;
    P.mC = a.C->mask;
    P.vC = a.C->val;
    P.dense_threshold = a.dense_threshold;
    P.small_max = a.small_max;
    P.max_a_dense = a.max_a_dense;
    P.colOccA = a.colOccA;
    P.small = static_cast<RowTileRec *>(a.small);
    P.cnt = a.cnt;
    switch (a.A->dtype) {
        case TSG_F64: launch_t<double, double>(P, a.n_dense, s, sd); break;
        case TSG_F32: launch_t<float, float>(P, a.n_dense, s, sd); break;
        default: launch_t<__half, float>(P, a.n_dense, s, sd);
    }
}

}  // namespace tsg
