// tsg_step23.cu -- SURVEY §8(a) rows a2 (step 2, bit-mask symbolic) and a4 (step 3, numeric with
// the adaptive accumulator) of Section 3.3.
//
// Step 2 (Alg 2 l.19-25): for every matched pair (A_IK, B_KJ) and every
// nonzero (r,c) of A_IK, mask_C[r] |= mask_B_KJ[c]; then popcounts, the 16 local row offsets and
// the tile nnz.  Step 3 (Alg 3): C(r,j) = sum over pairs (ascending K),
// over c (ascending) of A(r,c)*B(c,j); sparse accumulator addressed through mask_C below
// t_nnz, dense 16x16 accumulator at or above it (reading A7).
//
// Warps take groups of 32 consecutive C tiles (tile order keeps the B tiles of neighbouring tile
// rows hot in L2) and split each group by size so lanes stay busy (the paper uses one warp per
// tile):
//   step 2  light tiles (<= 16 (pair, c) items): one thread per tile, item driven
//           heavy tiles: a half warp per tile, lane r owns row r
//   step 3  small tiles (nnz <= 16): one thread per tile, item driven, mask-addressed slots
//           medium tiles: a half warp per tile, lane r owns row r (dense-in-j row accumulator)
//           dense tiles (nnz >= t_nnz): a warp per tile, both tiles staged densely
// An item is (pair, c) with c a column of A_IK whose row c of B_KJ is non-empty: it contributes
// the outer product (rows of A_IK's column c) x (columns of B_KJ's row c); pairs and columns
// without products are skipped through the occupancy words.
// Every accumulator slot has exactly one owner thread and products reach it in ascending k
// (pairs ascending K, then c ascending), so no atomics are needed and results are bitwise
// deterministic (readings A8/A16).
#include <algorithm>
#include <cstdlib>
#include <map>
#include <mutex>

#include "tsg_device.cuh"

namespace tsg {
namespace {

constexpr unsigned FULL = 0xffffffffu;
#ifndef TSG_T2
#define TSG_T2 256
#endif
#ifndef TSG_T3
#define TSG_T3 128
#endif
#ifndef TSG_TS
#define TSG_TS 256
#endif
constexpr int T2 = TSG_T2;  // step-2 CTA
constexpr int T3 = TSG_T3;  // step-3 CTA (4 warps; 7.7 KB of shared memory per warp)
constexpr int BATCH = 16;  // step 2: pairs staged per half warp at a time
constexpr int BATCH3 = 16; // step 3: pairs staged per half warp at a time (also the small path's 16 slots)

// ==========================================================================================
// step 2
// ==========================================================================================
// light tiles (<= LIGHT_WORK (pair, c) items): one thread per tile, item driven, row masks in 8
// thread-private shared words.  A separate kernel at full occupancy: the work is a chain of
// dependent loads (pair -> occupancy words -> masks), so the next pair's occupancy words are
// loaded while the current pair is OR-ed.
constexpr int T2L = 256;

__global__ void __launch_bounds__(T2L, 8) k_s2_light(StepParams P) { TSG_GRID_WAIT();
    __shared__ uint32_t wsm[8 * T2L];
    uint32_t *w = wsm + threadIdx.x;
    const int lane = threadIdx.x & 31;
    u64c nl = 0, nd = 0;
    // the 32 lanes of a warp hold the 32 tiles of one group
    WorkQueue wq(&P.cnt->q[0][0], (P.ntC + 31) / 32, P.qchunk[0], lane, T2L / 32);
    for (int64_t gq; wq.next(gq, lane);) {
        const int64_t t0 = gq * 32;
        const int64_t t = t0 + lane;
        int total = -1;
        if (t < P.ntC && P.work[t] <= (uint32_t)LIGHT_WORK) {
        nl++;
#pragma unroll
        for (int q = 0; q < 8; q++) w[q * T2L] = 0;
        const uint64_t *pp = P.pairs + P.pairBeg[t];
        const uint32_t np = P.pairCnt[t];
        if (P.recA) {
            // hypersparse operands: a pair of single-nonzero tiles contributes the one bit
            // (r_A, c_B) iff c_A == r_B, from the two records alone
            const uint4 *RA = reinterpret_cast<const uint4 *>(P.recA), *RB = reinterpret_cast<const uint4 *>(P.recB);
            uint64_t pr = pp[0];
            int64_t pA = (int64_t)(pr >> 32), pB = (int64_t)(uint32_t)pr;
            uint4 ra = RA[pA], rb = RB[pB];
            if (np > 1) pr = pp[1];
            for (uint32_t p = 0; p < np; p++) {
                const uint4 ca = ra, cb = rb;
                const int64_t cA = pA, cB = pB;
                if (p + 1 < np) {
                    pA = (int64_t)(pr >> 32);
                    pB = (int64_t)(uint32_t)pr;
                    ra = RA[pA];
                    rb = RB[pB];
                    if (p + 2 < np) pr = pp[p + 2];
                }
                const bool sa = (ca.w >> 24) & 1u, sb = (cb.w >> 24) & 1u;
                const uint32_t ia = (ca.w >> 16) & 0xffu, ib = (cb.w >> 16) & 0xffu;
                if (sa && sb) {
                    if ((ia & 15u) == (ib >> 4)) {
                        const int r = (int)(ia >> 4);
                        w[(r >> 1) * T2L] |= (1u << (ib & 15u)) << (16 * (r & 1));
                    }
                    continue;
                }
                uint32_t cx = (sa ? 1u << (ia & 15u) : (uint32_t)P.colOccA[cA]) & (cb.w & 0xffffu);
                const uint16_t *mb = P.mB + cB * TILE;
                const uint16_t *at = P.mTA + cA * TILE;
                while (cx) {
                    const int c = __ffs(cx) - 1;
                    cx &= cx - 1;
                    const uint32_t bits = sb ? 1u << (ib & 15u) : (uint32_t)mb[c];
                    uint32_t rows = sa ? 1u << (ia >> 4) : (uint32_t)at[c];
                    while (rows) {
                        const int r = __ffs(rows) - 1;
                        rows &= rows - 1;
                        w[(r >> 1) * T2L] |= bits << (16 * (r & 1));
                    }
                }
            }
        } else {
            uint64_t pr = pp[0];
            int64_t pA = (int64_t)(pr >> 32), pB = (int64_t)(uint32_t)pr;
            uint32_t x = (uint32_t)P.colOccA[pA] & P.rowOccB[pB];
            if (np > 1) pr = pp[1];
            for (uint32_t p = 0; p < np; p++) {
                const int64_t cA = pA, cB = pB;
                uint32_t cx = x;
                if (p + 1 < np) {
                    pA = (int64_t)(pr >> 32);
                    pB = (int64_t)(uint32_t)pr;
                    x = (uint32_t)P.colOccA[pA] & P.rowOccB[pB];
                    if (p + 2 < np) pr = pp[p + 2];
                }
                const uint16_t *mb = P.mB + cB * TILE;
                const uint16_t *at = P.mTA + cA * TILE;
                while (cx) {
                    const int c = __ffs(cx) - 1;
                    cx &= cx - 1;
                    const uint32_t bits = mb[c];
                    uint32_t rows = at[c];
                    while (rows) {
                        const int r = __ffs(rows) - 1;
                        rows &= rows - 1;
                        w[(r >> 1) * T2L] |= bits << (16 * (r & 1));
                    }
                }
            }
        }
        uint32_t m[8];
        uint32_t rp[4] = {0, 0, 0, 0};
        total = 0;
#pragma unroll
        for (int q = 0; q < 8; q++) m[q] = w[q * T2L];
#pragma unroll
        for (int r = 0; r < 16; r++) {
            rp[r >> 2] |= (uint32_t)total << (8 * (r & 3));
            total += __popc((m[r >> 1] >> (16 * (r & 1))) & 0xffffu);
        }
        uint4 *dm = reinterpret_cast<uint4 *>(P.mC + t * TILE);
        dm[0] = make_uint4(m[0], m[1], m[2], m[3]);
        dm[1] = make_uint4(m[4], m[5], m[6], m[7]);
        *reinterpret_cast<uint4 *>(P.rpC + t * TILE) = make_uint4(rp[0], rp[1], rp[2], rp[3]);
        P.tnzC[t] = total;
        nd += total >= P.dense_threshold;
        }
        // step-3 classes of the group's light tiles (medium / dense bit masks; heavy tiles: k_s2)
        const unsigned mm = __ballot_sync(FULL, total > P.small_max && total < P.dense_threshold);
        const unsigned dn = __ballot_sync(FULL, total >= P.dense_threshold);
        if (lane == 0) {
            P.medL[t0 >> 5] = mm;
            P.denL[t0 >> 5] = dn;
        }
    }
    for (int o = 16; o > 0; o >>= 1) nl += __shfl_xor_sync(FULL, nl, o);
    if ((threadIdx.x & 31) == 0 && nl) atomicAdd(&P.cnt->n2light, nl);
    for (int o = 16; o > 0; o >>= 1) nd += __shfl_xor_sync(FULL, nd, o);
    if ((threadIdx.x & 31) == 0 && nd) atomicAdd(&P.cnt->n2dense, nd);
}

#ifndef TSG_S2_MINB
#define TSG_S2_MINB 1
#endif
__global__ void __launch_bounds__(T2, TSG_S2_MINB) k_s2(StepParams P) { TSG_GRID_WAIT();
    __shared__ __align__(16) uint16_t sMA[T2 / 16][BATCH][TILE], sMB[T2 / 16][BATCH][TILE];
    __shared__ uint16_t sOB[T2 / 16][BATCH];
    const int lane = threadIdx.x & 31, r = lane & 15, half = lane >> 4, hw = threadIdx.x >> 4;
    const int64_t ngroups = (P.ntC + 31) / 32;
    WorkQueue wq(&P.cnt->q[1][0], ngroups, P.qchunk[1], lane, T2 / 32);
    for (int64_t g; wq.next(g, lane);) {
        const int64_t t = g * 32 + lane;
        const bool v = t < P.ntC;
        const bool light = v && P.work[t] <= (uint32_t)LIGHT_WORK;  // k_s2_light's class
        unsigned hm = __ballot_sync(FULL, v && !light);
        unsigned medH = 0, denH = 0;  // step-3 classes of the group's heavy tiles
        // heavy tiles: two at a time, a half warp each, lane r owns row r; per batch of 16 pairs
        // lane i stages pair i's A and B masks (4 x 16-byte cp.async, all in flight at once)
        while (hm) {
            const int f0 = __ffs(hm) - 1;
            hm &= hm - 1;
            const int f1 = hm ? __ffs(hm) - 1 : -1;
            if (hm) hm &= hm - 1;
            const int mine = half ? f1 : f0;
            const bool hv = mine >= 0;
            const int64_t th = g * 32 + (hv ? mine : 0);
            uint32_t acc = 0, np = 0;
            const uint64_t *pp = P.pairs;
            if (hv) {
                pp += P.pairBeg[th];
                np = P.pairCnt[th];
            }
            const uint32_t nbat = (np + BATCH - 1) / BATCH;
            const uint32_t nbw = max(nbat, __shfl_xor_sync(FULL, nbat, 16));
            for (uint32_t bt = 0; bt < nbw; bt++) {
                const uint32_t q = bt * BATCH + r;
                if (q < np) {
                    const uint64_t pr = pp[q];
                    const int64_t pA = (int64_t)(pr >> 32), pB = (int64_t)(uint32_t)pr;
                    cp16(&sMA[hw][r][0], P.mA + pA * TILE);
                    cp16(&sMA[hw][r][8], P.mA + pA * TILE + 8);
                    cp16(&sMB[hw][r][0], P.mB + pB * TILE);
                    cp16(&sMB[hw][r][8], P.mB + pB * TILE + 8);
                    sOB[hw][r] = P.rowOccB[pB];
                }
                asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;\n" ::: "memory");
                __syncwarp();
                const uint32_t nb = np > bt * BATCH ? min((uint32_t)BATCH, np - bt * BATCH) : 0u;
                for (uint32_t i = 0; i < nb; i++) {
                    uint32_t ma = sMA[hw][i][r] & sOB[hw][i];
                    const uint16_t *mb = sMB[hw][i];
                    while (ma) {
                        const int c = __ffs(ma) - 1;
                        ma &= ma - 1;
                        acc |= mb[c];
                    }
                }
                __syncwarp();
            }
            const int cnt = __popc(acc);
            int incl = cnt;
#pragma unroll
            for (int d = 1; d < 16; d <<= 1) {
                const int o = __shfl_up_sync(FULL, incl, d, 16);
                if (r >= d) incl += o;
            }
            const int tot = __shfl_sync(FULL, incl, 15, 16);
            if (hv) {
                P.mC[th * TILE + r] = (uint16_t)acc;
                P.rpC[th * TILE + r] = (uint8_t)(incl - cnt);
                if (r == 0) P.tnzC[th] = tot;
            }
            const unsigned dn = __ballot_sync(FULL, hv && r == 0 && tot >= P.dense_threshold);
            const unsigned md = __ballot_sync(FULL, hv && r == 0 && tot > P.small_max && tot < P.dense_threshold);
            if (lane == 0 && dn) atomicAdd(&P.cnt->n2dense, (u64c)__popc(dn));
            denH |= ((dn & 1u) ? 1u << f0 : 0u) | ((dn >> 16) & 1u ? 1u << f1 : 0u);
            medH |= ((md & 1u) ? 1u << f0 : 0u) | ((md >> 16) & 1u ? 1u << f1 : 0u);
        }
        if (lane == 0) {
            P.medH[g] = medH;
            P.denH[g] = denH;
        }
        const unsigned lm = __ballot_sync(FULL, light), vm = __ballot_sync(FULL, v);
        if (lane == 0 && vm != lm) atomicAdd(&P.cnt->n2heavy, (u64c)(__popc(vm) - __popc(lm)));
    }
}

// ==========================================================================================
// step 3
// ==========================================================================================
// per-warp shared scratch of the medium class: 4 KB of row accumulators + two MedStage (one per
// half warp)
constexpr int WACC = 4096;

struct MedStage {  // per half warp: staged metadata and tile masks / row offsets of up to 16 pairs
    uint16_t mA[BATCH3][TILE], mB[BATCH3][TILE];  // cp.async'd masks of A_IK and B_KJ
    uint8_t rA[BATCH3][TILE], rB[BATCH3][TILE];   // and their row offsets
    int64_t zA[BATCH3], zB[BATCH3];
    uint16_t oB[BATCH3];
};

constexpr int WREG = WACC + 2 * (int)sizeof(MedStage);
static_assert(BATCH3 == 16 && BATCH == 16, "staging lane r of a half warp stages pair r of the batch");
static_assert(sizeof(MedStage) % 16 == 0, "MedStage keeps 16-byte alignment");

// small tiles (nnz <= small_max): one lane per C nonzero (output-stationary; the paper's sparse
// accumulator, with each slot owned by one lane).  Entry q of tile t is (r, j): r =
// the last row whose offset row_ptr_C[r] <= q, j = the (q - row_ptr_C[r])-th set bit of
// mask_C[r].  The lane walks its tile's pairs in ascending K; for each, the intersection
// mask_A[r] & colmask_B[j] gives the contributing c (ascending), and A(r,c), B(c,j) are found by
// popcount addressing.  The kernel is latency bound (dependent chains pair -> tile metadata ->
// values), so it runs alone at full occupancy (no staging, few registers) and pipelines the
// per-pair metadata one pair ahead.
constexpr int TS = TSG_TS;  // small-class CTA
constexpr int SMAP = 32 * 16;  // entry -> tile map bytes per warp (small_max <= 16)

// STAGE (hypersparse inputs, where B's tile metadata misses in cache): a lane-private double buffer
// of the B tile's row offsets and row masks of the next pair ([buffer][chunk: row_ptr, mask rows
// 0-7, mask rows 8-15][thread], 16 bytes each) is filled by cp.async one pair ahead, so a
// product's B address needs a shared load instead of a dependent global one.  On cache-friendly
// inputs (stencils: B's metadata hits L1) the staging is pure overhead and STAGE is off.
// CTAs per SM of k_s3_small: 6 for the plain form (C2: 1.26 -> 1.21 ms against 5), 5 for the
// staged and record forms (C5's record form: step 3 170 ms at 5, 179 at 6; 7+ spills heavily)
#ifndef TSG_SMALL_MINB
#define TSG_SMALL_MINB 5
#endif
#ifndef TSG_SMALL_MINB_PLAIN
#define TSG_SMALL_MINB_PLAIN 6
#endif
// REC (hypersparse operands, the default there): per pair the two tiles' 16-byte records; a
// single-nonzero tile needs nothing else (its entry and value are inline), a multi-nonzero tile
// its masks and row offsets as in the plain form.
template <typename TO, typename TI>
__device__ __forceinline__ TO rec_value(const uint4 &r) {
    if constexpr (sizeof(TI) == 8) return vcvt<TO>(__hiloint2double((int)r.y, (int)r.x));
    else if constexpr (sizeof(TI) == 4) return vcvt<TO>(__int_as_float((int)r.x));
    else return vcvt<TO>(__ushort_as_half((unsigned short)(r.x & 0xffffu)));
}

template <typename TI, typename TO, int MODE>  // MODE 0: plain, 1: STAGE, 2: REC
__global__ void __launch_bounds__(TS, MODE == 0 ? TSG_SMALL_MINB_PLAIN : TSG_SMALL_MINB) k_s3_small(StepParams P) { TSG_GRID_WAIT();
    constexpr bool STAGE = MODE == 1;
    __shared__ uint8_t mapsm[TS / 32][SMAP];
    __shared__ __align__(16) uint4 stg[STAGE ? 2 : 1][3][STAGE ? TS : 1];
    const TI *vA = static_cast<const TI *>(P.vA), *vB = static_cast<const TI *>(P.vB);
    TO *vC = static_cast<TO *>(P.vC);
    const int lane = threadIdx.x & 31;
    uint8_t *map = mapsm[threadIdx.x >> 5];
    const int64_t ngroups = (P.ntC + 31) / 32;
    WorkQueue wq(&P.cnt->q[2][0], ngroups, P.qchunk[2], lane, TS / 32);
    for (int64_t g; wq.next(g, lane);) {
        const int64_t tl = g * 32 + lane;
        const bool v = tl < P.ntC;
        const int nz = v ? (int)(P.tnzC[tl + 1] - P.tnzC[tl]) : 0;
        const bool small = v && nz < P.dense_threshold && nz <= P.small_max;
        const int mine = small ? nz : 0;
        int incl = mine;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const int o = __shfl_up_sync(FULL, incl, d);
            if (lane >= d) incl += o;
        }
        const int excl = incl - mine;
        const int tot = __shfl_sync(FULL, incl, 31);
        const unsigned smask = __ballot_sync(FULL, small);
        if (lane == 0 && smask) atomicAdd(&P.cnt->n3small, (u64c)__popc(smask));
        if (tot == 0) continue;
        for (int q = 0; q < mine; q++) map[excl + q] = (uint8_t)lane;
        __syncwarp();
        for (int e0 = 0; e0 < tot; e0 += 32) {
            const int e = e0 + lane;
            const bool act = e < tot;
            const int f = act ? map[e] : 0;
            const int q = e - __shfl_sync(FULL, excl, f);
            if (act) {
                const int64_t t = g * 32 + f;
                const uint4 rp = *reinterpret_cast<const uint4 *>(P.rpC + t * TILE);
                const uint64_t *pp = P.pairs + P.pairBeg[t];
                const uint32_t np = P.pairCnt[t];
                const int64_t o = P.tnzC[t] + q;
                // r = #{r' in 1..15 : row_ptr[r'] <= q}  (bytewise compare; row_ptr[0] = 0)
                const uint32_t qq = (uint32_t)q * 0x01010101u;
                const int r = (__popc(__vcmpleu4(rp.x, qq)) + __popc(__vcmpleu4(rp.y, qq)) +
                               __popc(__vcmpleu4(rp.z, qq)) + __popc(__vcmpleu4(rp.w, qq))) / 8 - 1;
                const uint32_t rpw = r < 4 ? rp.x : r < 8 ? rp.y : r < 12 ? rp.z : rp.w;
                const int k = q - (int)((rpw >> (8 * (r & 3))) & 0xffu);
                const int j = (int)__fns((uint32_t)P.mC[t * TILE + r], 0, k + 1);
                const uint32_t lowj = (1u << j) - 1u;
                TO acc = 0;
                if constexpr (MODE == 2) {
                const uint4 *RA = reinterpret_cast<const uint4 *>(P.recA), *RB = reinterpret_cast<const uint4 *>(P.recB);
                uint64_t prn = pp[0];
                int64_t pA = (int64_t)(prn >> 32), pB = (int64_t)(uint32_t)prn;
                uint4 ra = RA[pA], rb = RB[pB];
                if (np > 1) prn = pp[1];
                for (uint32_t p = 0; p < np; p++) {
                    const uint4 ca = ra, cb = rb;
                    const int64_t cpA = pA, cpB = pB;
                    if (p + 1 < np) {  // the next pair's records are loaded while this one multiplies
                        pA = (int64_t)(prn >> 32);
                        pB = (int64_t)(uint32_t)prn;
                        ra = RA[pA];
                        rb = RB[pB];
                        if (p + 2 < np) prn = pp[p + 2];
                    }
                    const bool sa = (ca.w >> 24) & 1u, sb = (cb.w >> 24) & 1u;
                    const uint32_t ia = (ca.w >> 16) & 0xffu, ib = (cb.w >> 16) & 0xffu;
                    if (sa && sb) {
                        if ((int)(ia >> 4) == r && (ia & 15u) == (ib >> 4) && (int)(ib & 15u) == j)
                            acc = vfma(rec_value<TO, TI>(ca), rec_value<TO, TI>(cb), acc);
                        continue;
                    }
                    const uint32_t mAr = sa ? ((int)(ia >> 4) == r ? 1u << (ia & 15u) : 0u) : (uint32_t)P.mA[cpA * TILE + r];
                    const uint32_t mTj = sb ? ((int)(ib & 15u) == j ? 1u << (ib >> 4) : 0u) : (uint32_t)P.mTB[cpB * TILE + j];
                    uint32_t x = mAr & mTj;
                    if (!x) continue;
                    const int64_t zA = sa ? 0 : (int64_t)ca.x + ((int64_t)ca.y << 32) + P.recA_voff + P.rpA[cpA * TILE + r];
                    const int64_t zB = sb ? 0 : (int64_t)cb.x + ((int64_t)cb.y << 32);
                    while (x) {
                        const int c = __ffs(x) - 1;
                        x &= x - 1;
                        const TO a = sa ? rec_value<TO, TI>(ca) : vcvt<TO>(vA[zA + __popc(mAr & ((1u << c) - 1u))]);
                        const TO b = sb ? rec_value<TO, TI>(cb)
                                        : vcvt<TO>(vB[zB + P.rpB[cpB * TILE + c] + __popc((uint32_t)P.mB[cpB * TILE + c] & lowj)]);
                        acc = vfma(a, b, acc);
                    }
                }
                } else if constexpr (!STAGE) {
                // pair p's metadata is loaded while pair p-1 is being multiplied
                uint64_t prn = pp[0];
                int64_t pA = (int64_t)(prn >> 32), pB = (int64_t)(uint32_t)prn;
                uint32_t mAr = P.mA[pA * TILE + r], mTj = P.mTB[pB * TILE + j];
                int64_t zA = P.tnzA[pA] + P.rpA[pA * TILE + r], zB = P.tnzB[pB];
                if (np > 1) prn = pp[1];
                for (uint32_t p = 0; p < np; p++) {
                    const int64_t cB = pB, czA = zA, czB = zB;
                    uint32_t x = mAr & mTj;
                    const uint32_t cmA = mAr;
                    if (p + 1 < np) {
                        pA = (int64_t)(prn >> 32);
                        pB = (int64_t)(uint32_t)prn;
                        mAr = P.mA[pA * TILE + r];
                        mTj = P.mTB[pB * TILE + j];
                        zA = P.tnzA[pA] + P.rpA[pA * TILE + r];
                        zB = P.tnzB[pB];
                        if (p + 2 < np) prn = pp[p + 2];
                    }
                    while (x) {
                        const int c = __ffs(x) - 1;
                        x &= x - 1;
                        const TO a = vcvt<TO>(vA[czA + __popc(cmA & ((1u << c) - 1u))]);
                        const TO b = vcvt<TO>(vB[czB + P.rpB[cB * TILE + c] + __popc((uint32_t)P.mB[cB * TILE + c] & lowj)]);
                        acc = vfma(a, b, acc);
                    }
                }
                } else {
                // three-stage pipeline over the tile's pairs: pair p+2's row masks are loaded,
                // pair p+1's B row offsets and masks are staged (cp.async, only if the pair meets
                // this entry: mask_A[r] & colmask_B[j] != 0), pair p is multiplied
                const uint8_t *sb0 = reinterpret_cast<const uint8_t *>(&stg[0][0][threadIdx.x]);
                constexpr int BUFB = 3 * TS * 16, CHB = TS * 16;  // buffer / chunk strides in bytes
                auto stage = [&](int bf, int64_t b) {
                    cp16(&stg[bf][0][threadIdx.x], P.rpB + b * TILE);
                    cp16(&stg[bf][1][threadIdx.x], P.mB + b * TILE);
                    cp16(&stg[bf][2][threadIdx.x], P.mB + b * TILE + 8);
                };
                uint64_t prn = pp[0];
                int64_t pB = (int64_t)(uint32_t)prn, pA = (int64_t)(prn >> 32);
                uint32_t mAr = P.mA[pA * TILE + r];
                uint32_t x = mAr & P.mTB[pB * TILE + j];
                int64_t zA = P.tnzA[pA] + P.rpA[pA * TILE + r], zB = P.tnzB[pB];
                if (x) stage(0, pB);
                asm volatile("cp.async.commit_group;\n" ::: "memory");
                // pair p+1: masks in flight
                uint32_t mAn = 0, mTn = 0;
                int64_t zAn = 0, zBn = 0, pBn = 0;
                if (np > 1) {
                    prn = pp[1];
                    pA = (int64_t)(prn >> 32);
                    pBn = (int64_t)(uint32_t)prn;
                    mAn = P.mA[pA * TILE + r];
                    mTn = P.mTB[pBn * TILE + j];
                    zAn = P.tnzA[pA] + P.rpA[pA * TILE + r];
                    zBn = P.tnzB[pBn];
                    if (np > 2) prn = pp[2];
                }
                for (uint32_t p = 0; p < np; p++) {
                    const int64_t czA = zA, czB = zB;
                    const uint32_t cx = x, cmA = mAr;
                    const int buf = p & 1;
                    if (p + 1 < np) {
                        // pair p+1 becomes the staged pair; pair p+2's masks are loaded
                        mAr = mAn;
                        x = mAn & mTn;
                        zA = zAn;
                        zB = zBn;
                        if (x) stage(buf ^ 1, pBn);
                        if (p + 2 < np) {
                            pA = (int64_t)(prn >> 32);
                            pBn = (int64_t)(uint32_t)prn;
                            mAn = P.mA[pA * TILE + r];
                            mTn = P.mTB[pBn * TILE + j];
                            zAn = P.tnzA[pA] + P.rpA[pA * TILE + r];
                            zBn = P.tnzB[pBn];
                            if (p + 3 < np) prn = pp[p + 3];
                        }
                    }
                    asm volatile("cp.async.commit_group;\ncp.async.wait_group 1;\n" ::: "memory");
                    const uint8_t *sb = sb0 + buf * BUFB;
                    uint32_t xx = cx;
                    while (xx) {
                        const int c = __ffs(xx) - 1;
                        xx &= xx - 1;
                        const TO a = vcvt<TO>(vA[czA + __popc(cmA & ((1u << c) - 1u))]);
                        const uint32_t rb = sb[c];
                        const uint32_t mb = *reinterpret_cast<const uint16_t *>(sb + CHB * (1 + (c >> 3)) + 2 * (c & 7));
                        const TO b = vcvt<TO>(vB[czB + rb + __popc(mb & lowj)]);
                        acc = vfma(a, b, acc);
                    }
                }
                asm volatile("cp.async.wait_group 0;\n" ::: "memory");
                }
                P.ixC[o] = (uint8_t)((r << 4) | j);
                vC[o] = acc;
            }
        }
        __syncwarp();
    }
}

// A lane's item stream of one batch (medium tiles, lane r owns C row r).  An item is (pair i, c)
// with c in mask_A_i[r] & rowOcc(B_i): a = A_i(r,c) and B_i's row c (mask, first three values,
// pointer to the rest).  Items come pair-ascending then c-ascending, so every C(r,j) receives its
// products in ascending k.
template <typename TI, typename TO>
struct ItemStream {
    uint32_t rel;  // batch pairs that touch row r (mask_A_i[r] & rowOcc(B_i) != 0), not yet started
    int pi = 0;
    uint32_t mAr = 0, ma = 0;
    const TI *va = nullptr, *vbt = nullptr;
    // next item -> (a, b0..b2, mb, vb); false when the batch is exhausted
    __device__ __forceinline__ bool fetch(const StepParams &P, const MedStage &S, int r, TO &a, TO &b0, TO &b1,
                                          TO &b2, uint32_t &mb, const TI *&vb) {
        if (!ma) {
            if (!rel) return false;
            pi = __ffs(rel) - 1;
            rel &= rel - 1;
            mAr = S.mA[pi][r];
            ma = mAr & S.oB[pi];
            va = static_cast<const TI *>(P.vA) + S.zA[pi] + S.rA[pi][r];
            vbt = static_cast<const TI *>(P.vB) + S.zB[pi];
        }
        const int c = __ffs(ma) - 1;
        ma &= ma - 1;
        a = vcvt<TO>(va[__popc(mAr & ((1u << c) - 1u))]);
        mb = S.mB[pi][c];
        vb = vbt + S.rB[pi][c];
        const int n = __popc(mb);  // >= 1: row c of B_i is non-empty (rowOcc filter)
        b0 = vcvt<TO>(vb[0]);
        b1 = n > 1 ? vcvt<TO>(vb[1]) : (TO)0;
        b2 = n > 2 ? vcvt<TO>(vb[2]) : (TO)0;
        return true;
    }
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

// medium tile: a half warp, lane r owns C row r; dense-in-j 16-slot row accumulator in shared
// memory (conflict free), compacted through mask_C[r] at the end.  Pairs go in batches of 16:
// lane i stages pair i's A and B masks and row offsets (6 x 16-byte cp.async, all lanes and
// pairs in flight at once), so a lane's walk over its row touches global memory only for the
// values.  Each lane then runs its own flat item stream over the batch with two register sets
// (the next item's loads are in flight while the current one accumulates).  All 32 lanes must
// call.
// per-lane metadata of a medium tile, loaded one tile ahead (the chain tile -> pair list -> masks
// would otherwise be exposed at the start of every tile)
struct MedMeta {
    bool hv = false;
    int64_t t = 0;
    const uint64_t *pp = nullptr;
    uint32_t np = 0, mCr = 0;
    int64_t ob = 0;    // output offset of row r
    uint64_t pr = 0;   // pair r of the first batch
    __device__ __forceinline__ void load(const StepParams &P, int mine, int64_t g, int r) {
        hv = mine >= 0;
        t = g * 32 + (hv ? mine : 0);
        np = 0;
        mCr = 0;
        if (hv) {
            pp = P.pairs + P.pairBeg[t];
            np = P.pairCnt[t];
            mCr = P.mC[t * TILE + r];
            ob = P.tnzC[t] + P.rpC[t * TILE + r];
            if ((uint32_t)r < np) pr = pp[r];
        }
    }
};

template <typename TI, typename TO>
__device__ __forceinline__ void s3_medium(const StepParams &P, const MedMeta &M, TO *acc, MedStage &S, int r) {
    const uint32_t np = M.np, mCr = M.mCr;
    const uint64_t *pp = M.pp;
    const uint32_t nbat = (np + BATCH3 - 1) / BATCH3;
    const uint32_t nbw = max(nbat, __shfl_xor_sync(FULL, nbat, 16));
    for (uint32_t bt = 0; bt < nbw; bt++) {
        const uint32_t q = bt * BATCH3 + r;
        // lane r stages pair q of the batch and finds the rows of its A tile that meet a non-empty
        // row of its B tile (bit r' <=> mask_A[r'] & rowOcc(B) != 0); a bit transpose then gives
        // every lane the batch pairs that touch its own row
        uint32_t rows = 0;
        if (q < np) {
            const uint64_t pr = bt == 0 ? M.pr : pp[q];
            const int64_t pA = (int64_t)(pr >> 32), pB = (int64_t)(uint32_t)pr;
#ifdef TSG_MED_REL_LOOP
            cp16(&S.mA[r][0], P.mA + pA * TILE);
            cp16(&S.mA[r][8], P.mA + pA * TILE + 8);
#else
            const uint4 *ga = reinterpret_cast<const uint4 *>(P.mA + pA * TILE);
            const uint4 a0 = ga[0], a1 = ga[1];
#endif
            cp16(&S.mB[r][0], P.mB + pB * TILE);
            cp16(&S.mB[r][8], P.mB + pB * TILE + 8);
            cp16(&S.rA[r][0], P.rpA + pA * TILE);
            cp16(&S.rB[r][0], P.rpB + pB * TILE);
            S.zA[r] = P.tnzA[pA];
            S.zB[r] = P.tnzB[pB];
            const uint32_t ob = P.rowOccB[pB];
            S.oB[r] = (uint16_t)ob;
#ifndef TSG_MED_REL_LOOP
            reinterpret_cast<uint4 *>(&S.mA[r][0])[0] = a0;
            reinterpret_cast<uint4 *>(&S.mA[r][0])[1] = a1;
            rows = rows_meeting(a0, a1, ob);
#endif
        }
#ifndef TSG_MED_REL_LOOP
        const uint32_t rel = bit_transpose16(rows, r);
        cp_wait_all();
        __syncwarp();
#else
        cp_wait_all();
        __syncwarp();
        uint32_t rel = 0;
        {
            const int nb = np > bt * BATCH3 ? (int)min((uint32_t)BATCH3, np - bt * BATCH3) : 0;
            for (int i = 0; i < nb; i++) rel |= (S.mA[i][r] & S.oB[i]) ? (1u << i) : 0u;
        }
#endif
        if (rel) {
            ItemStream<TI, TO> it;
            it.rel = rel;
            // one item at a time (a second register set for the next item measured slower:
            // 5.26 vs 5.13 ms on C2, the registers it takes cost more than the overlap it buys)
            TO aX, bX0, bX1, bX2;
            uint32_t mX;
            const TI *vX;
            while (it.fetch(P, S, r, aX, bX0, bX1, bX2, mX, vX)) accumulate_row(aX, bX0, bX1, bX2, mX, vX, acc);
        }
        __syncwarp();
    }
    // compaction through mask_C[r]; every slot the tile touched is in mask_C[r] and is reset to
    // zero for the next tile (the accumulator is cleared once per warp at kernel start)
    if (mCr) {
        uint8_t *px = P.ixC + M.ob;
        TO *pv = static_cast<TO *>(P.vC) + M.ob;
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

// dense tile (nnz >= t_nnz): the whole warp, both tiles of a pair staged densely in shared
// memory, lane (r = lane/2, h = lane%2) owns C(r, 8h..8h+7) in registers; compaction through
// mask_C at the end.  Structurally absent A entries are skipped; absent B entries
// are staged as 0 so a finite a adds an exact +-0 (value unchanged); a non-finite a falls back to
// mask-predicated FMAs so Inf*0 never appears.
template <typename TI, typename TO>
__device__ __forceinline__ void s3_dense(const StepParams &P, int64_t t, unsigned char *wr, int lane) {
    constexpr int AP = 17;  // padded row pitch of the staged A tile (conflict-free column reads)
    const TI *vA = static_cast<const TI *>(P.vA), *vB = static_cast<const TI *>(P.vB);
    TO *Ad = reinterpret_cast<TO *>(wr);
    TO *Bd = reinterpret_cast<TO *>(wr + 2176);  // after 16 x 17 doubles: 16-byte aligned
    const int r = lane >> 1, h = lane & 1;
    TO acc[8];
#pragma unroll
    for (int j = 0; j < 8; j++) acc[j] = (TO)0;
    const uint64_t *pp = P.pairs + P.pairBeg[t];
    const uint32_t np = P.pairCnt[t];
    // A is read only at its structural positions (c in mask_A[r]), so it is never cleared; B is
    // cleared per pair (16-byte stores) and its nonzeros scattered over it
    for (uint32_t p = 0; p < np; p++) {
        const uint64_t pr = pp[p];
        const int64_t pA = (int64_t)(pr >> 32), pB = (int64_t)(uint32_t)pr;
#pragma unroll
        for (int e = lane; e < TILE * TILE * (int)sizeof(TO) / 16; e += 32)
            reinterpret_cast<uint4 *>(Bd)[e] = make_uint4(0u, 0u, 0u, 0u);
        __syncwarp();
        bool nf = false;
        for (int64_t e = P.tnzA[pA] + lane; e < P.tnzA[pA + 1]; e += 32) {
            const uint32_t ix = P.ixA[e];
            const TO v = vcvt<TO>(vA[e]);
            nf |= !isfinite(v);
            Ad[(ix >> 4) * AP + (ix & 15)] = v;
        }
        for (int64_t e = P.tnzB[pB] + lane; e < P.tnzB[pB + 1]; e += 32) {
            const uint32_t ix = P.ixB[e];
            Bd[(ix >> 4) * TILE + (ix & 15)] = vcvt<TO>(vB[e]);
        }
        const uint32_t mA = P.mA[pA * TILE + r];
        const bool anynf = __any_sync(FULL, nf);
        __syncwarp();
        if (!anynf) {
#pragma unroll
            for (int c = 0; c < TILE; c++) {
                if ((mA >> c) & 1u) {
                    const TO a = Ad[r * AP + c];
                    TO b[8];
                    lds8(Bd + c * TILE + 8 * h, b);
#pragma unroll
                    for (int jj = 0; jj < 8; jj++) acc[jj] = vfma(a, b[jj], acc[jj]);
                }
            }
        } else {
            const uint16_t *mbt = P.mB + pB * TILE;
            for (int c = 0; c < TILE; c++) {
                if ((mA >> c) & 1u) {
                    const TO a = Ad[r * AP + c];
                    const uint32_t mb = (uint32_t)mbt[c] >> (8 * h);
#pragma unroll
                    for (int jj = 0; jj < 8; jj++)
                        if ((mb >> jj) & 1u) acc[jj] = vfma(a, Bd[c * TILE + 8 * h + jj], acc[jj]);
                }
            }
        }
        __syncwarp();
    }
    const uint32_t mC = P.mC[t * TILE + r];
    const int64_t ob = P.tnzC[t] + P.rpC[t * TILE + r];
#pragma unroll
    for (int jj = 0; jj < 8; jj++) {
        const int j = 8 * h + jj;
        if ((mC >> j) & 1u) {
            const int q = __popc(mC & ((1u << j) - 1u));
            P.ixC[ob + q] = (uint8_t)((r << 4) | j);
            static_cast<TO *>(P.vC)[ob + q] = acc[jj];
        }
    }
    __syncwarp();
}

// medium tiles: warps take groups of 32 consecutive C tiles; the group's medium tiles go two at a
// time, a half warp each.  Register- and shared-memory-lean (no dense code): 7 CTAs per SM.
template <typename TI, typename TO>
#ifndef TSG_MED_MINB
#define TSG_MED_MINB 7
#endif
__global__ void __launch_bounds__(T3, TSG_MED_MINB) k_s3(StepParams P) { TSG_GRID_WAIT();
    __shared__ __align__(16) unsigned char wreg[T3 / 32][WREG];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, r = lane & 15, half = lane >> 4;
    unsigned char *wr = wreg[w];
    TO *acc = reinterpret_cast<TO *>(wr) + half * (TILE * TILE) + r;
#pragma unroll
    for (int j = 0; j < TILE; j++) acc[j * 16] = (TO)0;
    const int64_t ngroups = (P.ntC + 31) / 32;
    WorkQueue wq(&P.cnt->q[3][0], ngroups, P.qchunk[3], lane, T3 / 32);
    for (int64_t g; wq.next(g, lane);) {
        unsigned mm = P.medL[g] | P.medH[g];  // the group's medium tiles (step 2 classified them)
        if (!mm) continue;                    // warp-uniform
        if (lane == 0 && mm) atomicAdd(&P.cnt->n3medium, (u64c)__popc(mm));
        auto pop2 = [&]() {  // next two medium tiles of the group (one per half warp)
            const int f0 = __ffs(mm) - 1;
            mm &= mm - 1;
            const int f1 = mm ? __ffs(mm) - 1 : -1;
            if (mm) mm &= mm - 1;
            return half ? f1 : f0;
        };
        if (mm) {
            MedMeta cur, nxt;
            cur.load(P, pop2(), g, r);
            for (;;) {
                const bool more = mm != 0;  // warp-uniform
                if (more) nxt.load(P, pop2(), g, r);
                s3_medium<TI, TO>(P, cur, acc, *reinterpret_cast<MedStage *>(wr + WACC + half * sizeof(MedStage)), r);
                if (!more) break;
                cur = nxt;
            }
        }
    }
}

// dense tiles (nnz >= t_nnz): the whole warp each; launched only when step 2 counted any
#ifndef TSG_DENSE_MINB
#define TSG_DENSE_MINB 4
#endif
constexpr int DREG = 2176 + 2048;  // per-warp staging of the dense path: A 16 x 17 and B 16 x 16 (fp64)
template <typename TI, typename TO>
__global__ void __launch_bounds__(T3, TSG_DENSE_MINB) k_s3_dense(StepParams P, int split) { TSG_GRID_WAIT();
    __shared__ __align__(16) unsigned char wreg[T3 / 32][DREG];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    unsigned char *wr = wreg[w];
    // `split` warps share a group of 32 C tiles, warp `part` taking every split-th dense tile of
    // it: dense tiles cluster (FEM strips), and a group's dense tiles done by one warp one after
    // the other would make the kernel a chain of serial per-pair latencies
    const int64_t nunits = (P.ntC + 31) / 32 * split;
    WorkQueue wq(&P.cnt->q[4][0], nunits, P.qchunk[4], lane, T3 / 32);
    for (int64_t u; wq.next(u, lane);) {
        const int64_t g = u / split;
        const int part = (int)(u - g * split);
        unsigned dm = P.denL[g] | P.denH[g];  // the group's dense tiles (step 2 classified them)
        if (!dm) continue;                    // warp-uniform
        if (lane == 0 && part == 0 && dm) atomicAdd(&P.cnt->n3dense, (u64c)__popc(dm));
        unsigned dd = dm;
        for (int k = 0; dd; k = k + 1 == split ? 0 : k + 1) {
            const int f = __ffs(dd) - 1;
            dd &= dd - 1;
            if (k != part) continue;
            s3_dense<TI, TO>(P, g * 32 + f, wr, lane);
        }
    }
}

// Launch shape of a step-2/3 kernel over `units` work units (groups of 32 C tiles), `wpc` warps
// per CTA.  Many units per warp: a persistent grid (the CTAs resident at once: SM count x
// occupancy) with the work queue, so the warps running at any moment work on neighbouring C tiles
// (the A and B tiles their pairs read stay in L2) and the load balances; `chunk` units per
// request grows with the units per warp (C2: 1, R-MAT: 4-8) so the counter stays cold.  Few
// units per warp (C3), and dense tiles: static grid-stride over up to 32 CTAs per SM (measured
// faster there).
struct Shape {
    unsigned grid;
    int chunk;
};
template <typename K>
Shape step_shape(K kernel, int threads, int64_t units, int qoverride, int64_t min_per_warp = 4) {
    static std::mutex mu;
    static std::map<std::pair<const void *, int>, int> cache;  // (kernel, device) -> resident CTAs per GPU
    const int wpc = threads / 32;
    int dev = 0;
    cudaGetDevice(&dev);
    int resident;
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = cache.find({(const void *)kernel, dev});
        if (it == cache.end()) {
            int nsm = 148, occ = 1;
            cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, threads, 0);
            it = cache.emplace(std::make_pair((const void *)kernel, dev), nsm * std::max(occ, 1)).first;
        }
        resident = it->second;
    }
    units = std::max<int64_t>(units, 1);
    const int64_t per_warp = units / ((int64_t)resident * wpc);
    int64_t chunk = per_warp >= min_per_warp ? std::max<int64_t>(1, std::min<int64_t>(8, per_warp / 256)) : 0;
    if (qoverride >= 0) chunk = qoverride;  // TSG_QUEUE_CHUNK_SHIFT (tests of the distribution)
    if (chunk <= 0) return {(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(units, wpc), 148LL * 32)), 0};
    return {(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(units, wpc), resident)), (int)chunk};
}

}  // namespace

void launch_step2(const StepParams &P, cudaStream_t s) {
    if (P.ntC <= 0) return;
    const int64_t groups = (P.ntC + 31) / 32;
    StepParams Q = P;
    const Shape sl = step_shape(k_s2_light, T2L, groups, P.qoverride), sh = step_shape(k_s2, T2, groups, P.qoverride);
    Q.qchunk[0] = sl.chunk;
    Q.qchunk[1] = sh.chunk;
    TSG_LAUNCH(k_s2_light, sl.grid, T2L, 0, s, Q);
    TSG_LAUNCH(k_s2, sh.grid, T2, 0, s, Q);
}

template <typename TI, typename TO>
static void launch_step3_t(const StepParams &P, int64_t n_dense, cudaStream_t s) {
    const int64_t groups = (P.ntC + 31) / 32;
    StepParams Q = P;
    if (P.small_max > 0) {
        if (P.recA) {
            const Shape sp = step_shape(k_s3_small<TI, TO, 2>, TS, groups, P.qoverride);
            Q.qchunk[2] = sp.chunk;
            TSG_LAUNCH((k_s3_small<TI, TO, 2>), sp.grid, TS, 0, s, Q);
        } else if (P.small_stage) {
            const Shape sp = step_shape(k_s3_small<TI, TO, 1>, TS, groups, P.qoverride);
            Q.qchunk[2] = sp.chunk;
            TSG_LAUNCH((k_s3_small<TI, TO, 1>), sp.grid, TS, 0, s, Q);
        } else {
            const Shape sp = step_shape(k_s3_small<TI, TO, 0>, TS, groups, P.qoverride);
            Q.qchunk[2] = sp.chunk;
            TSG_LAUNCH((k_s3_small<TI, TO, 0>), sp.grid, TS, 0, s, Q);
        }
    }
    {
        const Shape sp = step_shape(k_s3<TI, TO>, T3, groups, P.qoverride);
        Q.qchunk[3] = sp.chunk;
        TSG_LAUNCH((k_s3<TI, TO>), sp.grid, T3, 0, s, Q);
    }
    if (n_dense > 0) {
        // dense tiles per group of 32: spread a group over up to 4 warps when dense tiles are common
        // (measured on C3: 2 / 4 / 8 / 16 / 32 warps -> 0.743 / 0.716 / 0.734 / 0.780 / 0.839 ms)
        int split = (int)std::max<int64_t>(1, std::min<int64_t>(4, 32 * n_dense / (groups * 4)));
        // (dense tiles: static distribution, measured faster on C3)
        const Shape sp = step_shape(k_s3_dense<TI, TO>, T3, groups * split, P.qoverride, INT64_MAX);
        Q.qchunk[4] = sp.chunk;
        TSG_LAUNCH((k_s3_dense<TI, TO>), sp.grid, T3, 0, s, Q, split);
    }
}

void launch_step3(const StepParams &P, int64_t n_dense, cudaStream_t s) {
    if (P.ntC <= 0) return;
    switch (P.dtype_in) {
        case TSG_F64: launch_step3_t<double, double>(P, n_dense, s); break;
        case TSG_F32: launch_step3_t<float, float>(P, n_dense, s); break;
        default: launch_step3_t<__half, float>(P, n_dense, s);
    }
}

}  // namespace tsg
