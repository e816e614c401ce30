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

#include "tsg_kernels.cuh"

namespace tsg {
namespace {

constexpr unsigned FULL = 0xffffffffu;
constexpr int T2 = 256;    // step-2 CTA
constexpr int T3 = 128;    // step-3 CTA (4 warps; 5.5 KB of shared memory per warp)
constexpr int BATCH = 16;  // step 2: pairs staged per half warp at a time
constexpr int BATCH3 = 16; // step 3: pairs staged per half warp at a time (also the small path's 16 slots)

// ==========================================================================================
// step 2
// ==========================================================================================
// light tile (<= LIGHT_WORK items): one thread, item driven; row masks in 8 thread-private words
__device__ __forceinline__ void s2_light(const StepParams &P, int64_t t, uint32_t *w, int stride) {
#pragma unroll
    for (int q = 0; q < 8; q++) w[q * stride] = 0;
    const uint64_t *pp = P.pairs + P.pairBeg[t];
    const uint32_t np = P.pairCnt[t];
    for (uint32_t p = 0; p < np; p++) {
        const uint64_t pr = pp[p];
        const int64_t pA = (int64_t)(pr >> 32), pB = (int64_t)(uint32_t)pr;
        uint32_t x = (uint32_t)P.colOccA[pA] & P.rowOccB[pB];
        const uint16_t *mb = P.mB + pB * TILE;
        const uint16_t *at = P.mTA + pA * TILE;
        while (x) {
            const int c = __ffs(x) - 1;
            x &= x - 1;
            const uint32_t bits = mb[c];
            uint32_t rows = at[c];
            while (rows) {
                const int r = __ffs(rows) - 1;
                rows &= rows - 1;
                w[(r >> 1) * stride] |= bits << (16 * (r & 1));
            }
        }
    }
    uint32_t m[8];
    uint32_t rp[4] = {0, 0, 0, 0};
    int total = 0;
#pragma unroll
    for (int q = 0; q < 8; q++) m[q] = w[q * stride];
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
}

__device__ __forceinline__ void cp16s(void *dst_smem, const void *src) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst_smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(d), "l"(src) : "memory");
}

__global__ void __launch_bounds__(T2) k_s2(StepParams P) {
    __shared__ uint32_t wsm[8 * T2];
    __shared__ __align__(16) uint16_t sMA[T2 / 16][BATCH][TILE], sMB[T2 / 16][BATCH][TILE];
    __shared__ uint16_t sOB[T2 / 16][BATCH];
    const int lane = threadIdx.x & 31, r = lane & 15, half = lane >> 4, hw = threadIdx.x >> 4;
    const int64_t ngroups = (P.ntC + 31) / 32;
    const int64_t gstride = (int64_t)gridDim.x * (T2 / 32);
    for (int64_t g = (int64_t)blockIdx.x * (T2 / 32) + (threadIdx.x >> 5); g < ngroups; g += gstride) {
        const int64_t t = g * 32 + lane;
        const bool v = t < P.ntC;
        const bool light = v && P.work[t] <= (uint32_t)LIGHT_WORK;
        if (light) s2_light(P, t, wsm + threadIdx.x, T2);
        unsigned hm = __ballot_sync(FULL, v && !light);
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
                    cp16s(&sMA[hw][r][0], P.mA + pA * TILE);
                    cp16s(&sMA[hw][r][8], P.mA + pA * TILE + 8);
                    cp16s(&sMB[hw][r][0], P.mB + pB * TILE);
                    cp16s(&sMB[hw][r][8], P.mB + pB * TILE + 8);
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
        }
        const unsigned lm = __ballot_sync(FULL, light), vm = __ballot_sync(FULL, v);
        if (lane == 0) {
            atomicAdd(&P.cnt->n2light, (u64c)__popc(lm));
            atomicAdd(&P.cnt->n2heavy, (u64c)(__popc(vm) - __popc(lm)));
        }
    }
}

// ==========================================================================================
// step 3
// ==========================================================================================
constexpr int WREG = 4224;  // bytes of per-warp shared scratch (small: 4 KB acc + 1.5 KB masks;
                            // medium: 4 KB of row accumulators; dense: 4.2 KB of staged tiles)

struct MedStage {  // per half warp: staged metadata and tile masks / row offsets of up to 16 pairs
    uint16_t mA[BATCH3][TILE], mB[BATCH3][TILE];  // cp.async'd masks of A_IK and B_KJ
    uint16_t mT[BATCH3][TILE];                   // transposed A mask (small-tile path)
    uint8_t rA[BATCH3][TILE], rB[BATCH3][TILE];   // and their row offsets
    int64_t zA[BATCH3], zB[BATCH3];
    uint16_t oB[BATCH3];
};

__device__ __forceinline__ void cp16(void *dst_smem, const void *src) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst_smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(d), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_wait_all() {
    asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;\n" ::: "memory");
}

// small tile (nnz <= 16): one thread, item driven.  Slot of C(r,j) is row_ptr_C[r] +
// popc(mask_C[r] & ((1<<j)-1)) (the mask-addressed accumulator); slots, masks and
// row offsets are thread-private (lane-strided words of the warp's scratch).
__device__ __forceinline__ void s3_small(const StepParams &P, int64_t t, unsigned char *wr, int lane, MedStage &S) {
    double *acc = reinterpret_cast<double *>(wr) + lane;                        // acc[q*32]
    uint32_t *ms = reinterpret_cast<uint32_t *>(wr + SMALL_NNZ * 32 * 8) + lane;  // ms[k*32], k < 8
    uint32_t *rs = ms + 8 * 32;                                                 // rs[k*32], k < 4
    const int sl = lane & 15;  // this thread's staging slot in its half warp's MedStage
    const int64_t z0 = P.tnzC[t];
    const int nz = (int)(P.tnzC[t + 1] - z0);
    {
        const uint4 *pm = reinterpret_cast<const uint4 *>(P.mC + t * TILE);
        const uint4 a = pm[0], b = pm[1];
        ms[0] = a.x; ms[32] = a.y; ms[64] = a.z; ms[96] = a.w;
        ms[128] = b.x; ms[160] = b.y; ms[192] = b.z; ms[224] = b.w;
        const uint4 rp = *reinterpret_cast<const uint4 *>(P.rpC + t * TILE);
        rs[0] = rp.x; rs[32] = rp.y; rs[64] = rp.z; rs[96] = rp.w;
    }
    for (int q = 0; q < nz; q++) acc[q * 32] = 0.0;
    const uint64_t *pp = P.pairs + P.pairBeg[t];
    const uint32_t np = P.pairCnt[t];
    for (uint32_t p = 0; p < np; p++) {
        const uint64_t pr = pp[p];
        const int64_t pA = (int64_t)(pr >> 32), pB = (int64_t)(uint32_t)pr;
        // the pair's masks, row offsets and transposed A mask: one round of cp.async instead of a
        // chain of dependent reads
        cp16(&S.mA[sl][0], P.mA + pA * TILE);
        cp16(&S.mA[sl][8], P.mA + pA * TILE + 8);
        cp16(&S.mB[sl][0], P.mB + pB * TILE);
        cp16(&S.mB[sl][8], P.mB + pB * TILE + 8);
        cp16(&S.rA[sl][0], P.rpA + pA * TILE);
        cp16(&S.rB[sl][0], P.rpB + pB * TILE);
        cp16(&S.mT[sl][0], P.mTA + pA * TILE);
        cp16(&S.mT[sl][8], P.mTA + pA * TILE + 8);
        uint32_t x = (uint32_t)P.colOccA[pA] & P.rowOccB[pB];
        const double *vbt = P.vB + P.tnzB[pB];
        const double *vat = P.vA + P.tnzA[pA];
        cp_wait_all();
        // columns c ascending, rows of A's column c: every slot (r, j) sees ascending c
        while (x) {
            const int c = __ffs(x) - 1;
            x &= x - 1;
            const uint32_t mbc = S.mB[sl][c];
            const double *vb = vbt + S.rB[sl][c];
            uint32_t rows = S.mT[sl][c];
            while (rows) {
                const int r = __ffs(rows) - 1;
                rows &= rows - 1;
                const double a = vat[S.rA[sl][r] + __popc((uint32_t)S.mA[sl][r] & ((1u << c) - 1u))];
                const uint32_t mcr = (ms[(r >> 1) * 32] >> (16 * (r & 1))) & 0xffffu;
                const int base = (rs[(r >> 2) * 32] >> (8 * (r & 3))) & 0xff;
                uint32_t mb = mbc;
                int ib = 0;
                while (mb) {
                    const int j = __ffs(mb) - 1;
                    mb &= mb - 1;
                    const int q = base + __popc(mcr & ((1u << j) - 1u));
                    acc[q * 32] = fma(a, vb[ib++], acc[q * 32]);
                }
            }
        }
    }
    int q = 0;
    for (int r = 0; r < TILE; r++) {
        uint32_t m = (ms[(r >> 1) * 32] >> (16 * (r & 1))) & 0xffffu;
        while (m) {
            const int j = __ffs(m) - 1;
            m &= m - 1;
            P.ixC[z0 + q] = (uint8_t)((r << 4) | j);
            P.vC[z0 + q] = acc[q * 32];
            q++;
        }
    }
}

// one column c of A's row r in flight: a = A(r,c), B's row c (mask, first 4 values, the rest)
struct BRow {
    double a, b0, b1, b2, b3;
    uint32_t m;
    const double *vb;
};
__device__ __forceinline__ BRow load_brow(const MedStage &S, int i, int c, uint32_t mAr, const double *va,
                                          const double *vbt) {
    BRow x;
    x.m = S.mB[i][c];
    x.vb = vbt + S.rB[i][c];
    x.a = va[__popc(mAr & ((1u << c) - 1u))];
    const int n = __popc(x.m);
    x.b0 = x.vb[0];  // every row c here is non-empty (filtered by rowOcc(B))
    x.b1 = n > 1 ? x.vb[1] : 0.0;
    x.b2 = n > 2 ? x.vb[2] : 0.0;
    x.b3 = n > 3 ? x.vb[3] : 0.0;
    return x;
}
// acc[16 j] += a * B(c, j) over B's row c in ascending j (row accumulator: lane-strided slots).
// The first four slots are distinct, so their loads, FMAs and stores are issued as a group
// (independent shared-memory round trips instead of a chain of four).
__device__ __forceinline__ void accumulate_brow(const BRow &x, double *acc) {
    uint32_t m = x.m;
    const int j0 = __ffs(m) - 1;
    m &= m - 1;
    const int j1 = m ? __ffs(m) - 1 : j0;
    m &= m - 1;
    const int j2 = m ? __ffs(m) - 1 : j0;
    m &= m - 1;
    const int j3 = m ? __ffs(m) - 1 : j0;
    m &= m - 1;
    const int n = __popc(x.m);
    double c0 = acc[j0 * 16], c1 = 0.0, c2 = 0.0, c3 = 0.0;
    if (n > 1) c1 = acc[j1 * 16];
    if (n > 2) c2 = acc[j2 * 16];
    if (n > 3) c3 = acc[j3 * 16];
    acc[j0 * 16] = fma(x.a, x.b0, c0);
    if (n > 1) acc[j1 * 16] = fma(x.a, x.b1, c1);
    if (n > 2) acc[j2 * 16] = fma(x.a, x.b2, c2);
    if (n > 3) acc[j3 * 16] = fma(x.a, x.b3, c3);
    const double *vb = x.vb + 4;
    while (m) {
        const int j = __ffs(m) - 1;
        m &= m - 1;
        acc[j * 16] = fma(x.a, *vb++, acc[j * 16]);
    }
}

// a lane's position in its flat (pair, c) item sequence of a batch
struct ItemCursor {
    uint32_t rel = 0, ma = 0, mAr = 0;
    int i = 0;
    const double *va = nullptr, *vbt = nullptr;
};
__device__ __forceinline__ bool next_item(const StepParams &P, const MedStage &S, int r, ItemCursor &it, BRow &out) {
    if (!it.ma) {
        if (!it.rel) return false;
        it.i = __ffs(it.rel) - 1;
        it.rel &= it.rel - 1;
        it.mAr = S.mA[it.i][r];
        it.ma = it.mAr & S.oB[it.i];
        it.va = P.vA + S.zA[it.i] + S.rA[it.i][r];
        it.vbt = P.vB + S.zB[it.i];
    }
    const int c = __ffs(it.ma) - 1;
    it.ma &= it.ma - 1;
    out = load_brow(S, it.i, c, it.mAr, it.va, it.vbt);
    return true;
}

// medium tile: a half warp, lane r owns C row r; dense-in-j 16-slot row accumulator in shared
// memory (conflict free), compacted through mask_C[r] at the end.  Pairs go in batches of 16:
// lane i stages pair i's A and B masks and row offsets (6 x 16-byte cp.async, all lanes and
// pairs in flight at once), so a lane's walk over its row touches global memory only for the
// values.  All 32 lanes must call.
__device__ __forceinline__ void s3_medium(const StepParams &P, bool hv, int64_t t, double *acc, MedStage &S,
                                          int r) {
    uint32_t np = 0, mCr = 0;
    const uint64_t *pp = P.pairs;
    if (hv) {
        pp += P.pairBeg[t];
        np = P.pairCnt[t];
        mCr = P.mC[t * TILE + r];
        uint32_t m = mCr;
        while (m) {
            const int j = __ffs(m) - 1;
            m &= m - 1;
            acc[j * 16] = 0.0;
        }
    }
    const uint32_t nbat = (np + BATCH3 - 1) / BATCH3;
    const uint32_t nbw = max(nbat, __shfl_xor_sync(FULL, nbat, 16));
    for (uint32_t bt = 0; bt < nbw; bt++) {
        const uint32_t q = bt * BATCH3 + r;
        if (r < BATCH3 && q < np) {
            const uint64_t pr = pp[q];
            const int64_t pA = (int64_t)(pr >> 32), pB = (int64_t)(uint32_t)pr;
            cp16(&S.mA[r][0], P.mA + pA * TILE);
            cp16(&S.mA[r][8], P.mA + pA * TILE + 8);
            cp16(&S.mB[r][0], P.mB + pB * TILE);
            cp16(&S.mB[r][8], P.mB + pB * TILE + 8);
            cp16(&S.rA[r][0], P.rpA + pA * TILE);
            cp16(&S.rB[r][0], P.rpB + pB * TILE);
            S.zA[r] = P.tnzA[pA];
            S.zB[r] = P.tnzB[pB];
            S.oB[r] = P.rowOccB[pB];
        }
        cp_wait_all();
        __syncwarp();
        const uint32_t nb = np > bt * BATCH3 ? min((uint32_t)BATCH3, np - bt * BATCH3) : 0u;
        if (mCr) {
            // the batch's pairs that touch row r, then one flat loop over this lane's (pair, c)
            // items in order (pairs ascending, c ascending): lanes whose rows see different pairs
            // (e.g. the 1-nonzero corner tiles of stencils touch one row) stay in step, and the
            // next item's loads are in flight while the current one accumulates
            uint32_t rel = 0;
            for (uint32_t i = 0; i < nb; i++) rel |= (S.mA[i][r] & S.oB[i]) ? (1u << i) : 0u;
            ItemCursor it;
            it.rel = rel;
            BRow cur;
            bool have = next_item(P, S, r, it, cur);
            while (have) {
                BRow nxt;
                const bool hn = next_item(P, S, r, it, nxt);
                accumulate_brow(cur, acc);
                cur = nxt;
                have = hn;
            }
        }
        __syncwarp();
    }
    if (hv && mCr) {
        const int64_t ob = P.tnzC[t] + P.rpC[t * TILE + r];
        uint32_t m = mCr;
        int qq = 0;
        while (m) {
            const int j = __ffs(m) - 1;
            m &= m - 1;
            P.ixC[ob + qq] = (uint8_t)((r << 4) | j);
            P.vC[ob + qq] = acc[j * 16];
            qq++;
        }
    }
    __syncwarp();
}

// dense tile (nnz >= t_nnz): the whole warp, both tiles of a pair staged densely in shared
// memory, lane (r = lane/2, h = lane%2) owns C(r, 8h..8h+7) in registers; compaction through
// mask_C at the end.  Structurally absent A entries are skipped; absent B entries
// are staged as 0 so a finite a adds an exact +-0 (value unchanged); a non-finite a falls back to
// mask-predicated FMAs so Inf*0 never appears.
__device__ __forceinline__ void s3_dense(const StepParams &P, int64_t t, unsigned char *wr, int lane) {
    constexpr int AP = 17;  // padded row pitch of the staged A tile (conflict-free column reads)
    double *Ad = reinterpret_cast<double *>(wr);
    double *Bd = Ad + TILE * AP;  // byte offset 2176: 16-byte aligned
    const int r = lane >> 1, h = lane & 1;
    double acc[8];
#pragma unroll
    for (int j = 0; j < 8; j++) acc[j] = 0.0;
    const uint64_t *pp = P.pairs + P.pairBeg[t];
    const uint32_t np = P.pairCnt[t];
    // A is read only at its structural positions (c in mask_A[r]), so it is never cleared; B is
    // cleared per pair (four 16-byte stores per lane) and its nonzeros scattered over it
    for (uint32_t p = 0; p < np; p++) {
        const uint64_t pr = pp[p];
        const int64_t pA = (int64_t)(pr >> 32), pB = (int64_t)(uint32_t)pr;
#pragma unroll
        for (int e = lane; e < TILE * TILE / 2; e += 32) reinterpret_cast<double2 *>(Bd)[e] = make_double2(0.0, 0.0);
        __syncwarp();
        bool nf = false;
        for (int64_t e = P.tnzA[pA] + lane; e < P.tnzA[pA + 1]; e += 32) {
            const uint32_t ix = P.ixA[e];
            const double v = P.vA[e];
            nf |= !isfinite(v);
            Ad[(ix >> 4) * AP + (ix & 15)] = v;
        }
        for (int64_t e = P.tnzB[pB] + lane; e < P.tnzB[pB + 1]; e += 32) {
            const uint32_t ix = P.ixB[e];
            Bd[(ix >> 4) * TILE + (ix & 15)] = P.vB[e];
        }
        const uint32_t mA = P.mA[pA * TILE + r];
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
            const uint16_t *mbt = P.mB + pB * TILE;
            for (int c = 0; c < TILE; c++) {
                if ((mA >> c) & 1u) {
                    const double a = Ad[r * AP + c];
                    const uint32_t mb = (uint32_t)mbt[c] >> (8 * h);
#pragma unroll
                    for (int jj = 0; jj < 8; jj++)
                        if ((mb >> jj) & 1u) acc[jj] = fma(a, Bd[c * TILE + 8 * h + jj], acc[jj]);
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
            P.vC[ob + q] = acc[jj];
        }
    }
    __syncwarp();
}

__global__ void __launch_bounds__(T3, 6) k_s3(StepParams P) {
    __shared__ __align__(16) unsigned char wreg[T3 / 32][WREG];
    __shared__ MedStage med[T3 / 16];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, r = lane & 15, half = lane >> 4;
    unsigned char *wr = wreg[w];
    const int64_t ngroups = (P.ntC + 31) / 32;
    const int64_t gstride = (int64_t)gridDim.x * (T3 / 32);
    for (int64_t g = (int64_t)blockIdx.x * (T3 / 32) + w; g < ngroups; g += gstride) {
        const int64_t t = g * 32 + lane;
        const bool v = t < P.ntC && !(P.skip && P.skip[t]);
        const int nz = v ? (int)(P.tnzC[t + 1] - P.tnzC[t]) : 0;
        const bool dense = v && nz >= P.dense_threshold;
        const bool small = v && !dense && nz <= SMALL_NNZ;
        const unsigned sm = __ballot_sync(FULL, small);
        const unsigned dm = __ballot_sync(FULL, dense);
        unsigned mm = __ballot_sync(FULL, v) & ~sm & ~dm;
        if (small) s3_small(P, t, wr, lane, med[threadIdx.x >> 4]);
        __syncwarp();
        // medium tiles: two at a time, a half warp each
        double *acc = reinterpret_cast<double *>(wr) + half * (TILE * TILE) + r;
        while (mm) {
            const int f0 = __ffs(mm) - 1;
            mm &= mm - 1;
            const int f1 = mm ? __ffs(mm) - 1 : -1;
            if (mm) mm &= mm - 1;
            const int mine = half ? f1 : f0;
            s3_medium(P, mine >= 0, g * 32 + (mine >= 0 ? mine : 0), acc, med[threadIdx.x >> 4], r);
        }
        // dense tiles: the whole warp each
        unsigned dd = dm;
        while (dd) {
            const int f = __ffs(dd) - 1;
            dd &= dd - 1;
            s3_dense(P, g * 32 + f, wr, lane);
        }
        const unsigned vm = __ballot_sync(FULL, v);
        if (lane == 0) {
            atomicAdd(&P.cnt->n3small, (u64c)__popc(sm));
            atomicAdd(&P.cnt->n3dense, (u64c)__popc(dm));
            atomicAdd(&P.cnt->n3medium, (u64c)(__popc(vm) - __popc(sm) - __popc(dm)));
        }
    }
}

unsigned grid_groups(int64_t ntC, int warps_per_cta) {
    const int64_t groups = (ntC + 31) / 32;
    const int64_t g = std::min<int64_t>(ceil_div(std::max<int64_t>(groups, 1), warps_per_cta), 148LL * 32);
    return (unsigned)std::max<int64_t>(g, 1);
}

}  // namespace

void launch_step2(const StepParams &P, cudaStream_t s) {
    if (P.ntC <= 0) return;
    TSG_LAUNCH(k_s2, grid_groups(P.ntC, T2 / 32), T2, 0, s, P);
}

void launch_step3(const StepParams &P, cudaStream_t s) {
    if (P.ntC <= 0) return;
    TSG_LAUNCH(k_s3, grid_groups(P.ntC, T3 / 32), T3, 0, s, P);
}

}  // namespace tsg
