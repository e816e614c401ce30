// tsg_step3row.cu -- SURVEY §8(a) row a4, step 3 (numeric phase) of Section 3.3 for whole C tile
// rows: Alg 3 with the adaptive accumulator (t_nnz P:1500-1502).
//
// The per-tile kernel of tsg_step23.cu walks a C tile's pairs with a chain of dependent L2 reads
// (pair -> tile -> row -> values) per product.  Here one CTA owns a whole C tile row I and first
// stages, with TMA bulk copies (cp.async.bulk, one mbarrier), everything the row touches that is
// contiguous in memory:
//   * C row I's masks, row offsets, nnz offsets, pair ranges (output of steps 1-2),
//   * A tile row I (masks, row offsets, nnz offsets, values) and the row's pair list,
//   * for every "heavy" A tile A_IK (> 2 distinct columns) the whole B tile row K (masks, row
//     offsets, nnz offsets, values), as far as the shared-memory budget allows.
// A tile row K of B is contiguous in the tile format (Section 3.2), so staging it is four bulk
// copies.  For a "light" A tile (<= 2 columns, e.g. the 1-nnz corner tiles of stencils) the warps
// gather only rows c in colOcc(A_IK) of every B_KJ (mask, values) into a shared pool, all light
// tiles of the row at once, while the bulk copies are in flight.
// Then thread u owns the C row segment (tile t, row r): it walks tile t's pairs in ascending K,
// A_IK's row r in ascending c, and B_KJ's row c, accumulating into shared memory:
//   sparse tile (nnz < t_nnz): slot rowPtr_C[r] + popc(mask_C[r] & ((1<<j)-1)) of the row's
//                              compact image, which is C's output layout;
//   dense tile (nnz >= t_nnz): a 16x16 block, slot 16r + j, compacted through mask_C at the end
//                              (P:1862-1870).
// Each slot has one owner and receives its products in ascending k = 16K + c: no atomics, results
// bitwise equal to the per-tile kernel and to the oracle's fma mode (readings A8/A16).  The
// finished row image is written to C with coalesced stores.
//
// Rows that exceed the caps (C tiles, A tiles, pairs, accumulator size; typically the hub rows of
// power-law graphs) are left to the per-tile kernel through the per-tile `skip` flags.
#include "tsg_kernels.cuh"

namespace tsg {
namespace {

constexpr unsigned FULL = 0xffffffffu;
constexpr uint32_t DENSE_FLAG = 0x80000000u;

// ------------------------------------------------------------------------------------------
// mbarrier + bulk-copy primitives (PTX; sm_90+).  One mbarrier per CTA, one phase per row.
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t *bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(count) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, unsigned bytes) {
    asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, unsigned parity) {
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory"); }

// copy the 16-byte aligned superset of [src, src + bytes) to dst (16-byte aligned shared memory);
// the first source byte lands at dst + ((uintptr_t)src & 15).  Issuing thread only.  The
// superset never leaves the 16-byte blocks of valid elements, hence never the allocation's pages.
__device__ __forceinline__ void bulk_stage(void *dst, const void *src, size_t bytes, uint64_t *bar) {
    if (bytes == 0) return;
    const uintptr_t s = (uintptr_t)src, s0 = s & ~(uintptr_t)15;
    const unsigned n = (unsigned)(((s - s0) + bytes + 15) & ~(size_t)15);
    mbar_expect_tx(bar, n);
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(
                     smem_u32(dst)),
                 "l"(s0), "r"(n), "r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ unsigned staged_bytes(const void *src, size_t bytes) {
    const uintptr_t s = (uintptr_t)src;
    return bytes ? (unsigned)(((s & 15) + bytes + 15) & ~(size_t)15) : 0u;
}
template <typename T>
__device__ __forceinline__ const T *staged_ptr(const unsigned char *dst, const void *src) {
    return reinterpret_cast<const T *>(dst + ((uintptr_t)src & 15));
}

__device__ __forceinline__ int64_t al16z(int64_t x) { return (x + 15) & ~(int64_t)15; }

// ------------------------------------------------------------------------------------------
// row classification: one warp per tile row
// ------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_s3_class(RowParams P) {
    const int lane = threadIdx.x & 31;
    const int64_t I = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (I >= P.tm) return;
    const int64_t t0 = P.tpC[I], t1 = P.tpC[I + 1], nt = t1 - t0;
    const int64_t na = P.tpA[I + 1] - P.tpA[I];
    int64_t nd = 0, np = 0;
    for (int64_t t = t0 + lane; t < t1; t += 32) {
        nd += (P.tnzC[t + 1] - P.tnzC[t]) >= P.dense_threshold;
        np += P.pairCnt[t];
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        nd += __shfl_xor_sync(FULL, nd, o);
        np += __shfl_xor_sync(FULL, np, o);
    }
    const int64_t acc = (P.tnzC[t1] - P.tnzC[t0]) + 256 * nd;
    // the fixed part of the row's shared-memory layout (k_s3_row): accumulator, C and A tables, pairs
    const int64_t fixed = al16z(8 * acc) + al16z(32 * nt) + al16z(16 * nt) + al16z(8 * (nt + 1) + 16) +
                          al16z(8 * nt + 16) + al16z(4 * nt + 16) + al16z(32 * na) + al16z(16 * na) +
                          al16z(8 * (na + 1) + 16) + al16z(8 * np + 16) + al16z(8 * np);
    const bool ok = nt > 0 && nt <= R3_NTC && na <= R3_NAC && np <= R3_NPC && acc <= R3_ACC && fixed <= R3_SMEM;
    if (lane == 0) {
        P.rowAcc[I] = ok ? (int32_t)acc : -1;
        if (ok) atomicAdd(&P.cnt->n3rows, 1ULL);
        else atomicAdd(&P.cnt->n3fallback, (u64c)nt);
        if (ok) atomicAdd(&P.cnt->n3dense, (u64c)nd);
    }
    for (int64_t t = t0 + lane; t < t1; t += 32) P.skip[t] = ok;
}

// ------------------------------------------------------------------------------------------
// the row kernel
// ------------------------------------------------------------------------------------------
struct RowHdr {
    int64_t I, a0, t0, z0, p0;
    int na, nt, zr, acc;
    // byte offsets of the staged arrays in dynamic shared memory
    unsigned oCM, oCR, oCT, oPB, oPC, oAM, oAR, oAT, oAV, oPR, oDS, oB;
    unsigned pool;  // bump pointer (bytes) of the light-tile value pool
    int avStaged;
};

__device__ __forceinline__ unsigned al16(unsigned x) { return (x + 15u) & ~15u; }

// A tile classes of a row: its B tile row K is staged whole (heavy: >= 3 distinct columns), or
// only the rows c in colOcc(A_IK) are gathered (light: <= 2 columns), or read from L2 (no room)
constexpr int LIGHT_COLS = 2;
enum PairKind : unsigned { KIND_HEAVY = 0, KIND_LIGHT = 1, KIND_GLOBAL = 2 };

__global__ void __launch_bounds__(R3_T, 2) k_s3_row(RowParams P) {
    extern __shared__ __align__(128) unsigned char sm[];
    __shared__ __align__(8) uint64_t bar;
    __shared__ RowHdr H;
    __shared__ int32_t sKb[R3_NAC];     // first B tile (global index) of the B tile row of local A tile
    __shared__ int32_t sBoff[R3_NAC];   // byte offset of its staged B tile row (heavy), else -1
    __shared__ int32_t sLoff[R3_NAC];   // byte offset of its gathered rows (light), else -1
    __shared__ int32_t sBn[R3_NAC];     // tiles in that B tile row
    __shared__ uint16_t sCol[R3_NAC];   // colOcc of the A tile
    __shared__ uint32_t sCoff[R3_NTC];  // accumulator base of each C tile (DENSE_FLAG: 16x16 block)
    __shared__ uint32_t sKey[R3_NTC];         // work estimate of each C tile
    __shared__ uint8_t sOrder[R3_NTC];        // C tiles by descending work
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) mbar_init(&bar, 1);
    __syncthreads();
    unsigned phase = 0;
    for (;;) {
        // ---------------- next row (dynamic scheduling: rows differ in cost)
        if (tid == 0) {
            int64_t I;
            do {
                I = (int64_t)atomicAdd(&P.cnt->next3, 1ULL);
            } while (I < P.tm && P.rowAcc[I] < 0);
            H.I = I;
            if (I < P.tm) {
                const int64_t a0 = P.tpA[I], t0 = P.tpC[I], t1 = P.tpC[I + 1];
                H.a0 = a0;
                H.na = (int)(P.tpA[I + 1] - a0);
                H.t0 = t0;
                H.nt = (int)(t1 - t0);
                H.z0 = P.tnzC[t0];
                H.zr = (int)(P.tnzC[t1] - H.z0);
                H.acc = P.rowAcc[I];
                H.p0 = P.pairBeg[t0];
                const int np = (int)(P.pairBeg[t1 - 1] + P.pairCnt[t1 - 1] - H.p0);
                const int na = H.na, nt = H.nt;
                // layout: accumulator, C row tables, A row tables, pairs, A values, B tile rows
                unsigned o = al16(8u * (unsigned)H.acc);
                H.oCM = o; o += al16(32u * nt);
                H.oCR = o; o += al16(16u * nt);
                H.oCT = o; o += al16(8u * (nt + 1) + 16);
                H.oPB = o; o += al16(8u * nt + 16);
                H.oPC = o; o += al16(4u * nt + 16);
                H.oAM = o; o += al16(32u * na);
                H.oAR = o; o += al16(16u * na);
                H.oAT = o; o += al16(8u * (na + 1) + 16);
                H.oPR = o; o += al16(8u * np + 16);
                H.oDS = o; o += al16(8u * np);
                const int64_t av = na ? (P.tnzA[a0 + na] - P.tnzA[a0]) : 0;
                const unsigned avb = staged_bytes(P.vA + P.tnzA[a0], 8 * (size_t)av);
                H.avStaged = (o + avb + 1024 <= (unsigned)R3_SMEM);
                H.oAV = o;
                if (H.avStaged) o += avb;
                H.oB = o;
            }
        }
        __syncthreads();
        const int64_t I = H.I;
        if (I >= P.tm) break;
        const int64_t a0 = H.a0, t0 = H.t0, p0 = H.p0;
        const int na = H.na, nt = H.nt;

        // ---------------- warp 0: classify the A tiles, issue every bulk copy of the row
        if (warp == 0) {
            const int la = lane;
            int32_t kb0 = 0, nbk = 0;
            uint32_t co = 0;
            unsigned need = 0, lneed = 0;
            const double *bv = nullptr;
            int64_t bvn = 0;
            if (la < na) {
                const int64_t K = P.tcA[a0 + la];
                kb0 = (int32_t)P.tpB[K];
                nbk = (int32_t)(P.tpB[K + 1] - kb0);
                co = P.colOccA[a0 + la];
                if (nbk > 0 && __popc(co) > LIGHT_COLS) {
                    const int64_t v0 = P.tnzB[kb0];
                    bvn = P.tnzB[kb0 + nbk] - v0;
                    bv = P.vB + v0;
                    need = al16(32u * nbk) + al16(16u * nbk) + al16(8u * (nbk + 1) + 16) +
                           staged_bytes(bv, 8 * (size_t)bvn);
                } else if (nbk > 0) {
                    lneed = al16(4u * LIGHT_COLS * nbk);  // gather entries; values go to the pool
                }
            }
            unsigned incl = need, lincl = lneed;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const unsigned x = __shfl_up_sync(FULL, incl, d), y = __shfl_up_sync(FULL, lincl, d);
                if (lane >= d) {
                    incl += x;
                    lincl += y;
                }
            }
            const bool staged = need && H.oB + incl <= (unsigned)R3_SMEM;
            const unsigned hb = __shfl_sync(FULL, staged ? incl : 0u, 31);  // heavy bytes (a prefix fits)
            unsigned hbytes = __reduce_max_sync(FULL, staged ? incl : 0u);
            (void)hb;
            const unsigned lbase = H.oB + hbytes;
            const unsigned ltot = __shfl_sync(FULL, lincl, 31);
            const bool lstaged = lneed && lbase + ltot <= (unsigned)R3_SMEM;
            if (la < na) {
                sKb[la] = kb0;
                sBn[la] = nbk;
                sCol[la] = (uint16_t)co;
                sBoff[la] = staged ? (int32_t)(H.oB + incl - need) : -1;
                sLoff[la] = lstaged ? (int32_t)(lbase + lincl - lneed) : -1;
            }
            if (lane == 0) H.pool = al16(lbase + (lbase + ltot <= (unsigned)R3_SMEM ? ltot : 0u));
            fence_proxy_async();  // the previous row's generic accesses before the async writes
            if (staged) {
                unsigned char *d = sm + H.oB + incl - need;
                bulk_stage(d, P.mB + (int64_t)kb0 * TILE, 32 * (size_t)nbk, &bar);
                d += al16(32u * nbk);
                bulk_stage(d, P.rpB + (int64_t)kb0 * TILE, 16 * (size_t)nbk, &bar);
                d += al16(16u * nbk);
                bulk_stage(d, P.tnzB + kb0, 8 * (size_t)(nbk + 1), &bar);
                d += al16(8u * (nbk + 1) + 16);
                bulk_stage(d, bv, 8 * (size_t)bvn, &bar);
            }
            if (lane == 0) {
                bulk_stage(sm + H.oCM, P.mC + t0 * TILE, 32 * (size_t)nt, &bar);
                bulk_stage(sm + H.oCR, P.rpC + t0 * TILE, 16 * (size_t)nt, &bar);
                bulk_stage(sm + H.oCT, P.tnzC + t0, 8 * (size_t)(nt + 1), &bar);
                bulk_stage(sm + H.oPB, P.pairBeg + t0, 8 * (size_t)nt, &bar);
                bulk_stage(sm + H.oPC, P.pairCnt + t0, 4 * (size_t)nt, &bar);
            } else if (lane == 1) {
                bulk_stage(sm + H.oAM, P.mA + a0 * TILE, 32 * (size_t)na, &bar);
                bulk_stage(sm + H.oAR, P.rpA + a0 * TILE, 16 * (size_t)na, &bar);
                bulk_stage(sm + H.oAT, P.tnzA + a0, 8 * (size_t)(na + 1), &bar);
            } else if (lane == 2) {
                const int64_t t1 = t0 + nt;
                const int np = (int)(P.pairBeg[t1 - 1] + P.pairCnt[t1 - 1] - p0);
                bulk_stage(sm + H.oPR, P.pairs + p0, 8 * (size_t)np, &bar);
                if (H.avStaged && na) {
                    const int64_t v0 = P.tnzA[a0];
                    bulk_stage(sm + H.oAV, P.vA + v0, 8 * (size_t)(P.tnzA[a0 + na] - v0), &bar);
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&bar);
        } else {
            // other warps: zero the accumulator while the copies fly
            double2 *acc2 = reinterpret_cast<double2 *>(sm);
            const int n2 = (H.acc + 1) >> 1;
            for (int i = tid - 32; i < n2; i += R3_T - 32) acc2[i] = make_double2(0.0, 0.0);
        }
        __syncthreads();

        // ---------------- warps 1..: gather the B rows c in colOcc of every light A tile (L2 reads,
        // all light tiles of the row in flight at once instead of once per pair and thread)
        if (warp > 0) {
            for (int la = warp - 1; la < na; la += R3_T / 32 - 1) {
                const int lo = sLoff[la];
                if (lo < 0) continue;
                const int nbk = sBn[la], kb0 = sKb[la];
                const uint32_t co = sCol[la];
                const int c0 = __ffs(co) - 1;
                const int c1 = (co & (co - 1)) ? __ffs(co & (co - 1)) - 1 : -1;
                uint32_t *ent = reinterpret_cast<uint32_t *>(sm + lo);
                bool ok = true;
                for (int b0 = 0; b0 < nbk; b0 += 32) {
                    const int b = b0 + lane;
                    uint32_t m0 = 0, m1 = 0;
                    int r0 = 0, r1 = 0;
                    int64_t z = 0;
                    if (b < nbk) {
                        const int64_t t = (int64_t)kb0 + b;
                        m0 = P.mB[t * TILE + c0];
                        r0 = P.rpB[t * TILE + c0];
                        if (c1 >= 0) {
                            m1 = P.mB[t * TILE + c1];
                            r1 = P.rpB[t * TILE + c1];
                        }
                        z = P.tnzB[t];
                    }
                    const int n0 = __popc(m0), n1 = __popc(m1), cnt = n0 + n1;
                    int inc = cnt;
#pragma unroll
                    for (int d = 1; d < 32; d <<= 1) {
                        const int x = __shfl_up_sync(FULL, inc, d);
                        if (lane >= d) inc += x;
                    }
                    const int tot = __shfl_sync(FULL, inc, 31);
                    unsigned base = 0;
                    if (lane == 0) base = atomicAdd(&H.pool, 8u * (unsigned)tot);
                    base = __shfl_sync(FULL, base, 0);
                    if (base + 8u * tot > (unsigned)R3_SMEM) {
                        ok = false;
                        break;
                    }
                    const unsigned vi = (base >> 3) + (unsigned)(inc - cnt);  // pool index (doubles)
                    double *pv = reinterpret_cast<double *>(sm) + vi;
                    const double *g = P.vB + z;
                    for (int e = 0; e < n0; e++) pv[e] = g[r0 + e];
                    for (int e = 0; e < n1; e++) pv[n0 + e] = g[r1 + e];
                    if (b < nbk) {
                        ent[LIGHT_COLS * b] = m0 | (vi << 16);
                        ent[LIGHT_COLS * b + 1] = m1 | ((vi + n0) << 16);
                    }
                }
                if (!ok && lane == 0) sLoff[la] = -1;
            }
        }
        mbar_wait(&bar, phase);
        phase ^= 1u;

        const uint16_t *cM = reinterpret_cast<const uint16_t *>(sm + H.oCM);
        const uint8_t *cR = sm + H.oCR;
        const int64_t *cT = staged_ptr<int64_t>(sm + H.oCT, P.tnzC + t0);
        const int64_t *cPB = staged_ptr<int64_t>(sm + H.oPB, P.pairBeg + t0);
        const uint32_t *cPC = staged_ptr<uint32_t>(sm + H.oPC, P.pairCnt + t0);
        const uint16_t *aM = reinterpret_cast<const uint16_t *>(sm + H.oAM);
        const uint8_t *aR = sm + H.oAR;
        const int64_t *aT = staged_ptr<int64_t>(sm + H.oAT, P.tnzA + a0);
        const uint64_t *pr = staged_ptr<uint64_t>(sm + H.oPR, P.pairs + p0);
        const double *aVs = staged_ptr<double>(sm + H.oAV, P.vA + aT[0]);  // A row values (if staged)
        double *acc = reinterpret_cast<double *>(sm);
        const double *pool = reinterpret_cast<const double *>(sm);

        // ---- accumulator bases (warp 0)
        if (warp == 0) {
            int base = 0;
            for (int l0 = 0; l0 < nt; l0 += 32) {
                const int lt = l0 + lane;
                const bool v = lt < nt;
                const int64_t z = v ? cT[lt] - cT[0] : 0;
                const bool dn = v && (cT[lt + 1] - cT[lt]) >= P.dense_threshold;
                const unsigned dm = __ballot_sync(FULL, dn);
                if (v)
                    sCoff[lt] = dn ? (DENSE_FLAG | (unsigned)(H.zr + 256 * (base + __popc(dm & ((1u << lane) - 1u)))))
                                   : (unsigned)z;
                base += __popc(dm);
            }
        }
        __syncthreads();
        // ---- per C tile: pair descriptors (where B_KJ's mask, row offsets and values live, decoded
        // once per pair instead of once per (pair, row)) and the work key sum of nnz(A_IK)
        {
            uint64_t *desc = reinterpret_cast<uint64_t *>(sm + H.oDS);
            for (int lt = tid; lt < nt; lt += R3_T) {
                const int q0 = (int)(cPB[lt] - p0), q1 = q0 + (int)cPC[lt];
                uint32_t key = 0;
                for (int q = q0; q < q1; q++) {
                    const uint64_t pq = pr[q];
                    const int la = (int)((int64_t)(pq >> 32) - a0);
                    const int64_t pB = (int64_t)(uint32_t)pq;
                    const int lb = (int)(pB - sKb[la]);
                    const int boff = sBoff[la], loff = sLoff[la];
                    key += (uint32_t)(aT[la + 1] - aT[la]);
                    uint64_t d;
                    if (loff >= 0) {
                        d = (uint64_t)(loff + 4 * LIGHT_COLS * lb) | ((uint64_t)KIND_LIGHT << 59);
                    } else if (boff >= 0) {
                        const int nb = sBn[la];
                        const unsigned mo = (unsigned)boff + 32u * lb;
                        const unsigned ro = (unsigned)boff + al16(32u * nb) + 16u * lb;
                        const unsigned tb = (unsigned)boff + al16(32u * nb) + al16(16u * nb);
                        const int64_t *bt = staged_ptr<int64_t>(sm + tb, P.tnzB + sKb[la]);
                        const unsigned vb0 =
                            tb + al16(8u * (nb + 1) + 16) + (unsigned)((uintptr_t)(P.vB + bt[0]) & 15);
                        const unsigned vo = vb0 + 8u * (unsigned)(bt[lb] - bt[0]);
                        d = (uint64_t)mo | ((uint64_t)ro << 18) | ((uint64_t)vo << 36) | ((uint64_t)KIND_HEAVY << 59);
                    } else {
                        d = (uint64_t)pB | ((uint64_t)KIND_GLOBAL << 59);
                    }
                    desc[q] = d | ((uint64_t)la << 54);
                }
                sKey[lt] = key;
            }
        }
        __syncthreads();
        // tiles by descending work (stable): the two half warps of a warp get similar tiles
        for (int lt = tid; lt < nt; lt += R3_T) {
            const uint32_t k = sKey[lt];
            int rk = 0;
            for (int l2 = 0; l2 < nt; l2++) {
                const uint32_t k2 = sKey[l2];
                rk += (k2 > k) || (k2 == k && l2 < lt);
            }
            sOrder[rk] = (uint8_t)lt;
        }
        __syncthreads();
        const uint64_t *desc = reinterpret_cast<const uint64_t *>(sm + H.oDS);

        const bool avs = H.avStaged;
        // ---------------- numeric phase: a half warp per C tile (tiles by descending work), lane r
        // owns row r; pairs in ascending K, columns c ascending
        {
            const int hw = tid >> 4, r = tid & 15;
            for (int k = hw; k < nt; k += R3_T / 16) {
                const int lt = sOrder[k];
                const int u = lt * TILE + r;
                const uint32_t mCr = cM[u];
                const uint32_t off = sCoff[lt];
                const bool dense = off & DENSE_FLAG;
                const int sbase = dense ? (int)(off & ~DENSE_FLAG) + 16 * r : (int)off + cR[u];
                const int q0 = (int)(cPB[lt] - p0), q1 = q0 + (int)cPC[lt];
                for (int q = q0; q < q1; q++) {
                    const uint64_t d = desc[q];
                    const int la = (int)(d >> 54) & 31;
                    const uint32_t mAr = mCr ? aM[la * TILE + r] : 0u;
                    if (!mAr) continue;
                    const int ia = (int)(aT[la] - aT[0]) + aR[la * TILE + r];
                    const unsigned kind = (unsigned)(d >> 59);
                    if (kind == KIND_LIGHT) {
                        const unsigned eo = (unsigned)(d & 0x3ffffu);
                        const uint32_t co = sCol[la];
                        uint32_t x = mAr;
                        while (x) {
                            const int c = __ffs(x) - 1;
                            x &= x - 1;
                            const uint32_t en =
                                *reinterpret_cast<const uint32_t *>(sm + eo + 4 * __popc(co & ((1u << c) - 1u)));
                            uint32_t mbc = en & 0xffffu;
                            if (!mbc) continue;
                            const double a = avs ? aVs[ia + __popc(mAr & ((1u << c) - 1u))]
                                                 : P.vA[aT[0] + ia + __popc(mAr & ((1u << c) - 1u))];
                            const double *vb = pool + (en >> 16);
                            while (mbc) {
                                const int j = __ffs(mbc) - 1;
                                mbc &= mbc - 1;
                                const int slot = sbase + (dense ? j : __popc(mCr & ((1u << j) - 1u)));
                                acc[slot] = fma(a, *vb++, acc[slot]);
                            }
                        }
                    } else if (kind == KIND_HEAVY) {
                        const unsigned mo = (unsigned)(d & 0x3ffffu), ro = (unsigned)((d >> 18) & 0x3ffffu);
                        const unsigned vo = (unsigned)((d >> 36) & 0x3ffffu);
                        uint32_t x = mAr;
                        while (x) {
                            const int c = __ffs(x) - 1;
                            x &= x - 1;
                            uint32_t mbc = *reinterpret_cast<const uint16_t *>(sm + mo + 2 * c);
                            if (!mbc) continue;
                            const double a = avs ? aVs[ia + __popc(mAr & ((1u << c) - 1u))]
                                                 : P.vA[aT[0] + ia + __popc(mAr & ((1u << c) - 1u))];
                            const double *vb = reinterpret_cast<const double *>(sm + vo) + sm[ro + c];
                            while (mbc) {
                                const int j = __ffs(mbc) - 1;
                                mbc &= mbc - 1;
                                const int slot = sbase + (dense ? j : __popc(mCr & ((1u << j) - 1u)));
                                acc[slot] = fma(a, *vb++, acc[slot]);
                            }
                        }
                    } else {
                        const int64_t pB = (int64_t)(uint32_t)d;
                        const uint16_t *bm = P.mB + pB * TILE;
                        const uint8_t *br = P.rpB + pB * TILE;
                        const double *bv = P.vB + P.tnzB[pB];
                        uint32_t x = mAr;
                        while (x) {
                            const int c = __ffs(x) - 1;
                            x &= x - 1;
                            uint32_t mbc = bm[c];
                            if (!mbc) continue;
                            const double a = P.vA[aT[0] + ia + __popc(mAr & ((1u << c) - 1u))];
                            const double *vb = bv + br[c];
                            while (mbc) {
                                const int j = __ffs(mbc) - 1;
                                mbc &= mbc - 1;
                                const int slot = sbase + (dense ? j : __popc(mCr & ((1u << j) - 1u)));
                                acc[slot] = fma(a, *vb++, acc[slot]);
                            }
                        }
                    }
                }
            }
        }
        __syncthreads();
        // ---------------- compaction of dense blocks into the image, idx of every segment
        uint8_t *ix = P.ixC + H.z0;
        for (int u = tid; u < TILE * nt; u += R3_T) {
            const int lt = u >> 4, r = u & 15;
            uint32_t m = cM[u];
            if (!m) continue;
            const uint32_t off = sCoff[lt];
            const int zo = (int)(cT[lt] - cT[0]) + cR[u];
            int e = 0;
            if (off & DENSE_FLAG) {
                const double *blk = acc + (off & ~DENSE_FLAG) + 16 * r;
                while (m) {
                    const int j = __ffs(m) - 1;
                    m &= m - 1;
                    acc[zo + e] = blk[j];
                    ix[zo + e] = (uint8_t)((r << 4) | j);
                    e++;
                }
            } else {
                while (m) {
                    const int j = __ffs(m) - 1;
                    m &= m - 1;
                    ix[zo + e] = (uint8_t)((r << 4) | j);
                    e++;
                }
            }
        }
        __syncthreads();
        // ---------------- the row image is C's value layout: coalesced write-out
        double *out = P.vC + H.z0;
        for (int i = tid; i < H.zr; i += R3_T) out[i] = acc[i];
        __syncthreads();
    }
}

}  // namespace

void launch_step3_class(const RowParams &R, cudaStream_t s) {
    TSG_LAUNCH(k_s3_class, grid_for(R.tm, 8), 256, 0, s, R);
}

void launch_step3_rows(const RowParams &R, cudaStream_t s) {
    static int attr_done = -1;
    int dev = 0;
    TSG_CUDA(cudaGetDevice(&dev));
    if (attr_done != dev) {
        TSG_CUDA(cudaFuncSetAttribute(k_s3_row, cudaFuncAttributeMaxDynamicSharedMemorySize, R3_SMEM));
        attr_done = dev;
    }
    int per_sm = 0, sms = 0;
    TSG_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_s3_row, R3_T, R3_SMEM));
    TSG_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    const int64_t g = std::min<int64_t>((int64_t)std::max(per_sm, 1) * sms, std::max<int64_t>(R.tm, 1));
    TSG_LAUNCH(k_s3_row, (unsigned)g, R3_T, R3_SMEM, s, R);
}

}  // namespace tsg
