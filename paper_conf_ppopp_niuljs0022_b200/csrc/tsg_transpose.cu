// tsg_transpose.cu -- tile-level transpose of a sparse-tile matrix, for the paper's second
// workload C = A*A^T (Fig 8).
//
// Tile (I, J) of A becomes tile (J, I) of A^T with its 16x16 pattern transposed: the new row
// masks are A's column masks, the new row offsets their prefix popcounts, and the values are
// re-ordered from A's row-major (r, c) order to (c, r) order.  Steps:
//   1. tiles per tile column J of A (atomic counts) -> scan -> tile_ptr of A^T
//   2. each tile row I drops its tiles into their column's slot range (atomic cursor per column)
//   3. a warp per column ranks its slots by I (tile rows are unique within a column), which
//      gives the ascending-I order of A^T's tile row J without a global sort; columns wider than
//      64 tiles (hubs) take a CTA with a tile-row bitmap and popcount ranks (linear, not k^2)
//   4. nnz offsets of A^T (scan), then a thread per tile writes the transposed tile.
// Exact (a permutation of A's data): compared bit for bit with the oracle's CSR transpose.
#include <algorithm>

#include "tsg_kernels.cuh"

namespace tsg {
namespace {

__global__ void k_tp_count(int64_t nt, const int32_t *__restrict__ tcol, unsigned long long *__restrict__ cnt) { TSG_GRID_WAIT();
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t < nt) atomicAdd(&cnt[tcol[t]], 1ULL);
}

// warp per tile row I of A: its tiles go to their column's slot range (any order)
__global__ void k_tp_place(int64_t tm, const int64_t *__restrict__ tp, const int32_t *__restrict__ tcol,
                           unsigned long long *__restrict__ cursor, int32_t *__restrict__ slotI,
                           int64_t *__restrict__ slotSrc) { TSG_GRID_WAIT();
    const int lane = threadIdx.x & 31;
    const int64_t I = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (I >= tm) return;
    for (int64_t t = tp[I] + lane; t < tp[I + 1]; t += 32) {
        const int64_t s = (int64_t)atomicAdd(&cursor[tcol[t]], 1ULL);
        slotI[s] = (int32_t)I;
        slotSrc[s] = t;
    }
}

// warp per tile column J: rank each slot by its tile row I -> A^T's tile (J, I) in ascending I.
// Columns of at most TP_SMALL tiles compare their slots directly (k^2 / 32 steps per lane); wider
// ones (R-MAT hub columns) go to a list for k_tp_rank_wide.
constexpr int TP_SMALL = 64;
__global__ void k_tp_rank(int64_t tn, const int64_t *__restrict__ tpT, const int32_t *__restrict__ slotI,
                          const int64_t *__restrict__ slotSrc, int64_t *__restrict__ perm,
                          int32_t *__restrict__ tcolT, int32_t *__restrict__ wide, unsigned long long *nwide) { TSG_GRID_WAIT();
    const int lane = threadIdx.x & 31;
    const int64_t J = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (J >= tn) return;
    const int64_t b = tpT[J], e = tpT[J + 1];
    if (e - b > TP_SMALL) {
        if (lane == 0) wide[atomicAdd(nwide, 1ULL)] = (int32_t)J;
        return;
    }
    for (int64_t s = b + lane; s < e; s += 32) {
        const int32_t I = slotI[s];
        int64_t rank = 0;
        for (int64_t s2 = b; s2 < e; s2++) rank += slotI[s2] < I;
        perm[b + rank] = slotSrc[s];
        tcolT[b + rank] = I;
    }
}

// fallback for the wide columns when the tile-row bitmap would not fit shared memory: a warp per
// wide column, ranks by comparison
__global__ void k_tp_rank_all(int64_t tn, const int64_t *__restrict__ tpT, const int32_t *__restrict__ slotI,
                              const int64_t *__restrict__ slotSrc, int64_t *__restrict__ perm,
                              int32_t *__restrict__ tcolT, const int32_t *__restrict__ wide,
                              const unsigned long long *nwide) { TSG_GRID_WAIT();
    const int lane = threadIdx.x & 31;
    const int64_t k = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    if (k >= (int64_t)*nwide) return;
    const int64_t J = wide[k];
    const int64_t b = tpT[J], e = tpT[J + 1];
    for (int64_t s = b + lane; s < e; s += 32) {
        const int32_t I = slotI[s];
        int64_t rank = 0;
        for (int64_t s2 = b; s2 < e; s2++) rank += slotI[s2] < I;
        perm[b + rank] = slotSrc[s];
        tcolT[b + rank] = I;
    }
}

// wide columns: a CTA each (persistent over the list), the column's tile rows marked in a
// shared-memory bitmap over all tile rows; a slot's rank is the number of marked rows before its
// own (per-word popcount prefix), as in step 1's rank kernel -- linear in the column's tiles
constexpr int TPW_T = 512;
__global__ void __launch_bounds__(TPW_T) k_tp_rank_wide(int64_t tm, const int64_t *__restrict__ tpT,
                                                       const int32_t *__restrict__ slotI,
                                                       const int64_t *__restrict__ slotSrc, int64_t *__restrict__ perm,
                                                       int32_t *__restrict__ tcolT, const int32_t *__restrict__ wide,
                                                       const unsigned long long *nwide) { TSG_GRID_WAIT();
    extern __shared__ uint32_t bm[];  // [words] bitmap, [words] exclusive popcount prefix
    __shared__ uint32_t wsum[TPW_T / 32 + 1];
    const int words = (int)((tm + 31) / 32);
    uint32_t *pre = bm + words;
    const int64_t n = (int64_t)*nwide;
    for (int64_t k = blockIdx.x; k < n; k += gridDim.x) {
        const int64_t J = wide[k];
        const int64_t b = tpT[J], e = tpT[J + 1];
        for (int w = threadIdx.x; w < words; w += TPW_T) bm[w] = 0;
        __syncthreads();
        for (int64_t s = b + threadIdx.x; s < e; s += TPW_T) {
            const int32_t I = slotI[s];
            atomicOr(&bm[I >> 5], 1u << (I & 31));
        }
        __syncthreads();
        // exclusive prefix of the word popcounts: blocked ownership, then a CTA scan of the sums
        const int per = (words + TPW_T - 1) / TPW_T;
        const int w0 = min(words, (int)threadIdx.x * per), w1 = min(words, w0 + per);
        uint32_t c = 0;
        for (int w = w0; w < w1; w++) c += __popc(bm[w]);
        const int lane = threadIdx.x & 31, wp = threadIdx.x >> 5;
        uint32_t incl = c;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t o = __shfl_up_sync(0xffffffffu, incl, d);
            if (lane >= d) incl += o;
        }
        if (lane == 31) wsum[wp] = incl;
        __syncthreads();
        if (threadIdx.x == 0) {
            uint32_t acc = 0;
            for (int q = 0; q < TPW_T / 32; q++) {
                const uint32_t x = wsum[q];
                wsum[q] = acc;
                acc += x;
            }
        }
        __syncthreads();
        uint32_t run = wsum[wp] + incl - c;
        for (int w = w0; w < w1; w++) {
            pre[w] = run;
            run += __popc(bm[w]);
        }
        __syncthreads();
        for (int64_t s = b + threadIdx.x; s < e; s += TPW_T) {
            const int32_t I = slotI[s];
            const int64_t rank = pre[I >> 5] + __popc(bm[I >> 5] & ((1u << (I & 31)) - 1u));
            perm[b + rank] = slotSrc[s];
            tcolT[b + rank] = I;
        }
        __syncthreads();
    }
}

__global__ void k_tp_nnz(int64_t nt, const int64_t *__restrict__ perm, const int64_t *__restrict__ tnz,
                         int64_t *__restrict__ tnzT) { TSG_GRID_WAIT();
    const int64_t d = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (d < nt) tnzT[d] = tnz[perm[d] + 1] - tnz[perm[d]];
}

// thread per tile of A^T: transpose source tile perm[d] (whose column masks are maskTs)
template <typename W>  // raw value words (8/4/2 bytes): a permutation of T's values
__global__ void k_tp_fill(int64_t nt, const int64_t *__restrict__ perm, const int64_t *__restrict__ tnz,
                          const uint16_t *__restrict__ mask, const uint16_t *__restrict__ maskTs,
                          const W *__restrict__ val, const int64_t *__restrict__ tnzT,
                          uint8_t *__restrict__ rpT, uint16_t *__restrict__ maskT, uint8_t *__restrict__ idxT,
                          W *__restrict__ valT) { TSG_GRID_WAIT();
    const int64_t d = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (d >= nt) return;
    const int64_t t = perm[d];
    const uint4 *pc = reinterpret_cast<const uint4 *>(maskTs + t * TILE);
    const uint4 c0 = pc[0], c1 = pc[1];
    reinterpret_cast<uint4 *>(maskT + d * TILE)[0] = c0;
    reinterpret_cast<uint4 *>(maskT + d * TILE)[1] = c1;
    const uint32_t cw[8] = {c0.x, c0.y, c0.z, c0.w, c1.x, c1.y, c1.z, c1.w};
    uint32_t rpw[4] = {0, 0, 0, 0};
    int offs[TILE];
    int run = 0;
#pragma unroll
    for (int c = 0; c < TILE; c++) {
        offs[c] = run;
        rpw[c >> 2] |= (uint32_t)run << (8 * (c & 3));
        run += __popc((cw[c >> 1] >> (16 * (c & 1))) & 0xffffu);
    }
    *reinterpret_cast<uint4 *>(rpT + d * TILE) = make_uint4(rpw[0], rpw[1], rpw[2], rpw[3]);
    // source entries in row-major (r, c) order; entry (r, c) lands in A^T's row c at rank of r
    int64_t z = tnz[t];
    const int64_t zT = tnzT[d];
    for (int r = 0; r < TILE; r++) {
        uint32_t m = mask[t * TILE + r];
        while (m) {
            const int c = __ffs(m) - 1;
            m &= m - 1;
            const uint32_t col = (cw[c >> 1] >> (16 * (c & 1))) & 0xffffu;  // rows r' of source column c
            const int pos = offs[c] + __popc(col & ((1u << r) - 1u));
            valT[zT + pos] = val[z];
            idxT[zT + pos] = (uint8_t)((c << 4) | r);
            z++;
        }
    }
}

}  // namespace

void launch_transpose_tiles(const tsg_tiles *T, const Allocator &al, cudaStream_t s, tsg_tiles *O) {
    Buffers tmp(al, s, true), out(al, s);
    const int64_t nt = T->nt, tmT = T->tn, tnT = T->tm;
    unsigned long long *cnt = tmp.get<unsigned long long>(tmT + 1);
    TSG_CUDA(cudaMemsetAsync(cnt, 0, sizeof(unsigned long long) * (tmT + 1), s));
    TSG_LAUNCH(k_tp_count, grid_for(nt, 256), 256, 0, s, nt, T->tile_col, cnt);
    int64_t *tpT = out.get<int64_t>(tmT + 1);
    exclusive_scan<int64_t>(reinterpret_cast<const int64_t *>(cnt), tpT, tmT, s, tmp);
    unsigned long long *cursor = tmp.get<unsigned long long>(tmT + 1);
    TSG_CUDA(cudaMemcpyAsync(cursor, tpT, sizeof(int64_t) * (tmT + 1), cudaMemcpyDeviceToDevice, s));
    int32_t *slotI = tmp.get<int32_t>(nt);
    int64_t *slotSrc = tmp.get<int64_t>(nt);
    TSG_LAUNCH(k_tp_place, grid_for(T->tm, 8), 256, 0, s, T->tm, T->tile_ptr, T->tile_col, cursor, slotI, slotSrc);
    int64_t *perm = tmp.get<int64_t>(nt);
    int32_t *tcolT = out.get<int32_t>(nt);
    int32_t *wide = tmp.get<int32_t>(tmT + 1);
    unsigned long long *nwide = reinterpret_cast<unsigned long long *>(cursor + tmT);  // zeroed below
    TSG_CUDA(cudaMemsetAsync(nwide, 0, sizeof(unsigned long long), s));
    TSG_LAUNCH(k_tp_rank, grid_for(tmT, 8), 256, 0, s, tmT, tpT, slotI, slotSrc, perm, tcolT, wide, nwide);
    const int64_t words = (T->tm + 31) / 32;
    const size_t smem = (size_t)words * 8;
    if (smem <= 200 * 1024) {  // tile rows of A <= 819200 (else the wide columns rank by comparisons)
        int dev = 0, nsm = 148;
        TSG_CUDA(cudaGetDevice(&dev));
        TSG_CUDA(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
        TSG_CUDA(cudaFuncSetAttribute(k_tp_rank_wide, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        TSG_LAUNCH(k_tp_rank_wide, (unsigned)std::min<int64_t>(std::max<int64_t>(tmT, 1), 2LL * nsm), TPW_T, smem, s,
                   T->tm, tpT, slotI, slotSrc, perm, tcolT, wide, nwide);
    } else {
        TSG_LAUNCH(k_tp_rank_all, grid_for(tmT, 8), 256, 0, s, tmT, tpT, slotI, slotSrc, perm, tcolT, wide, nwide);
    }
    int64_t *tnzT = out.get<int64_t>(nt + 1);
    TSG_LAUNCH(k_tp_nnz, grid_for(nt, 256), 256, 0, s, nt, perm, T->tile_nnz, tnzT);
    exclusive_scan<int64_t>(tnzT, tnzT, nt, s, tmp);
    uint16_t *mTs = tmp.get<uint16_t>(TILE * nt);
    launch_transpose(T->mask, nt, mTs, s);
    uint8_t *rpT = out.get<uint8_t>(TILE * nt);
    uint16_t *maskT = out.get<uint16_t>(TILE * nt);
    uint8_t *idxT = out.get<uint8_t>(T->nnz);
    void *valT = out.get<uint8_t>((int64_t)T->vsize() * T->nnz);
    switch (T->vsize()) {
        case 8:
            TSG_LAUNCH(k_tp_fill<uint64_t>, grid_for(nt, 128), 128, 0, s, nt, perm, T->tile_nnz, T->mask, mTs,
                       (const uint64_t *)T->val, tnzT, rpT, maskT, idxT, (uint64_t *)valT);
            break;
        case 4:
            TSG_LAUNCH(k_tp_fill<uint32_t>, grid_for(nt, 128), 128, 0, s, nt, perm, T->tile_nnz, T->mask, mTs,
                       (const uint32_t *)T->val, tnzT, rpT, maskT, idxT, (uint32_t *)valT);
            break;
        default:
            TSG_LAUNCH(k_tp_fill<uint16_t>, grid_for(nt, 128), 128, 0, s, nt, perm, T->tile_nnz, T->mask, mTs,
                       (const uint16_t *)T->val, tnzT, rpT, maskT, idxT, (uint16_t *)valT);
    }
    O->m = T->n;
    O->n = T->m;
    O->tm = tmT;
    O->tn = tnT;
    O->nt = nt;
    O->nnz = T->nnz;
    O->dtype = T->dtype;
    O->tile_ptr = tpT;
    O->tile_col = tcolT;
    O->tile_nnz = tnzT;
    O->row_ptr = rpT;
    O->mask = maskT;
    O->idx = idxT;
    O->val = valT;
    void *arr[7] = {tpT, tcolT, tnzT, rpT, maskT, idxT, valT};
    for (int k = 0; k < 7; k++) {
        O->bytes[k] = out.take(arr[k]);
        O->owns[k] = true;
    }
    O->al = al;
}

}  // namespace tsg
