// tsg_convert.cu -- CSR <-> sparse-tile conversion kernels.
//
// Format (Section 3.2): per tile row, tiles in ascending tile column; per tile, the
// nonzeros in row-major (r, c) order; idx = (r<<4)|c (reading A1); 16 local row offsets
// (reading A3); 16 row bit masks, bit c = column c (reading A2).
//
// Mapping: one warp handles two tile rows, one per 16-lane half; lane r of a half owns global
// row 16*I + r and walks its (sorted) CSR row.  Each round the half agrees on the smallest tile
// column J still pending (xor-shuffle min), the lanes owning entries in J consume them, and the
// tile's row offsets come from a 16-lane shuffle scan -- no atomics, no sorting: the CSR rows are
// already sorted, so a 16-way merge by tile column yields tiles in ascending J.
#include "tsg_internal.cuh"

namespace tsg {
namespace {

constexpr unsigned FULL = 0xffffffffu;
constexpr int NOJ = 0x7fffffff;

__device__ __forceinline__ int half_min(int v) {
#pragma unroll
    for (int o = 8; o > 0; o >>= 1) v = min(v, __shfl_xor_sync(FULL, v, o));
    return v;
}

// exclusive scan inside each 16-lane half (all 32 lanes must call)
__device__ __forceinline__ int half_excl_scan(int v, int r, int *total) {
    int incl = v;
#pragma unroll
    for (int d = 1; d < 16; d <<= 1) {
        int o = __shfl_up_sync(FULL, incl, d, 16);
        if (r >= d) incl += o;
    }
    *total = __shfl_sync(FULL, incl, 15, 16);
    return incl - v;
}

// TSG_VALIDATE: *bad = 2 if row_ptr is inconsistent with nnz (row_ptr[0] != 0, decreasing, or
// row_ptr[m] != nnz: the arrays are sized by nnz), else 1 for unsorted / duplicate / out-of-range
// columns (reading A12)
__global__ void k_validate_csr(int64_t m, int64_t n, int64_t nnz, const int64_t *__restrict__ rp,
                               const int32_t *__restrict__ ci, int *__restrict__ bad) { TSG_GRID_WAIT();
    int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= m) return;
    int64_t b = rp[i], e = rp[i + 1];
    if (b > e || b < 0 || e > nnz || (i == 0 && b != 0) || (i == m - 1 && e != nnz)) {
        atomicMax(bad, 2);
        return;
    }
    int64_t prev = -1;
    for (int64_t p = b; p < e; p++) {
        int64_t c = ci[p];
        if (c <= prev || c >= n) {
            atomicMax(bad, 1);
            return;
        }
        prev = c;
    }
}

// pass 1: number of non-empty tiles per tile row
__global__ void __launch_bounds__(256) k_c2t_count(int64_t m, int64_t tm, const int64_t *__restrict__ rp,
                                                   const int32_t *__restrict__ ci, int64_t *__restrict__ ntiles) { TSG_GRID_WAIT();
    const int lane = threadIdx.x & 31, r = lane & 15;
    const int64_t I = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 2 + (lane >> 4);
    const bool active = I < tm;
    const int64_t i = I * TILE + r;
    int64_t p = 0, e = 0;
    if (active && i < m) {
        p = rp[i];
        e = rp[i + 1];
    }
    int cur = (p < e) ? (ci[p] >> 4) : NOJ;
    int64_t cnt = 0;
    while (__any_sync(FULL, cur != NOJ)) {
        int jm = half_min(cur);
        if (jm != NOJ) {
            if (cur == jm) {
                do {
                    p++;
                } while (p < e && (ci[p] >> 4) == jm);
                cur = (p < e) ? (ci[p] >> 4) : NOJ;
            }
            cnt++;
        }
    }
    if (active && r == 0) ntiles[I] = cnt;
}

// pass 2: emit the seven arrays
// values are moved as raw words W of the value type's size (8/4/2 bytes): a permutation
template <typename W>
__global__ void __launch_bounds__(256) k_c2t_fill(int64_t m, int64_t tm, const int64_t *__restrict__ rp,
                                                  const int32_t *__restrict__ ci, const W *__restrict__ v,
                                                  const int64_t *__restrict__ tile_ptr, int32_t *__restrict__ tile_col,
                                                  int64_t *__restrict__ tile_nnz, uint8_t *__restrict__ row_ptr,
                                                  uint16_t *__restrict__ mask, uint8_t *__restrict__ idx,
                                                  W *__restrict__ val) { TSG_GRID_WAIT();
    const int lane = threadIdx.x & 31, r = lane & 15;
    const int64_t I = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 2 + (lane >> 4);
    const bool active = I < tm;
    const int64_t i = I * TILE + r;
    int64_t p = 0, e = 0, t = 0, off = 0;
    if (active) {
        t = tile_ptr[I];
        off = rp[I * TILE];  // the tile row's nonzeros are a permutation of its CSR range
        if (i < m) {
            p = rp[i];
            e = rp[i + 1];
        }
    }
    int cur = (p < e) ? (ci[p] >> 4) : NOJ;
    while (__any_sync(FULL, cur != NOJ)) {
        int jm = half_min(cur);
        int64_t p0 = p;
        uint32_t mk = 0;
        if (jm != NOJ && cur == jm) {
            do {
                mk |= 1u << (ci[p] & 15);
                p++;
            } while (p < e && (ci[p] >> 4) == jm);
            cur = (p < e) ? (ci[p] >> 4) : NOJ;
        }
        int c_r = (int)(p - p0), tot;
        int excl = half_excl_scan(c_r, r, &tot);
        if (jm != NOJ) {
            row_ptr[t * TILE + r] = (uint8_t)excl;
            mask[t * TILE + r] = (uint16_t)mk;
            if (r == 0) {
                tile_col[t] = jm;
                tile_nnz[t] = off;
            }
            for (int q = 0; q < c_r; q++) {
                int64_t pos = off + excl + q;
                idx[pos] = (uint8_t)((r << 4) | (ci[p0 + q] & 15));
                val[pos] = v[p0 + q];
            }
            off += tot;
            t++;
        }
    }
}

__global__ void k_set_i64(int64_t *p, int64_t v) { TSG_GRID_WAIT(); *p = v; }

// tiles -> CSR: lane r of a half owns global row 16I+r; row lengths are popcounts of the row's
// masks across the tile row; the CSR row offsets follow from the tile row's nonzero base.
template <typename W>
__global__ void __launch_bounds__(256) k_t2c(int64_t m, int64_t tm, const int64_t *__restrict__ tile_ptr,
                                             const int32_t *__restrict__ tile_col, const int64_t *__restrict__ tile_nnz,
                                             const uint8_t *__restrict__ row_ptr, const uint16_t *__restrict__ mask,
                                             const uint8_t *__restrict__ idx, const W *__restrict__ val,
                                             int64_t *__restrict__ out_rp, int32_t *__restrict__ out_ci,
                                             W *__restrict__ out_v) { TSG_GRID_WAIT();
    const int lane = threadIdx.x & 31, r = lane & 15;
    const int64_t I = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * 2 + (lane >> 4);
    const bool active = I < tm;
    int64_t t0 = 0, t1 = 0, base = 0;
    if (active) {
        t0 = tile_ptr[I];
        t1 = tile_ptr[I + 1];
        base = tile_nnz[t0];
    }
    int len = 0;
    for (int64_t t = t0; t < t1; t++) len += __popc(mask[t * TILE + r]);
    int tot;
    int excl = half_excl_scan(len, r, &tot);
    const int64_t i = I * TILE + r;
    if (!active || i >= m) return;
    int64_t pos = base + excl;
    out_rp[i] = pos;
    for (int64_t t = t0; t < t1; t++) {
        int c = __popc(mask[t * TILE + r]);
        if (!c) continue;
        int64_t src = tile_nnz[t] + row_ptr[t * TILE + r];
        int32_t J16 = tile_col[t] * TILE;
        for (int q = 0; q < c; q++) {
            out_ci[pos + q] = J16 + (idx[src + q] & 15);
            out_v[pos + q] = val[src + q];
        }
        pos += c;
    }
}

}  // namespace

void launch_csr_to_tiles(int64_t m, int64_t n, int64_t nnz, const int64_t *rp, const int32_t *ci, const void *v,
                         int32_t dtype, bool validate, const Allocator &al, cudaStream_t s, tsg_tiles *T) {
    Buffers tmp(al, s, true), out(al, s);
    const int64_t tm = ceil_div(m, TILE), tn = ceil_div(n, TILE);
    const unsigned grid = grid_for(ceil_div(tm, 2), 8);  // 8 warps x 2 tile rows per CTA
    if (validate && m > 0) {
        int *bad = tmp.get<int>(1);
        TSG_CUDA(cudaMemsetAsync(bad, 0, sizeof(int), s));
        TSG_LAUNCH(k_validate_csr, grid_for(m, 256), 256, 0, s, m, n, nnz, rp, ci, bad);
        int hbad = 0;
        read_device({{&hbad, bad, sizeof(int)}}, s);
        TSG_REQUIRE(hbad != 2, TSG_ERR_INVALID_ARG, "CSR row_ptr inconsistent with nnz (row_ptr[0] != 0, decreasing, or row_ptr[m] != nnz)");
        TSG_REQUIRE(!hbad, TSG_ERR_UNSORTED, "CSR input has unsorted, duplicate or out-of-range columns");
    }
    int64_t *tile_ptr = out.get<int64_t>(tm + 1);
    int64_t *ntiles = tmp.get<int64_t>(tm + 1);
    TSG_LAUNCH(k_c2t_count, grid, 256, 0, s, m, tm, rp, ci, ntiles);
    exclusive_scan<int64_t>(ntiles, tile_ptr, tm, s, tmp);
    const int64_t nt = read_scalar(tile_ptr + tm, s);
    TSG_REQUIRE(nt < ((int64_t)1 << 31), TSG_ERR_OVERFLOW, "more than 2^31 tiles");
    int32_t *tile_col = out.get<int32_t>(nt);
    int64_t *tile_nnz = out.get<int64_t>(nt + 1);
    uint8_t *row_ptr = out.get<uint8_t>(16 * nt);
    uint16_t *mask = out.get<uint16_t>(16 * nt);
    uint8_t *idx = out.get<uint8_t>(nnz);
    void *val = out.get<uint8_t>((int64_t)dtype_size(dtype) * nnz);
    switch (dtype_size(dtype)) {
        case 8:
            TSG_LAUNCH(k_c2t_fill<uint64_t>, grid, 256, 0, s, m, tm, rp, ci, (const uint64_t *)v, tile_ptr, tile_col,
                       tile_nnz, row_ptr, mask, idx, (uint64_t *)val);
            break;
        case 4:
            TSG_LAUNCH(k_c2t_fill<uint32_t>, grid, 256, 0, s, m, tm, rp, ci, (const uint32_t *)v, tile_ptr, tile_col,
                       tile_nnz, row_ptr, mask, idx, (uint32_t *)val);
            break;
        default:
            TSG_LAUNCH(k_c2t_fill<uint16_t>, grid, 256, 0, s, m, tm, rp, ci, (const uint16_t *)v, tile_ptr, tile_col,
                       tile_nnz, row_ptr, mask, idx, (uint16_t *)val);
    }
    TSG_LAUNCH(k_set_i64, 1, 1, 0, s, tile_nnz + nt, nnz);
    T->m = m;
    T->n = n;
    T->tm = tm;
    T->tn = tn;
    T->nt = nt;
    T->nnz = nnz;
    T->dtype = dtype;
    void *arr[7] = {tile_ptr, tile_col, tile_nnz, row_ptr, mask, idx, val};
    T->tile_ptr = tile_ptr;
    T->tile_col = tile_col;
    T->tile_nnz = tile_nnz;
    T->row_ptr = row_ptr;
    T->mask = mask;
    T->idx = idx;
    T->val = val;
    for (int k = 0; k < 7; k++) {
        T->bytes[k] = out.take(arr[k]);
        T->owns[k] = true;
    }
}

void launch_tiles_to_csr(const tsg_tiles *T, int64_t *rp, int32_t *ci, void *v, cudaStream_t s) {
    const unsigned grid = grid_for(ceil_div(T->tm, 2), 8);
    switch (T->vsize()) {
        case 8:
            TSG_LAUNCH(k_t2c<uint64_t>, grid, 256, 0, s, T->m, T->tm, T->tile_ptr, T->tile_col, T->tile_nnz, T->row_ptr,
                       T->mask, T->idx, (const uint64_t *)T->val, rp, ci, (uint64_t *)v);
            break;
        case 4:
            TSG_LAUNCH(k_t2c<uint32_t>, grid, 256, 0, s, T->m, T->tm, T->tile_ptr, T->tile_col, T->tile_nnz, T->row_ptr,
                       T->mask, T->idx, (const uint32_t *)T->val, rp, ci, (uint32_t *)v);
            break;
        default:
            TSG_LAUNCH(k_t2c<uint16_t>, grid, 256, 0, s, T->m, T->tm, T->tile_ptr, T->tile_col, T->tile_nnz, T->row_ptr,
                       T->mask, T->idx, (const uint16_t *)T->val, rp, ci, (uint16_t *)v);
    }
    TSG_LAUNCH(k_set_i64, 1, 1, 0, s, rp + T->m, T->nnz);
}

}  // namespace tsg
