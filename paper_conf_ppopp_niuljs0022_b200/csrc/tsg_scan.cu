// tsg_scan.cu -- device exclusive prefix sum with int64 output (the "device prefix-sum
// allocation" between the steps: tile offsets, nonzero offsets).
//
// Three phases per level: (1) each 1024-thread CTA reduces 8192 inputs to one sum, (2) the sums
// are scanned (recursively, same code), (3) each CTA rescans its 8192 inputs and adds its base.
// HBM traffic: 2 reads + 1 write of the input; used on arrays of at most a few hundred M entries.
#include "tsg_internal.cuh"

namespace tsg {

namespace {

constexpr int SCAN_T = 1024;
constexpr int SCAN_IPT = 8;
constexpr int SCAN_TILE = SCAN_T * SCAN_IPT;

__device__ __forceinline__ int64_t warp_incl_scan(int64_t v) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        int64_t o = __shfl_up_sync(0xffffffffu, v, d);
        if (lane >= d) v += o;
    }
    return v;
}

// exclusive scan of one value per thread across the CTA; returns this thread's prefix and
// writes the CTA total to *total
__device__ __forceinline__ int64_t block_excl_scan(int64_t v, int64_t *total) {
    __shared__ int64_t warp_sums[SCAN_T / 32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int64_t incl = warp_incl_scan(v);
    if (lane == 31) warp_sums[w] = incl;
    __syncthreads();
    if (w == 0) {
        int64_t x = (lane < (int)(blockDim.x >> 5)) ? warp_sums[lane] : 0;
        x = warp_incl_scan(x);
        warp_sums[lane] = x;  // inclusive over warps
    }
    __syncthreads();
    int64_t base = (w > 0) ? warp_sums[w - 1] : 0;
    *total = warp_sums[(blockDim.x >> 5) - 1];
    __syncthreads();
    return base + incl - v;
}

template <typename Tin>
__global__ void __launch_bounds__(SCAN_T) k_scan_reduce(const Tin *__restrict__ in, int64_t n,
                                                        int64_t *__restrict__ sums) {
    int64_t base = (int64_t)blockIdx.x * SCAN_TILE + (int64_t)threadIdx.x * SCAN_IPT;
    int64_t s = 0;
#pragma unroll
    for (int i = 0; i < SCAN_IPT; i++)
        if (base + i < n) s += (int64_t)in[base + i];
    int64_t total;
    block_excl_scan(s, &total);
    if (threadIdx.x == 0) sums[blockIdx.x] = total;
}

template <typename Tin>
__global__ void __launch_bounds__(SCAN_T) k_scan_down(const Tin *in, int64_t n, int64_t *out,
                                                      const int64_t *__restrict__ block_base) {
    int64_t base = (int64_t)blockIdx.x * SCAN_TILE + (int64_t)threadIdx.x * SCAN_IPT;
    int64_t v[SCAN_IPT];
    int64_t s = 0;
#pragma unroll
    for (int i = 0; i < SCAN_IPT; i++) {
        v[i] = (base + i < n) ? (int64_t)in[base + i] : 0;
        s += v[i];
    }
    int64_t total;
    int64_t pre = block_excl_scan(s, &total);  // all reads of `in` by this CTA happen before
    pre += block_base ? block_base[blockIdx.x] : 0;
#pragma unroll
    for (int i = 0; i < SCAN_IPT; i++) {
        if (base + i < n) out[base + i] = pre;
        pre += v[i];
    }
    if (base < n && base + SCAN_IPT >= n) out[n] = pre;  // the thread holding the last element
}

__global__ void k_set_zero_i64(int64_t *p) { *p = 0; }

}  // namespace

template <typename Tin>
void exclusive_scan(const Tin *in, int64_t *out, int64_t n, cudaStream_t s, Buffers &tmp) {
    if (n <= 0) {
        TSG_LAUNCH(k_set_zero_i64, 1, 1, 0, s, out);
        return;
    }
    int64_t nb = ceil_div(n, SCAN_TILE);
    if (nb == 1) {
        TSG_LAUNCH((k_scan_down<Tin>), 1, SCAN_T, 0, s, in, n, out, (const int64_t *)nullptr);
        return;
    }
    int64_t *sums = tmp.get<int64_t>(nb + 1);
    TSG_LAUNCH((k_scan_reduce<Tin>), (unsigned)nb, SCAN_T, 0, s, in, n, sums);
    exclusive_scan<int64_t>(sums, sums, nb, s, tmp);
    TSG_LAUNCH((k_scan_down<Tin>), (unsigned)nb, SCAN_T, 0, s, in, n, out, (const int64_t *)sums);
}

template void exclusive_scan<int64_t>(const int64_t *, int64_t *, int64_t, cudaStream_t, Buffers &);
template void exclusive_scan<int32_t>(const int32_t *, int64_t *, int64_t, cudaStream_t, Buffers &);
template void exclusive_scan<uint32_t>(const uint32_t *, int64_t *, int64_t, cudaStream_t, Buffers &);

}  // namespace tsg
