// tsg_scan.cu -- device exclusive prefix sum with int64 output (the "device prefix-sum
// allocation" between the steps: tile offsets, nonzero offsets).
//
// Single pass (chained scan with decoupled look-back): each 1024-thread CTA takes the next 8192
// inputs in launch order (ticket counter), publishes its sum, finds its prefix from the closest
// predecessors' published sums / inclusive prefixes (warp-parallel look-back, 32 predecessors per
// round), publishes its inclusive prefix and writes its outputs.  HBM traffic: 1 read + 1 write;
// one memset + one launch per scan.  In place (in == out) is allowed: a CTA reads all its inputs
// before writing.
#include "tsg_internal.cuh"

namespace tsg {

namespace {

constexpr int SCAN_T = 1024;
// inputs per thread: 16 for long arrays (half the CTAs, so half the look-back chain: C4's scans
// 3.29 -> 2.64 ms), 8 for short ones (a single CTA's latency: C1)
constexpr int SCAN_IPT_SHORT = 8, SCAN_IPT_LONG = 16;
constexpr int64_t SCAN_LONG_N = 1 << 16;

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

// tile status word: flag in the top 2 bits (0 = not ready, 1 = aggregate, 2 = inclusive prefix),
// value in the low 62 bits (all scanned quantities are counts < 2^62)
constexpr uint64_t ST_AGG = 1ull << 62, ST_PRE = 2ull << 62, ST_VAL = (1ull << 62) - 1;

__device__ __forceinline__ uint64_t ld_status(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_status(uint64_t *p, uint64_t v) {
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

template <typename Tin, int SCAN_IPT>
__global__ void __launch_bounds__(SCAN_T) k_scan_1pass(const Tin *in, int64_t n, int64_t *out, uint64_t *status,
                                                      unsigned long long *ticket, ExportArgs ex) { TSG_GRID_WAIT();
    __shared__ int64_t s_bid, s_base;
    if (threadIdx.x == 0) s_bid = gridDim.x == 1 ? 0 : (int64_t)atomicAdd(ticket, 1ull);
    __syncthreads();
    const int64_t b = s_bid;
    constexpr int SCAN_TILE = SCAN_T * SCAN_IPT;
    const int64_t base = b * SCAN_TILE + (int64_t)threadIdx.x * SCAN_IPT;
    int64_t v[SCAN_IPT];
    int64_t sum = 0;
    // a thread's SCAN_IPT consecutive inputs as 16-byte vector loads when the run is whole and
    // aligned (the element-wise form touches the same lines SCAN_IPT times)
    const bool vec = base + SCAN_IPT <= n && ((reinterpret_cast<uintptr_t>(in + base) & 15u) == 0);
    if (vec) {
        const uint4 *q = reinterpret_cast<const uint4 *>(in + base);
        constexpr int PER = 16 / (int)sizeof(Tin);
#pragma unroll
        for (int k = 0; k < SCAN_IPT / PER; k++) {
            const uint4 w = q[k];
            if constexpr (sizeof(Tin) == 8) {
                v[2 * k] = (int64_t)(((uint64_t)w.y << 32) | w.x);
                v[2 * k + 1] = (int64_t)(((uint64_t)w.w << 32) | w.z);
            } else {
                v[4 * k] = (int64_t)(Tin)w.x;
                v[4 * k + 1] = (int64_t)(Tin)w.y;
                v[4 * k + 2] = (int64_t)(Tin)w.z;
                v[4 * k + 3] = (int64_t)(Tin)w.w;
            }
        }
#pragma unroll
        for (int i = 0; i < SCAN_IPT; i++) sum += v[i];
    } else {
#pragma unroll
        for (int i = 0; i < SCAN_IPT; i++) {
            v[i] = (base + i < n) ? (int64_t)in[base + i] : 0;
            sum += v[i];
        }
    }
    int64_t total;
    int64_t pre = block_excl_scan(sum, &total);  // all reads of `in` by this CTA happen before
    if (threadIdx.x < 32) {
        const int lane = threadIdx.x;
        int64_t excl = 0;
        if (b == 0) {
            if (lane == 0 && gridDim.x > 1) st_status(status, ST_PRE | (uint64_t)total);
        } else {
            if (lane == 0) st_status(status + b, ST_AGG | (uint64_t)total);
            for (int64_t j = b - 1;; j -= 32) {
                const int64_t idx = j - lane;  // lane 0 = closest predecessor
                uint64_t st = idx >= 0 ? ld_status(status + idx) : ST_PRE;
                while (__any_sync(0xffffffffu, (st >> 62) == 0))
                    if ((st >> 62) == 0) st = ld_status(status + idx);
                const unsigned pm = __ballot_sync(0xffffffffu, (st >> 62) == 2);
                const int first = pm ? __ffs(pm) - 1 : 32;
                int64_t x = lane <= first ? (int64_t)(st & ST_VAL) : 0;
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
                excl += x;
                if (pm) break;
            }
            if (lane == 0) st_status(status + b, ST_PRE | (uint64_t)(excl + total));
        }
        if (lane == 0) s_base = excl;
    }
    __syncthreads();
    pre += s_base;
    if (base + SCAN_IPT <= n && ((reinterpret_cast<uintptr_t>(out + base) & 15u) == 0)) {
        uint4 *q = reinterpret_cast<uint4 *>(out + base);
#pragma unroll
        for (int k = 0; k < SCAN_IPT / 2; k++) {
            const int64_t x0 = pre;
            pre += v[2 * k];
            const int64_t x1 = pre;
            pre += v[2 * k + 1];
            q[k] = make_uint4((unsigned)x0, (unsigned)((uint64_t)x0 >> 32), (unsigned)x1, (unsigned)((uint64_t)x1 >> 32));
        }
    } else {
#pragma unroll
        for (int i = 0; i < SCAN_IPT; i++) {
            if (base + i < n) out[base + i] = pre;
            pre += v[i];
        }
    }
    if (base < n && base + SCAN_IPT >= n) out[n] = pre;  // the thread holding the last element
    if (ex.n && b == (int64_t)gridDim.x - 1) export_segments(ex);  // the CTA that wrote out[n]
}

__global__ void k_set_zero_i64(int64_t *p) { TSG_GRID_WAIT(); *p = 0; }
__global__ void k_export_only(ExportArgs a) { TSG_GRID_WAIT(); export_segments(a); }

}  // namespace

template <typename Tin>
void exclusive_scan(const Tin *in, int64_t *out, int64_t n, cudaStream_t s, Buffers &tmp, const ExportArgs *ex) {
    if (n <= 0) {
        TSG_LAUNCH(k_set_zero_i64, 1, 1, 0, s, out);
        if (ex) TSG_LAUNCH(k_export_only, 1, 256, 0, s, *ex);
        return;
    }
    const bool lng = n > SCAN_LONG_N;
    const int64_t nb = ceil_div(n, (int64_t)SCAN_T * (lng ? SCAN_IPT_LONG : SCAN_IPT_SHORT));
    uint64_t *status = tmp.get<uint64_t>(nb + 1);  // [0, nb): tile status, [nb]: ticket
    if (nb > 1) TSG_CUDA(cudaMemsetAsync(status, 0, sizeof(uint64_t) * (nb + 1), s));  // one CTA: no look-back
    if (lng)
        TSG_LAUNCH((k_scan_1pass<Tin, SCAN_IPT_LONG>), (unsigned)nb, SCAN_T, 0, s, in, n, out, status,
                   reinterpret_cast<unsigned long long *>(status + nb), ex ? *ex : ExportArgs{});
    else
        TSG_LAUNCH((k_scan_1pass<Tin, SCAN_IPT_SHORT>), (unsigned)nb, SCAN_T, 0, s, in, n, out, status,
                   reinterpret_cast<unsigned long long *>(status + nb), ex ? *ex : ExportArgs{});
}

template void exclusive_scan<int64_t>(const int64_t *, int64_t *, int64_t, cudaStream_t, Buffers &, const ExportArgs *);
template void exclusive_scan<int32_t>(const int32_t *, int64_t *, int64_t, cudaStream_t, Buffers &, const ExportArgs *);
template void exclusive_scan<uint32_t>(const uint32_t *, int64_t *, int64_t, cudaStream_t, Buffers &, const ExportArgs *);

}  // namespace tsg
