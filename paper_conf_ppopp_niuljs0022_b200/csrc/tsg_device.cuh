// tsg_device.cuh -- device helpers shared by the step kernels (tsg_step1.cu, tsg_step23.cu,
// tsg_rows.cu): value-type conversion / FMA of the precision variants, 16-byte cp.async, the
// step-2/3 work queue, 8-wide shared-memory vector loads.
#pragma once

#include <cuda_fp16.h>

#include "tsg_kernels.cuh"

namespace tsg {

constexpr unsigned FULLW = 0xffffffffu;

// ---- value types: TI = stored input type, TO = accumulator/output type
// (double x double -> double, float x float -> float, half x half -> float)
template <typename TO> __device__ __forceinline__ TO vcvt(double x) { return (TO)x; }
template <typename TO> __device__ __forceinline__ TO vcvt(float x) { return (TO)x; }
template <typename TO> __device__ __forceinline__ TO vcvt(__half x) { return (TO)__half2float(x); }
__device__ __forceinline__ double vfma(double a, double b, double c) { return fma(a, b, c); }
__device__ __forceinline__ float vfma(float a, float b, float c) { return fmaf(a, b, c); }

// 16-byte global -> shared copy (LDGSTS), completion through cp_wait_all()
__device__ __forceinline__ void cp16(void *dst_smem, const void *src) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst_smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(d), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_wait_all() {
    asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;\n" ::: "memory");
}

// Dynamic work distribution: warps take the next `chunk` units from a per-kernel counter, so the
// warps running at any moment work on neighbouring units (their A and B tiles stay in L2) and a
// warp that drew light units takes more.  The next chunk is requested one chunk ahead, so the
// atomic's latency overlaps the current work.  chunk == 0: static grid-stride distribution.
struct WorkQueue {
    unsigned long long *ctr;
    int64_t n;
    int chunk;
    long long nxt = 0;  // lane 0: first unit of the next chunk
    int64_t cur = 0, end = 0, stride = 0;
    __device__ WorkQueue(unsigned long long *c, int64_t units, int ch, int lane, int warps_per_cta)
        : ctr(c), n(units), chunk(ch) {
        if (ch == 0) {
            cur = (int64_t)blockIdx.x * warps_per_cta + (threadIdx.x >> 5);
            stride = (int64_t)gridDim.x * warps_per_cta;
        } else if (lane == 0) {
            nxt = (long long)atomicAdd(ctr, (unsigned long long)ch);
        }
    }
    __device__ __forceinline__ bool next(int64_t &u, int lane) {
        if (chunk == 0) {
            u = cur;
            cur += stride;
            return u < n;
        }
        if (cur >= end) {
            cur = (int64_t)__shfl_sync(FULLW, nxt, 0);
            if (cur >= n) return false;
            end = min(cur + (int64_t)chunk, n);
            if (lane == 0) nxt = (long long)atomicAdd(ctr, (unsigned long long)chunk);
        }
        u = cur++;
        return true;
    }
};

// 16x16 bit-matrix transpose across the 16 lanes of a half warp: lane i holds row i (bit c =
// M[i][c]); afterwards lane c holds column c (bit i = M[i][c]).  Four butterfly stages.
__device__ __forceinline__ uint32_t bit_transpose16(uint32_t v, int r) {
#pragma unroll
    for (int s = 8; s > 0; s >>= 1) {
        const uint32_t m = s == 8 ? 0x00ffu : s == 4 ? 0x0f0fu : s == 2 ? 0x3333u : 0x5555u;
        const uint32_t x = __shfl_xor_sync(FULLW, v, s);
        v = (r & s) ? ((v & ~m & 0xffffu) | ((x >> s) & m)) : ((v & m) | ((x << s) & ~m & 0xffffu));
    }
    return v;
}

// rows r of a 16x16 tile (mask words w[0..7], two rows per word) with mask[r] & occ != 0, as bits
__device__ __forceinline__ uint32_t rows_meeting(const uint4 &a0, const uint4 &a1, uint32_t occ) {
    const uint32_t o2 = occ * 0x10001u;
    const uint32_t w[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
    uint32_t rows = 0;
#pragma unroll
    for (int k = 0; k < 8; k++) {
        const uint32_t h = __vcmpne2(w[k] & o2, 0u);
        rows |= ((h & 1u) << (2 * k)) | (((h >> 16) & 1u) << (2 * k + 1));
    }
    return rows;
}

// eight consecutive accumulator-type values from shared memory (16-byte vector loads)
__device__ __forceinline__ void lds8(const double *p, double (&b)[8]) {
#pragma unroll
    for (int k = 0; k < 4; k++) {
        const double2 v = reinterpret_cast<const double2 *>(p)[k];
        b[2 * k] = v.x;
        b[2 * k + 1] = v.y;
    }
}
__device__ __forceinline__ void lds8(const float *p, float (&b)[8]) {
#pragma unroll
    for (int k = 0; k < 2; k++) {
        const float4 v = reinterpret_cast<const float4 *>(p)[k];
        b[4 * k] = v.x;
        b[4 * k + 1] = v.y;
        b[4 * k + 2] = v.z;
        b[4 * k + 3] = v.w;
    }
}

}  // namespace tsg
