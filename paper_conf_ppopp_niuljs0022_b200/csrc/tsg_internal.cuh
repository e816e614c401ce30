// tsg_internal.cuh -- shared internals of libtsg (handle layout, allocation, errors, launches).
// Nothing here is visible through the C ABI (include/tsg.h).
#pragma once

#include <utility>

#include <initializer_list>

#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <atomic>
#include <string>
#include <vector>

#include "../../include/tsg.h"

namespace tsg {

constexpr int TILE = TSG_TILE;

// ------------------------------------------------------------------------------------------
// errors: thrown inside the library, converted to tsg_status at the ABI boundary
// ------------------------------------------------------------------------------------------
struct Error {
    tsg_status status;
    std::string msg;
};
// a call whose optimistically sized scratch overflowed: redo it once (the arena has grown)
struct Retry {};

void set_last_error(const std::string &msg);

[[noreturn]] inline void fail(tsg_status s, const std::string &msg) { throw Error{s, msg}; }

#define TSG_CUDA(call)                                                                          \
    do {                                                                                        \
        cudaError_t e_ = (call);                                                                \
        if (e_ != cudaSuccess)                                                                  \
            ::tsg::fail(e_ == cudaErrorMemoryAllocation ? TSG_ERR_OOM : TSG_ERR_CUDA,           \
                        std::string(#call) + ": " + cudaGetErrorString(e_) + " @" __FILE__ ":" + \
                            std::to_string(__LINE__));                                          \
    } while (0)

#define TSG_REQUIRE(cond, status, msg)                    \
    do {                                                  \
        if (!(cond)) ::tsg::fail((status), (msg));        \
    } while (0)

// launch bookkeeping: every kernel goes through TSG_LAUNCH so the evidence counter is exact
extern std::atomic<int64_t> g_launches;

// Programmatic dependent launch (sm_90+): every kernel is launched with programmatic stream
// serialization, and every kernel's first statement is TSG_GRID_WAIT() (griddepcontrol.wait:
// block until the preceding kernel of the stream has completed and its writes are visible), so
// stream order is kept while the next launch is prepared during the previous kernel's tail --
// chains of small kernels (C1-sized calls) lose part of the per-launch gap.  TSG_PDL=0 builds
// plain launches.
#ifndef TSG_PDL
#define TSG_PDL 1
#endif
#if defined(__CUDA_ARCH__)
#define TSG_GRID_WAIT() asm volatile("griddepcontrol.wait;\n" ::: "memory")
#else
#define TSG_GRID_WAIT()
#endif

template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kernel)(KArgs...), unsigned grid, unsigned block, size_t smem, cudaStream_t s,
                              Args &&...args) {
#if TSG_PDL
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(block);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
#else
    kernel<<<grid, block, smem, s>>>(std::forward<Args>(args)...);
    return cudaGetLastError();
#endif
}

#define TSG_LAUNCH(kernel, grid, block, smem, stream, ...)                                     \
    do {                                                                                        \
        if ((grid) > 0) {                                                                       \
            TSG_CUDA(::tsg::launch_pdl(kernel, (unsigned)(grid), (unsigned)(block), (size_t)(smem), \
                                       (stream), ##__VA_ARGS__));                               \
            ::tsg::g_launches.fetch_add(1, std::memory_order_relaxed);                          \
            ::tsg::note_launch();                                                               \
        }                                                                                       \
    } while (0)

void note_launch();  // per-call counter (thread-local)

// host-time accounting of one call (thread-local): blocked in scalar reads / allocation calls
extern thread_local double t_host_alloc_ms, t_host_sync_ms;
double now_ms();

// ------------------------------------------------------------------------------------------
// allocation: either the user's stream-ordered hook or cudaMallocAsync on the default pool
// ------------------------------------------------------------------------------------------
struct Allocator {
    tsg_allocator hook{};
    bool custom = false;
    static Allocator from(const tsg_allocator *al) {
        Allocator a;
        if (al && al->alloc && al->free) {
            a.hook = *al;
            a.custom = true;
        }
        return a;
    }
    void *alloc(size_t bytes, cudaStream_t s) const;
    void free(void *p, size_t bytes, cudaStream_t s) const;
};

// Scratch arena (per host thread and device): one cached device buffer handed out as a stack.
// Scratch of a call never goes back to the allocator, so the stream-ordered pool only holds
// outputs and its layout stays stable run to run (no pool growth -- i.e. no synchronous memory
// mapping -- inside a timed call once the arena has reached the workload's peak).  The arena is
// grown after a call that overflowed it; a CUDA event orders its reuse on another stream.
struct Arena {
    int dev = -1;
    char *base = nullptr;
    size_t cap = 0, off = 0, want = 0;
    int64_t u_hint = 0;  // step-1 candidates to reserve scratch for (the largest call seen)
    cudaEvent_t done = nullptr;
    cudaStream_t last = nullptr;
    int depth = 0;
};
Arena &thread_arena();
void arena_release_all(cudaStream_t s);  // free the calling thread's arena (stream-ordered)

// RAII list of device buffers; frees (stream-ordered) whatever is still owned at scope exit.
// With scratch=true (and no user allocator) buffers come from the thread's arena.
class Buffers {
   public:
    Buffers(const Allocator &al, cudaStream_t s, bool scratch = false) : al_(al), s_(s) {
        if (scratch && !al.custom) {
            arena_ = &thread_arena();
            enter_arena();
        }
    }
    ~Buffers() {
        release_all();
        if (arena_) leave_arena();
    }
    template <typename T>
    T *get(int64_t count) {
        size_t bytes = sizeof(T) * (size_t)(count > 0 ? count : 0);
        if (bytes < 256) bytes = 256;  // never hand out NULL; keep 256-byte alignment
        bytes = (bytes + 255) & ~(size_t)255;
        handed_ += bytes;
        if (arena_) {
            Arena &a = *arena_;
            if (a.off + bytes <= a.cap) {
                void *p = a.base + a.off;
                a.off += bytes;
                return static_cast<T *>(p);
            }
            // overflow: served by the allocator below; keep counting so the arena is grown to
            // this call's whole scratch peak for the next call
            a.off += bytes;
            if (a.off > a.want) a.want = a.off;
        }
        const double t0 = now_ms();
        void *p = al_.alloc(bytes, s_);
        t_host_alloc_ms += now_ms() - t0;
        if (!p) fail(TSG_ERR_OOM, "device allocation of " + std::to_string(bytes) + " bytes failed");
        items_.push_back({p, bytes});
        return static_cast<T *>(p);
    }
    // detach a buffer from the list (ownership moves to a handle); returns its byte size
    size_t take(void *p) {
        for (size_t i = 0; i < items_.size(); i++)
            if (items_[i].p == p) {
                size_t b = items_[i].bytes;
                items_[i] = items_.back();
                items_.pop_back();
                return b;
            }
        fail(TSG_ERR_INTERNAL, "take() of an unknown buffer");
    }
    void release_all() {
        for (auto &it : items_) al_.free(it.p, it.bytes, s_);
        items_.clear();
    }
    // bytes handed out by get() so far (scratch is a stack within a call: this is its peak)
    size_t handed() const { return handed_; }
    // the cached arena: whether this list draws from it, its free bytes, and a request that the
    // next call find at least `bytes` more free than this one had (the arena grows on entry)
    bool arena_backed() const { return arena_ != nullptr; }
    size_t arena_free() const { return arena_ && arena_->off < arena_->cap ? arena_->cap - arena_->off : 0; }
    void arena_need(size_t bytes) {
        if (arena_) arena_->want = std::max(arena_->want, arena_->off + bytes);
    }
    int64_t *arena_hint() { return arena_ ? &arena_->u_hint : nullptr; }

   private:
    void enter_arena();
    void leave_arena();
    struct Item {
        void *p;
        size_t bytes;
    };
    Allocator al_;
    cudaStream_t s_;
    std::vector<Item> items_;
    Arena *arena_ = nullptr;
    size_t mark_ = 0;
    size_t handed_ = 0;
};

}  // namespace tsg

namespace tsg {
inline size_t dtype_size(int32_t d) { return d == TSG_F64 ? 8 : d == TSG_F32 ? 4 : 2; }
inline bool dtype_ok(int32_t d) { return d == TSG_F64 || d == TSG_F32 || d == TSG_F16; }
}  // namespace tsg

// ------------------------------------------------------------------------------------------
// the handle (opaque in the ABI)
// ------------------------------------------------------------------------------------------
struct tsg_tiles {
    int64_t m = 0, n = 0, tm = 0, tn = 0, nt = 0, nnz = 0;
    int64_t *tile_ptr = nullptr;
    int32_t *tile_col = nullptr;
    int64_t *tile_nnz = nullptr;
    uint8_t *row_ptr = nullptr;
    uint16_t *mask = nullptr;
    uint8_t *idx = nullptr;
    void *val = nullptr;
    int32_t dtype = TSG_F64;  // tsg_dtype of val
    size_t vsize() const { return tsg::dtype_size(dtype); }
    // ownership: which arrays this handle frees, their byte sizes, and through what
    tsg::Allocator al;
    bool owns[7] = {false, false, false, false, false, false, false};
    size_t bytes[7] = {0, 0, 0, 0, 0, 0, 0};
    void *array(int i) const {
        void *a[7] = {tile_ptr, tile_col, tile_nnz, row_ptr, mask, idx, val};
        return a[i];
    }
};

namespace tsg {

// ------------------------------------------------------------------------------------------
// device scan: out[0] = 0, out[i+1] = out[i] + in[i]; out has n+1 entries; out may alias in
// when Tin == int64_t.  Three-phase (reduce / scan sums / downsweep), recursive on the sums.
// ------------------------------------------------------------------------------------------
struct ExportArgs;
template <typename Tin>
void exclusive_scan(const Tin *in, int64_t *out, int64_t n, cudaStream_t s, Buffers &tmp,
                    const ExportArgs *ex = nullptr);  // ex: the CTA that writes out[n] then exports

// read one int64 from device memory (blocking on stream s)
int64_t read_scalar(const int64_t *dptr, cudaStream_t s);
// blocking read of up to 4 small device ranges (<= 4 KB in total) into host memory, through a
// kernel writing mapped pinned memory (no D2H copy-engine traffic); counts into t_host_sync_ms
struct DevRead {
    void *host;
    const void *dev;
    size_t bytes;
};
void read_device(std::initializer_list<DevRead> segs, cudaStream_t s);
// A blocking read whose export runs at the end of a kernel the call launches anyway (the scan
// producing the value read): begin_read() lays the segments out in the thread's mapped buffer,
// the kernel copies them and raises the flag, finish_read() waits for it and copies them out.
struct ExportArgs {
    const uint8_t *src[4];
    uint32_t bytes[4], off[4];
    int n;  // 0: no export
    uint8_t *dst;
    volatile unsigned int *flag;  // written last, after a system-scope fence
    unsigned int seq;
};
ExportArgs begin_read(std::initializer_list<DevRead> segs);
void finish_read(const ExportArgs &a, std::initializer_list<DevRead> segs, cudaStream_t s);
// inside a kernel, by one whole CTA, after everything the segments cover is written
__device__ __forceinline__ void export_segments(const ExportArgs &a) {
    __syncthreads();
    __threadfence();
    for (int k = 0; k < a.n; k++)
        for (uint32_t i = threadIdx.x; i < a.bytes[k]; i += blockDim.x)
            a.dst[a.off[k] + i] = *((volatile const uint8_t *)a.src[k] + i);
    __threadfence_system();
    __syncthreads();
    if (threadIdx.x == 0) *a.flag = a.seq;
}

// per-call launch counter (thread-local)
void reset_call_launches();
int64_t call_launches();

// kernels shared by the API translation units
void launch_csr_to_tiles(int64_t m, int64_t n, int64_t nnz, const int64_t *rp, const int32_t *ci,
                         const void *v, int32_t dtype, bool validate, const Allocator &al, cudaStream_t s,
                         tsg_tiles *out);
void launch_tiles_to_csr(const tsg_tiles *T, int64_t *rp, int32_t *ci, void *v, cudaStream_t s);
void launch_rebase(const int64_t *src, int64_t *dst, int64_t count, cudaStream_t s);
void launch_add_i64(int64_t *a, int64_t count, int64_t v, cudaStream_t s);  // a[0..count) += v
void launch_transpose_tiles(const tsg_tiles *T, const Allocator &al, cudaStream_t s, tsg_tiles *O);
void run_spgemm(const tsg_tiles *A, const tsg_tiles *B, uint32_t flags, const Allocator &al,
                cudaStream_t s, tsg_tiles *C, tsg_stats *stats);

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }
inline unsigned grid_for(int64_t work, int per_block, int64_t cap = 1 << 30) {
    int64_t g = ceil_div(work, per_block);
    if (g > cap) g = cap;
    return (unsigned)(g > 0 ? g : 0);
}

}  // namespace tsg
