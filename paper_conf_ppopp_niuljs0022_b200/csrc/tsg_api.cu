// tsg_api.cu -- the extern "C" boundary of libtsg (include/tsg.h): argument validation, handle
// lifetime, allocation policy, error translation.  Every compute step lives in the kernels of
// tsg_convert.cu / tsg_spgemm.cu; this file launches nothing but two tiny rebase kernels.
#include <chrono>
#include <cstring>

#include "tsg_kernels.cuh"

namespace tsg {

std::atomic<int64_t> g_launches{0};
thread_local double t_host_alloc_ms = 0.0, t_host_sync_ms = 0.0;
double now_ms() {
    return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}
static thread_local std::string t_last_error;
static thread_local int64_t t_call_launches = 0;

void set_last_error(const std::string &msg) { t_last_error = msg; }
void note_launch() { t_call_launches++; }
void reset_call_launches() {
    t_call_launches = 0;
    t_host_alloc_ms = 0.0;
    t_host_sync_ms = 0.0;
}
int64_t call_launches() { return t_call_launches; }

static void ensure_pool_cached() {
    // keep freed blocks in the device's default pool (a caching allocator, reading A15)
    static std::atomic<int> done{-1};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return;
    if (done.load() == dev) return;
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
        uint64_t thr = UINT64_MAX;
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
    done.store(dev);
}

Arena &thread_arena() {
    static thread_local Arena arenas[16];
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0) dev = 0;
    Arena &a = arenas[dev & 15];
    a.dev = dev;
    return a;
}

void Buffers::enter_arena() {
    Arena &a = *arena_;
    if (a.depth++ == 0) {
        // the previous user of the arena may still run on another stream
        if (a.done && a.last != s_) TSG_CUDA(cudaStreamWaitEvent(s_, a.done, 0));
        // grow after a call that overflowed (stream-ordered free of the old buffer)
        if (a.want > a.cap) {
            if (a.base) cudaFreeAsync(a.base, s_);
            a.base = nullptr;
            a.cap = 0;
            const size_t cap = (a.want + (a.want >> 3) + ((size_t)1 << 20)) & ~(size_t)255;
            const double t0 = now_ms();
            void *p = nullptr;
            ensure_pool_cached();
            if (cudaMallocAsync(&p, cap, s_) == cudaSuccess) {
                a.base = static_cast<char *>(p);
                a.cap = cap;
            } else {
                cudaGetLastError();
            }
            t_host_alloc_ms += now_ms() - t0;
        }
        a.want = 0;
        a.off = 0;
    }
    mark_ = a.off;
}

void Buffers::leave_arena() {
    Arena &a = *arena_;
    a.off = mark_;
    if (--a.depth == 0) {
        if (!a.done) cudaEventCreateWithFlags(&a.done, cudaEventDisableTiming);
        if (a.done) cudaEventRecord(a.done, s_);
        a.last = s_;
    }
}

void arena_release_all(cudaStream_t s) {
    Arena &a = thread_arena();
    if (a.depth) return;
    if (a.base) cudaFreeAsync(a.base, s);
    a.base = nullptr;
    a.cap = a.off = a.want = 0;
}

void *Allocator::alloc(size_t bytes, cudaStream_t s) const {
    if (custom) return hook.alloc(bytes, (void *)s, hook.ctx);
    ensure_pool_cached();
    void *p = nullptr;
    cudaError_t e = cudaMallocAsync(&p, bytes, s);
    if (e != cudaSuccess) {
        cudaGetLastError();  // clear the sticky-free error state of a failed allocation
        return nullptr;
    }
    return p;
}

void Allocator::free(void *p, size_t bytes, cudaStream_t s) const {
    if (!p) return;
    if (custom)
        hook.free(p, bytes, (void *)s, hook.ctx);
    else
        cudaFreeAsync(p, s);
}

// Small device -> host reads (the blocking scalar reads between the steps) go through a kernel
// that writes them into mapped pinned host memory, not through a D2H copy: a D2H copy queues
// behind whatever the copy engine is already doing (a caller streaming the previous result to
// the host), a kernel's posted writes do not.
namespace {
__global__ void k_export(ExportArgs a) { TSG_GRID_WAIT(); export_segments(a); }
struct Mapped {
    uint8_t *h = nullptr;
    uint8_t *d = nullptr;
    unsigned int seq = 0;
};
constexpr size_t MAPPED_BYTES = 4096;
constexpr size_t FLAG_OFF = MAPPED_BYTES - 64;  // the completion flag's slot
}  // namespace

// The host waits for the export by spinning on its completion flag in mapped memory (microseconds
// sooner than a stream synchronisation wakes up), for up to SPIN_US; then -- long steps, or a
// failed kernel that never writes the flag -- it falls back to cudaStreamSynchronize, which also
// reports errors.  Either way the stream has passed the export when this returns.
constexpr double SPIN_US = 200.0;

static Mapped &mapped() {
    int dev = 0;
    TSG_CUDA(cudaGetDevice(&dev));
    static thread_local Mapped m[16];
    Mapped &mp = m[dev & 15];
    if (!mp.h) {
        void *h = nullptr, *d = nullptr;
        TSG_CUDA(cudaHostAlloc(&h, MAPPED_BYTES, cudaHostAllocMapped | cudaHostAllocPortable));
        TSG_CUDA(cudaHostGetDevicePointer(&d, h, 0));
        mp.h = static_cast<uint8_t *>(h);
        mp.d = static_cast<uint8_t *>(d);
        *reinterpret_cast<volatile unsigned int *>(mp.h + FLAG_OFF) = 0u;
    }
    return mp;
}

ExportArgs begin_read(std::initializer_list<DevRead> segs) {
    Mapped &mp = mapped();
    ExportArgs a{};
    uint32_t off = 0;
    TSG_REQUIRE(segs.size() <= 4, TSG_ERR_INTERNAL, "too many device reads");
    for (const DevRead &r : segs) {
        TSG_REQUIRE(off + r.bytes <= FLAG_OFF, TSG_ERR_INTERNAL, "device read too large");
        a.src[a.n] = static_cast<const uint8_t *>(r.dev);
        a.bytes[a.n] = (uint32_t)r.bytes;
        a.off[a.n] = off;
        a.n++;
        off += (uint32_t)((r.bytes + 15) & ~(size_t)15);
    }
    a.dst = mp.d;
    a.flag = reinterpret_cast<volatile unsigned int *>(mp.d + FLAG_OFF);
    a.seq = ++mp.seq;
    return a;
}

void finish_read(const ExportArgs &a, std::initializer_list<DevRead> segs, cudaStream_t s) {
    Mapped &mp = mapped();
    const double t0 = now_ms();
    volatile unsigned int *hf = reinterpret_cast<volatile unsigned int *>(mp.h + FLAG_OFF);
    bool seen = false;
    while (!(seen = (*hf == a.seq)) && (now_ms() - t0) * 1e3 < SPIN_US) {
    }
    if (seen) {
        std::atomic_thread_fence(std::memory_order_acquire);
        // the stream is past the export once its flag is visible; keep the stream-ordered
        // semantics of the old synchronisation for what the caller launches next
    } else {
        TSG_CUDA(cudaStreamSynchronize(s));
    }
    t_host_sync_ms += now_ms() - t0;
    int k = 0;
    for (const DevRead &r : segs) {
        memcpy(r.host, mp.h + a.off[k], r.bytes);
        k++;
    }
}

void read_device(std::initializer_list<DevRead> segs, cudaStream_t s) {
    const ExportArgs a = begin_read(segs);
    TSG_LAUNCH(k_export, 1, 256, 0, s, a);
    finish_read(a, segs, s);
}

int64_t read_scalar(const int64_t *dptr, cudaStream_t s) {
    int64_t v = 0;
    read_device({{&v, dptr, sizeof(v)}}, s);
    return v;
}

namespace {
__global__ void k_rebase(const int64_t *__restrict__ src, int64_t *__restrict__ dst, int64_t count) { TSG_GRID_WAIT();
    int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < count) dst[i] = src[i] - src[0];
}
}  // namespace

__global__ void k_add_i64(int64_t *__restrict__ a, int64_t count, int64_t v) { TSG_GRID_WAIT();
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < count) a[i] += v;
}
void launch_add_i64(int64_t *a, int64_t count, int64_t v, cudaStream_t s) {
    TSG_LAUNCH(k_add_i64, grid_for(count, 256), 256, 0, s, a, count, v);
}

void launch_rebase(const int64_t *src, int64_t *dst, int64_t count, cudaStream_t s) {
    TSG_LAUNCH(k_rebase, grid_for(count, 256), 256, 0, s, src, dst, count);
}

static void destroy_handle(tsg_tiles *T, cudaStream_t s) {
    if (!T) return;
    for (int i = 0; i < 7; i++)
        if (T->owns[i]) T->al.free(T->array(i), T->bytes[i], s);
    delete T;
}

template <typename F>
static tsg_status guarded(F &&f) {
    try {
        f();
        return TSG_OK;
    } catch (const Error &e) {
        set_last_error(e.msg);
        return e.status;
    } catch (const std::bad_alloc &) {
        set_last_error("host allocation failed");
        return TSG_ERR_OOM;
    } catch (...) {
        set_last_error("unknown internal error");
        return TSG_ERR_INTERNAL;
    }
}

}  // namespace tsg

using namespace tsg;

extern "C" {

const char *tsg_status_string(tsg_status s) {
    switch (s) {
        case TSG_OK: return "TSG_OK";
        case TSG_ERR_INVALID_ARG: return "TSG_ERR_INVALID_ARG";
        case TSG_ERR_SHAPE: return "TSG_ERR_SHAPE";
        case TSG_ERR_UNSORTED: return "TSG_ERR_UNSORTED";
        case TSG_ERR_OVERFLOW: return "TSG_ERR_OVERFLOW";
        case TSG_ERR_OOM: return "TSG_ERR_OOM";
        case TSG_ERR_CUDA: return "TSG_ERR_CUDA";
        case TSG_ERR_INTERNAL: return "TSG_ERR_INTERNAL";
    }
    return "TSG_ERR_UNKNOWN";
}

const char *tsg_last_error(void) { return t_last_error.c_str(); }
int tsg_abi_version(void) { return TSG_ABI_VERSION; }
int64_t tsg_kernel_launch_count(void) { return g_launches.load(); }

tsg_status tsg_csr_to_tiles(int64_t m, int64_t n, int64_t nnz, const int64_t *row_ptr,
                            const int32_t *col_idx, const double *val, uint32_t flags,
                            const tsg_allocator *al, void *stream, tsg_tiles **out) {
    return tsg_csr_to_tiles_typed(m, n, nnz, row_ptr, col_idx, val, TSG_F64, flags, al, stream, out);
}

tsg_status tsg_csr_to_tiles_typed(int64_t m, int64_t n, int64_t nnz, const int64_t *row_ptr,
                                  const int32_t *col_idx, const void *val, int32_t dtype, uint32_t flags,
                                  const tsg_allocator *al, void *stream, tsg_tiles **out) {
    if (out) *out = nullptr;
    return guarded([&] {
        TSG_REQUIRE(dtype_ok(dtype), TSG_ERR_INVALID_ARG, "unknown dtype");
        TSG_REQUIRE(out, TSG_ERR_INVALID_ARG, "out is NULL");
        TSG_REQUIRE(m >= 0 && n >= 0 && nnz >= 0, TSG_ERR_INVALID_ARG, "negative size");
        TSG_REQUIRE(row_ptr, TSG_ERR_INVALID_ARG, "row_ptr is NULL");
        TSG_REQUIRE(nnz == 0 || (col_idx && val), TSG_ERR_INVALID_ARG, "col_idx/val NULL with nnz > 0");
        TSG_REQUIRE((flags & ~(uint32_t)(TSG_INPUT_HOST | TSG_VALIDATE)) == 0, TSG_ERR_INVALID_ARG, "unknown flag");
        TSG_REQUIRE(n < ((int64_t)1 << 31) && m < ((int64_t)1 << 35), TSG_ERR_OVERFLOW, "dimension too large");
        cudaStream_t s = (cudaStream_t)stream;
        Allocator A = Allocator::from(al);
        tsg_tiles *T = new tsg_tiles();
        T->al = A;
        try {
            if (flags & TSG_INPUT_HOST) {
                Buffers staging(A, s, true);
                int64_t *drp = staging.get<int64_t>(m + 1);
                int32_t *dci = staging.get<int32_t>(nnz);
                void *dv = staging.get<uint8_t>((int64_t)dtype_size(dtype) * nnz);
                TSG_CUDA(cudaMemcpyAsync(drp, row_ptr, sizeof(int64_t) * (m + 1), cudaMemcpyHostToDevice, s));
                if (nnz) {
                    TSG_CUDA(cudaMemcpyAsync(dci, col_idx, sizeof(int32_t) * nnz, cudaMemcpyHostToDevice, s));
                    TSG_CUDA(cudaMemcpyAsync(dv, val, dtype_size(dtype) * nnz, cudaMemcpyHostToDevice, s));
                }
                launch_csr_to_tiles(m, n, nnz, drp, dci, dv, dtype, flags & TSG_VALIDATE, A, s, T);
            } else {
                launch_csr_to_tiles(m, n, nnz, row_ptr, col_idx, val, dtype, flags & TSG_VALIDATE, A, s, T);
            }
        } catch (...) {
            destroy_handle(T, s);
            throw;
        }
        *out = T;
    });
}

tsg_status tsg_spgemm(const tsg_tiles *A, const tsg_tiles *B, uint32_t flags, const tsg_allocator *al,
                      void *stream, tsg_tiles **C, tsg_stats *stats) {
    if (C) *C = nullptr;
    return guarded([&] {
        TSG_REQUIRE(A && B && C, TSG_ERR_INVALID_ARG, "NULL handle");
        TSG_REQUIRE(A->n == B->m, TSG_ERR_SHAPE, "A.n != B.m");
        cudaStream_t s = (cudaStream_t)stream;
        Allocator al_ = Allocator::from(al);
        tsg_tiles *T = new tsg_tiles();
        T->al = al_;
        try {
            try {
                run_spgemm(A, B, flags, al_, s, T, stats);
            } catch (const Retry &) {
                // step 1's scratch did not fit the cached arena (first call of a larger problem):
                // the arena grows on entry to the second attempt
                const int64_t syncs0 = 1;
                run_spgemm(A, B, flags, al_, s, T, stats);
                if (stats) stats->host_syncs += (int32_t)syncs0;
            }
        } catch (...) {
            destroy_handle(T, s);
            throw;
        }
        *C = T;
    });
}

tsg_status tsg_partition_tile_rows(const tsg_tiles *A, const tsg_tiles *B, int64_t parts, void *stream,
                                   int64_t *cuts, int64_t *products) {
    return guarded([&] {
        TSG_REQUIRE(A && B && cuts, TSG_ERR_INVALID_ARG, "NULL argument");
        TSG_REQUIRE(parts >= 1 && parts <= 500, TSG_ERR_INVALID_ARG, "parts must be in [1, 500]");
        TSG_REQUIRE(A->tn == B->tm, TSG_ERR_SHAPE, "tile shapes disagree");
        cudaStream_t s = (cudaStream_t)stream;
        Buffers tmp(Allocator{}, s, true);
        int32_t *rnnz = tmp.get<int32_t>(TILE * B->tm);
        int64_t *w = tmp.get<int64_t>(A->tm);
        int64_t *pre = tmp.get<int64_t>(A->tm + 1);
        int64_t *dcuts = tmp.get<int64_t>(parts + 1);
        launch_row_products(A->tm, A->tile_ptr, A->tile_col, A->mask, B->tm, B->tile_ptr, B->mask, rnnz, w, s);
        exclusive_scan<int64_t>(w, pre, A->tm, s, tmp);
        launch_cuts(pre, A->tm, parts, dcuts, s);
        int64_t tot = 0;
        read_device({{cuts, dcuts, sizeof(int64_t) * (size_t)(parts + 1)}, {&tot, pre + A->tm, sizeof(int64_t)}}, s);
        if (products) *products = tot;
    });
}

tsg_status tsg_tiles_transpose(const tsg_tiles *T, const tsg_allocator *al, void *stream, tsg_tiles **out) {
    if (out) *out = nullptr;
    return guarded([&] {
        TSG_REQUIRE(T && out, TSG_ERR_INVALID_ARG, "NULL argument");
        TSG_REQUIRE(T->m < ((int64_t)1 << 31), TSG_ERR_OVERFLOW, "A^T would have >= 2^31 columns");
        TSG_REQUIRE(((uintptr_t)T->mask & 15) == 0, TSG_ERR_INVALID_ARG, "mask must be 16-byte aligned");
        cudaStream_t s = (cudaStream_t)stream;
        Allocator A = Allocator::from(al);
        tsg_tiles *O = new tsg_tiles();
        O->al = A;
        try {
            launch_transpose_tiles(T, A, s, O);
        } catch (...) {
            destroy_handle(O, s);
            throw;
        }
        *out = O;
    });
}

tsg_status tsg_tiles_to_csr(const tsg_tiles *T, const tsg_allocator *al, void *stream, int64_t **row_ptr,
                            int32_t **col_idx, void **val, int64_t *nnz) {
    if (row_ptr) *row_ptr = nullptr;
    if (col_idx) *col_idx = nullptr;
    if (val) *val = nullptr;
    return guarded([&] {
        TSG_REQUIRE(T && row_ptr && col_idx && val, TSG_ERR_INVALID_ARG, "NULL argument");
        cudaStream_t s = (cudaStream_t)stream;
        Allocator A = Allocator::from(al);
        Buffers out(A, s);
        int64_t *rp = out.get<int64_t>(T->m + 1);
        int32_t *ci = out.get<int32_t>(T->nnz);
        void *v = out.get<uint8_t>((int64_t)T->vsize() * T->nnz);
        launch_tiles_to_csr(T, rp, ci, v, s);
        out.take(rp);
        out.take(ci);
        out.take(v);
        *row_ptr = rp;
        *col_idx = ci;
        *val = v;
        if (nnz) *nnz = T->nnz;
    });
}

tsg_status tsg_tiles_get_view(const tsg_tiles *T, tsg_tiles_view *o) {
    return guarded([&] {
        TSG_REQUIRE(T && o, TSG_ERR_INVALID_ARG, "NULL argument");
        o->m = T->m;
        o->n = T->n;
        o->tile_m = T->tm;
        o->tile_n = T->tn;
        o->num_tiles = T->nt;
        o->nnz = T->nnz;
        o->tile_ptr = T->tile_ptr;
        o->tile_col = T->tile_col;
        o->tile_nnz = T->tile_nnz;
        o->row_ptr = T->row_ptr;
        o->mask = T->mask;
        o->idx = T->idx;
        o->val = T->val;
        o->dtype = T->dtype;
    });
}

tsg_status tsg_tiles_wrap(const tsg_tiles_view *v, const tsg_allocator *owner, tsg_tiles **out) {
    if (out) *out = nullptr;
    return guarded([&] {
        TSG_REQUIRE(v && out, TSG_ERR_INVALID_ARG, "NULL argument");
        TSG_REQUIRE(v->m >= 0 && v->n >= 0 && v->num_tiles >= 0 && v->nnz >= 0, TSG_ERR_INVALID_ARG, "negative size");
        TSG_REQUIRE(v->tile_m == ceil_div(v->m, TILE) && v->tile_n == ceil_div(v->n, TILE), TSG_ERR_INVALID_ARG,
                    "tile_m/tile_n inconsistent with m/n");
        TSG_REQUIRE(v->tile_ptr && v->tile_nnz, TSG_ERR_INVALID_ARG, "tile_ptr/tile_nnz NULL");
        TSG_REQUIRE(dtype_ok(v->dtype), TSG_ERR_INVALID_ARG, "unknown dtype");
        tsg_tiles *T = new tsg_tiles();
        T->dtype = v->dtype;
        T->m = v->m;
        T->n = v->n;
        T->tm = v->tile_m;
        T->tn = v->tile_n;
        T->nt = v->num_tiles;
        T->nnz = v->nnz;
        T->tile_ptr = const_cast<int64_t *>(v->tile_ptr);
        T->tile_col = const_cast<int32_t *>(v->tile_col);
        T->tile_nnz = const_cast<int64_t *>(v->tile_nnz);
        T->row_ptr = const_cast<uint8_t *>(v->row_ptr);
        T->mask = const_cast<uint16_t *>(v->mask);
        T->idx = const_cast<uint8_t *>(v->idx);
        T->val = const_cast<void *>(v->val);
        if (owner) {
            T->al = Allocator::from(owner);
            TSG_REQUIRE(T->al.custom, TSG_ERR_INVALID_ARG, "owner allocator needs alloc and free");
            size_t b[7] = {sizeof(int64_t) * (size_t)(T->tm + 1), sizeof(int32_t) * (size_t)T->nt,
                           sizeof(int64_t) * (size_t)(T->nt + 1), (size_t)(16 * T->nt),
                           sizeof(uint16_t) * (size_t)(16 * T->nt), (size_t)T->nnz, T->vsize() * (size_t)T->nnz};
            for (int i = 0; i < 7; i++) {
                T->owns[i] = true;
                T->bytes[i] = b[i];
            }
        }
        *out = T;
    });
}

tsg_status tsg_tiles_slice_rows(const tsg_tiles *T, int64_t b, int64_t e, void *stream, tsg_tiles **view) {
    if (view) *view = nullptr;
    return guarded([&] {
        TSG_REQUIRE(T && view, TSG_ERR_INVALID_ARG, "NULL argument");
        TSG_REQUIRE(0 <= b && b <= e && e <= T->tm, TSG_ERR_INVALID_ARG, "tile row range out of bounds");
        cudaStream_t s = (cudaStream_t)stream;
        int64_t t0 = 0, t1 = 0, z0 = 0, z1 = 0;
        read_device({{&t0, T->tile_ptr + b, 8}, {&t1, T->tile_ptr + e, 8}}, s);
        read_device({{&z0, T->tile_nnz + t0, 8}, {&z1, T->tile_nnz + t1, 8}}, s);
        Allocator A;  // default pool for the two rebased offset arrays
        Buffers buf(A, s);
        int64_t *tp = buf.get<int64_t>(e - b + 1);
        int64_t *tz = buf.get<int64_t>(t1 - t0 + 1);
        launch_rebase(T->tile_ptr + b, tp, e - b + 1, s);
        launch_rebase(T->tile_nnz + t0, tz, t1 - t0 + 1, s);
        tsg_tiles *V = new tsg_tiles();
        V->m = std::min<int64_t>(TILE * (e - b), T->m - TILE * b);
        if (V->m < 0) V->m = 0;
        V->n = T->n;
        V->tm = e - b;
        V->tn = T->tn;
        V->nt = t1 - t0;
        V->nnz = z1 - z0;
        V->tile_ptr = tp;
        V->tile_col = T->tile_col + t0;
        V->tile_nnz = tz;
        V->row_ptr = T->row_ptr + 16 * t0;
        V->mask = T->mask + 16 * t0;
        V->idx = T->idx + z0;
        V->val = static_cast<uint8_t *>(T->val) + T->vsize() * (size_t)z0;
        V->dtype = T->dtype;
        V->al = A;
        V->owns[0] = V->owns[2] = true;
        V->bytes[0] = buf.take(tp);
        V->bytes[2] = buf.take(tz);
        *view = V;
    });
}

static tsg_status copy_to_host(const tsg_tiles *T, void *stream, int64_t *tile_ptr, int32_t *tile_col,
                               int64_t *tile_nnz, uint8_t *row_ptr, uint16_t *mask, uint8_t *idx, void *val,
                               bool blocking) {
    return guarded([&] {
        TSG_REQUIRE(T, TSG_ERR_INVALID_ARG, "NULL handle");
        cudaStream_t s = (cudaStream_t)stream;
        auto cp = [&](void *dst, const void *src, size_t bytes) {
            if (dst && bytes) TSG_CUDA(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, s));
        };
        cp(tile_ptr, T->tile_ptr, sizeof(int64_t) * (T->tm + 1));
        cp(tile_col, T->tile_col, sizeof(int32_t) * T->nt);
        cp(tile_nnz, T->tile_nnz, sizeof(int64_t) * (T->nt + 1));
        cp(row_ptr, T->row_ptr, 16 * T->nt);
        cp(mask, T->mask, sizeof(uint16_t) * 16 * T->nt);
        cp(idx, T->idx, T->nnz);
        cp(val, T->val, T->vsize() * T->nnz);
        if (blocking) TSG_CUDA(cudaStreamSynchronize(s));
    });
}

tsg_status tsg_tiles_copy_to_host(const tsg_tiles *T, void *stream, int64_t *tile_ptr, int32_t *tile_col,
                                  int64_t *tile_nnz, uint8_t *row_ptr, uint16_t *mask, uint8_t *idx, void *val) {
    return copy_to_host(T, stream, tile_ptr, tile_col, tile_nnz, row_ptr, mask, idx, val, true);
}

tsg_status tsg_tiles_copy_to_host_async(const tsg_tiles *T, void *stream, int64_t *tile_ptr, int32_t *tile_col,
                                        int64_t *tile_nnz, uint8_t *row_ptr, uint16_t *mask, uint8_t *idx,
                                        void *val) {
    return copy_to_host(T, stream, tile_ptr, tile_col, tile_nnz, row_ptr, mask, idx, val, false);
}

void tsg_tiles_destroy(tsg_tiles *T, void *stream) { destroy_handle(T, (cudaStream_t)stream); }

void tsg_free(void *ptr, size_t bytes, const tsg_allocator *al, void *stream) {
    Allocator::from(al).free(ptr, bytes, (cudaStream_t)stream);
}

size_t tsg_workspace_release(void *stream) {
    const size_t held = thread_arena().cap;
    arena_release_all((cudaStream_t)stream);
    return held;
}

}  // extern "C"
