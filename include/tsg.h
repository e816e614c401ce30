/*
 * tsg.h -- C ABI of the B200-native TileSpGEMM hot path.
 *
 * Method: Niu, Lu, Ji, Zhang, Liu, "TileSpGEMM: A Tiled Algorithm for Parallel Sparse General
 * Matrix-Matrix Multiplication on GPUs", PPoPP'22.  Citations "P:a-b" are lines of
 * /root/reference/PAPER.md; readings A1..A17 are listed in DESIGN.md §2.
 *
 * Problem statement: C = A*B with A, B and C sparse.  Input CSR,
 * output C in the sparse-tile format of Section 3.2, which can be fed back as an
 * input without conversion.
 *
 * Conventions shared by every entry point
 *  - Memory: unless a flag says otherwise every array pointer is a DEVICE pointer on the
 *    current CUDA device.  Index/offset arrays are int64 where they count nonzeros or tiles
 *    (reading A4: nnz(C) may exceed 2^31), int32 for column ids (n < 2^31 required).
 *  - Streams: every call is stream-ordered on `stream` (a cudaStream_t passed as void*,
 *    NULL = legacy default stream).  Inputs are borrowed: keep them alive until the stream has
 *    passed the call.  Calls that must know a size before allocating perform a blocking
 *    device->host read of a few scalars on `stream` (documented per call).
 *  - Ownership: output handles/arrays are allocated through `al` (NULL = cudaMallocAsync on the
 *    device's default memory pool, whose release threshold the library raises so freed blocks
 *    stay cached).  A handle records its allocator; tsg_tiles_destroy frees through it.
 *  - Errors: every call returns a tsg_status; no C++ exception crosses the ABI and nothing
 *    aborts.  On error the output pointers are set to NULL and all partial allocations are
 *    released.  tsg_last_error() gives a thread-local human-readable detail string.
 *  - Thread safety: distinct handles may be used from distinct threads; one handle must not be
 *    destroyed while another thread uses it.
 */
#ifndef TSG_H_
#define TSG_H_

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define TSG_API __attribute__((visibility("default")))
#else
#define TSG_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

#define TSG_TILE 16          /* tile size, fixed by the paper */
#define TSG_DENSE_NNZ 96     /* t_nnz: dense accumulator iff tile nnz >= 96 (the paper's 192, re-tuned
                                for these kernels on B200: reading A7) */
#define TSG_ABI_VERSION 3

typedef enum {
    TSG_OK = 0,
    TSG_ERR_INVALID_ARG = 1, /* NULL pointer, negative size, bad flag */
    TSG_ERR_SHAPE = 2,       /* A.n != B.m */
    TSG_ERR_UNSORTED = 3,    /* CSR columns not strictly increasing within a row, or out of range */
    TSG_ERR_OVERFLOW = 4,    /* a size exceeds the index width (n >= 2^31, >= 2^31 tiles) */
    TSG_ERR_OOM = 5,         /* device allocation failed */
    TSG_ERR_CUDA = 6,        /* a CUDA runtime error (detail in tsg_last_error) */
    TSG_ERR_INTERNAL = 7     /* an internal consistency check failed */
} tsg_status;

/* Stream-ordered allocator hook.  alloc returns NULL on failure. */
typedef struct {
    void *(*alloc)(size_t bytes, void *stream, void *ctx);
    void (*free)(void *ptr, size_t bytes, void *stream, void *ctx);
    void *ctx;
} tsg_allocator;

/* Opaque, device-resident matrix in sparse-tile form; owns (or borrows) its arrays. */
typedef struct tsg_tiles tsg_tiles;

/* Value types.  The paper's main runs are fp64; its Section 4.7 runs TileSpGEMM
 * with half-precision input and single-precision output.  A product's C type:
 * F64 x F64 -> F64, F32 x F32 -> F32, F16 x F16 -> F32 (accumulated in fp32); any other mix is
 * TSG_ERR_INVALID_ARG.  Steps 1 and 2 do not look at values. */
typedef enum { TSG_F64 = 0, TSG_F32 = 1, TSG_F16 = 2 } tsg_dtype;

/* Read-only view of the Section 3.2 arrays, all device pointers.
 *   tile_ptr [tile_m+1]     int64  offsets of the tiles of each tile row
 *   tile_col [num_tiles]    int32  tile column ids, strictly ascending per row
 *   tile_nnz [num_tiles+1]  int64  offsets of each tile's nonzeros
 *   row_ptr  [16*num_tiles] uint8  local row offsets, 16 per tile, no 17th       (A3)
 *   mask     [16*num_tiles] uint16 bit c of row r <=> nonzero at (r,c)           (A2)
 *   idx      [nnz]          uint8  (r<<4)|c of each nonzero                      (A1)
 *   val      [nnz]          dtype  values in tile order (double/float/half)
 * Every stored tile is non-empty (reading A6). */
typedef struct {
    int64_t m, n, tile_m, tile_n, num_tiles, nnz;
    const int64_t *tile_ptr;
    const int32_t *tile_col;
    const int64_t *tile_nnz;
    const uint8_t *row_ptr;
    const uint16_t *mask;
    const uint8_t *idx;
    const void *val;
    int32_t dtype;            /* tsg_dtype of val */
} tsg_tiles_view;

/* Per-call statistics of tsg_spgemm (all counts exact; times only with TSG_STATS_TIMING).
 * Filling the counts costs one extra blocking read at the end of the call; pass NULL in timed
 * production calls. */
typedef struct {
    int64_t products;         /* sum_i sum_{k in A(i,:)} nnz(B(k,:)) (Table 2 caption P:2531-2538);
                                 -1 unless TSG_STATS_PRODUCTS */
    int64_t tiles_structural; /* |C'| = tiles of the structural tile product A'B' of the paper's step 1, empty
                                 tiles included; -1 unless TSG_STATS_STRUCTURAL */
    int64_t tiles_c;          /* non-empty C tiles (= C.num_tiles) */
    int64_t nnz_c;
    int64_t candidates;       /* tile-pair candidates examined by step 1 */
    int64_t pairs;            /* contributing (A_IK, B_KJ) pairs */
    int64_t tiles_dense;      /* C tiles computed with the dense accumulator */
    int64_t tiles_sparse;
    int64_t kernel_launches;  /* kernels this call launched */
    int32_t step1_list_tiles; /* A tiles that used the B-row-list expansion (mode ii) */
    int32_t host_syncs;       /* blocking device->host scalar reads performed (the stats read excluded) */
    float ms_index, ms_step1, ms_step2, ms_alloc, ms_step3, ms_total; /* CUDA-event times; on the row path
                                 ms_step1 is the plan and ms_step2 the fused step-1 merge + step-2 masks */
    float ms_host_sync, ms_host_alloc; /* host wall time blocked in scalar reads / allocation calls */
    int64_t path;             /* TSG_PATH_ROWS (1): fused per-tile-row kernels (every tile row narrow, and the
                                 call small or A's tiles dense, or TSG_PATH_ROWS_FORCE); TSG_PATH_TILES (0):
                                 the per-C-tile pipeline */
    int64_t step1_big_rows;   /* tile rows whose step 1 ran in global memory (bitmap rank / radix sort) */
    int64_t step1_merge_rows; /* tile rows whose step 1 ran as a warp k-way merge (<= 32 A tiles) */
    int64_t bytes_scratch;    /* device scratch of the call (its peak; f4, cf. Fig 9 peak space P:2938-2968) */
    int64_t bytes_out;        /* device bytes of C's seven arrays (allocation sizes; Fig 11) */
} tsg_stats;

#define TSG_PATH_TILES 0
#define TSG_PATH_ROWS 1

/* flags for tsg_csr_to_tiles */
#define TSG_INPUT_HOST 0x1u     /* row_ptr/col_idx/val are host memory; copied in on `stream` */
#define TSG_VALIDATE 0x2u       /* check row_ptr against nnz (INVALID_ARG) and sorted/unique/in-range columns
                                   (UNSORTED); without it the input is trusted */

/* flags for tsg_spgemm.  None of them changes the result: every combination returns the same C
 * bit for bit (they select work splits, diagnostics and timing only). */
#define TSG_STATS_TIMING 0x1u     /* record per-step CUDA events (read with the stats at the end) */
#define TSG_STATS_STRUCTURAL 0x2u /* also count |C'| into stats->tiles_structural (diagnostic pass over the
                                     structural tile product; tile columns of B <= 1.6e6) */
#define TSG_STEP1_SCAN_ONLY 0x4u  /* force mode (i) tile-row scans in step 1 */
#define TSG_STEP1_LIST_ALWAYS 0x8u/* build B-row lists and use them wherever they are cheaper */
#define TSG_STATS_PRODUCTS 0x10u  /* also count intermediate products into stats->products */
#define TSG_PATH_GENERAL 0x20u    /* use the per-C-tile pipeline even when every tile row is narrow */
#define TSG_STEP1_SORT_ONLY 0x40u /* step 1: no warp merge; every tile row expands + radix-sorts (implies
                                     the per-C-tile pipeline) */
#define TSG_PATH_ROWS_FORCE 0x400u /* take the row path whenever every tile row is narrow (by default only
                                      for small calls or dense-tile-heavy A; TSG_PATH_GENERAL wins) */
#define TSG_SMALL_STAGE_ON 0x100u  /* step 3 small tiles: stage B row metadata by cp.async (default: iff nnz(B) < 4 tiles(B)) */
#define TSG_SMALL_STAGE_OFF 0x200u /* step 3 small tiles: plain dependent loads (same results either way) */
#define TSG_DEBUG_HIGH_OFFSETS 0x800u /* test aid: steps 2-3 address C's nonzeros with offsets
                                        biased by 2^32 (high words set) against base pointers shifted back by
                                        2^32 elements, rebased at the end -- any 32-bit truncation of a
                                        nonzero offset faults or corrupts; same C */
#define TSG_DENSE_THRESHOLD_SHIFT 16 /* bits 16..24: override t_nnz (0 = TSG_DENSE_NNZ; 257 disables dense) */
#define TSG_QUEUE_CHUNK_SHIFT 25     /* bits 25..28: per-C-tile pipeline work distribution, v = 0: automatic,
                                        v = 1: static grid-stride, v >= 2: work queue with v-1 groups per request */
#define TSG_SPGEMM_FLAGS 0x1fff0f7fu /* every defined bit (anything else is INVALID_ARG) */

/*
 * tsg_csr_to_tiles -- CSR -> sparse-tile format (Section 3.2; conversion is timed
 * separately from SpGEMM, reading A14).
 *   m, n          matrix shape (m, n >= 0, n < 2^31)
 *   nnz           number of nonzeros (== row_ptr[m])
 *   row_ptr       int64 [m+1]   CSR row offsets, row_ptr[0] == 0
 *   col_idx       int32 [nnz]   column ids, strictly increasing within a row (reading A12)
 *   val           double [nnz]
 *   flags         TSG_INPUT_HOST | TSG_VALIDATE
 *   out           receives a new handle owning all seven arrays
 * Syncs: one blocking read of the tile count (plus one validation flag with TSG_VALIDATE).
 * Errors: INVALID_ARG, OVERFLOW, UNSORTED (only with TSG_VALIDATE), OOM, CUDA.
 */
TSG_API tsg_status tsg_csr_to_tiles(int64_t m, int64_t n, int64_t nnz, const int64_t *row_ptr,
                            const int32_t *col_idx, const double *val, uint32_t flags,
                            const tsg_allocator *al, void *stream, tsg_tiles **out);

/* tsg_csr_to_tiles_typed -- the same with values of type `dtype` (val: [nnz] double, float or
 * IEEE half; f3).  The handle records the dtype. */
TSG_API tsg_status tsg_csr_to_tiles_typed(int64_t m, int64_t n, int64_t nnz, const int64_t *row_ptr,
                                  const int32_t *col_idx, const void *val, int32_t dtype, uint32_t flags,
                                  const tsg_allocator *al, void *stream, tsg_tiles **out);

/*
 * tsg_spgemm -- C = A*B, both in sparse-tile form; the three steps of Section 3.3
 * (P:880-1888): step 1 tile layout of C, step 2 bit-mask symbolic phase with
 * prefix-sum allocation (Alg 2), step 3 numeric phase with the
 * adaptive sparse/dense accumulator (Alg 3).  The timed region of the paper
 * (steps 1-3 plus all allocation) is this whole call (reading A15).
 *   A, B    input handles (may be the same handle, e.g. C = A^2)
 *   flags   TSG_STATS_* / TSG_STEP1_* / dense-threshold override
 *   C       receives a new handle; C excludes empty tiles (reading A6)
 *   stats   optional (NULL allowed)
 * Values: C(r,j) = sum over pairs in ascending K, over c ascending, of A(r,c)*B(c,j) with
 * fused multiply-add, i.e. ascending global k (reading A8/A16): deterministic run to run.
 * Value types: C's dtype follows tsg_dtype's rules (F16 inputs are widened exactly to fp32 and
 * accumulated with fp32 FMA); mixed input dtypes are INVALID_ARG.
 * Syncs: 2 blocking scalar reads (through mapped host memory), the paper's allocation points
 * (P:982-988): after step 1 (C's tile count, with the step-1 candidate total) and after step 2
 * (nnz(C)).  Step 1's scratch is reserved from the calling thread's cached workspace before its
 * size is known; when it does not fit (the first call of a larger problem) the call is redone
 * once with the workspace grown (+1 read).  With a caller allocator (no workspace) the candidate
 * total is read first (+1).  One more read at the end when `stats` is non-NULL (not counted).
 * Alignment: mask and row_ptr of A and B must be 16-byte aligned, val 8-byte aligned (tiles are
 * staged into shared memory in 16-byte chunks); handles made by this library always are.
 * Errors: INVALID_ARG (incl. alignment), SHAPE, OVERFLOW, OOM, CUDA, INTERNAL.
 */
TSG_API tsg_status tsg_spgemm(const tsg_tiles *A, const tsg_tiles *B, uint32_t flags,
                      const tsg_allocator *al, void *stream, tsg_tiles **C, tsg_stats *stats);

/*
 * tsg_tiles_to_csr -- sparse tiles -> CSR (inverse of tsg_csr_to_tiles; used for checking,
 * P:4637-4639).  Outputs are new device arrays allocated through `al` (free them with
 * tsg_free using the same allocator):  row_ptr int64 [m+1], col_idx int32 [nnz],
 * val [nnz] of T's dtype; *nnz receives nnz.  Syncs: none beyond reading the handle's own sizes.
 */
TSG_API tsg_status tsg_tiles_to_csr(const tsg_tiles *T, const tsg_allocator *al, void *stream,
                            int64_t **row_ptr, int32_t **col_idx, void **val, int64_t *nnz);

/*
 * tsg_tiles_transpose -- A^T in sparse-tile form, for the paper's second workload C = A*A^T
 * (SURVEY §8(f) f1): tile (I, J) becomes tile (J, I) with its pattern and
 * values transposed.  Exact (a permutation of T's data); stream-ordered on `stream`, no host sync.
 *   T       input handle (borrowed; m < 2^31 so that A^T's column ids fit int32)
 *   al      allocator for the result's arrays (NULL = cudaMallocAsync)
 *   out     receives a new handle (destroy with tsg_tiles_destroy)
 * Errors: INVALID_ARG (NULL, unaligned mask), OVERFLOW, OOM, CUDA.
 */
TSG_API tsg_status tsg_tiles_transpose(const tsg_tiles *T, const tsg_allocator *al, void *stream, tsg_tiles **out);

/*
 * tsg_partition_tile_rows -- product-balanced split of C's tile rows for the multi-GPU path
 * (the paper itself runs on one GPU).  Computes on the device the
 * intermediate products of every tile row of A*B (Table 2's "products") and cuts
 * [0, tile_m) into `parts` contiguous ranges at equal shares of their prefix sum: cuts[g] is the
 * first tile row whose prefix reaches g * total / parts (monotone; cuts[0] = 0, cuts[parts] =
 * A.tile_m).  Rank g then computes C's tile rows [cuts[g], cuts[g+1]) from
 * tsg_tiles_slice_rows(A, cuts[g], cuts[g+1]) and all of B.
 *   A, B      the operands (device handles; A.n == B.m)
 *   parts     1..500
 *   cuts      HOST array of parts + 1 int64 (written)
 *   products  optional HOST int64: the total intermediate products of A*B
 * Syncs: one blocking read (the cuts).  Errors: INVALID_ARG, SHAPE, OOM, CUDA.
 */
TSG_API tsg_status tsg_partition_tile_rows(const tsg_tiles *A, const tsg_tiles *B, int64_t parts, void *stream,
                                           int64_t *cuts, int64_t *products);

/* Fill *out with the handle's arrays and sizes (pointers stay owned by the handle). */
TSG_API tsg_status tsg_tiles_get_view(const tsg_tiles *T, tsg_tiles_view *out);

/*
 * tsg_tiles_wrap -- make a handle over existing device arrays described by *v (e.g. arrays
 * gathered from other ranks).  owner == NULL: the handle borrows them (destroy frees only the
 * handle's own helper state).  owner != NULL: the handle takes ownership and frees each array
 * through owner->free.  The arrays must satisfy the Section 3.2 invariants (not re-checked).
 */
TSG_API tsg_status tsg_tiles_wrap(const tsg_tiles_view *v, const tsg_allocator *owner, tsg_tiles **out);

/*
 * tsg_tiles_slice_rows -- zero-copy view of tile rows [tile_row_begin, tile_row_end) of T as
 * a (rows x T.n) matrix (rows = 16*(end-begin), clipped to T.m).  The view borrows T's arrays
 * and owns a rebased copy of tile_ptr/tile_nnz (2 small kernels on `stream`); T must outlive
 * it.  Used to give each rank its A shard when B = A.
 */
TSG_API tsg_status tsg_tiles_slice_rows(const tsg_tiles *T, int64_t tile_row_begin, int64_t tile_row_end,
                                void *stream, tsg_tiles **view);

/*
 * tsg_tiles_copy_to_host -- copy the seven arrays into caller-provided HOST buffers (pinned
 * for speed), sized from tsg_tiles_get_view (val: nnz elements of the view's dtype); NULL skips
 * an array.  Blocks until done.
 */
TSG_API tsg_status tsg_tiles_copy_to_host(const tsg_tiles *T, void *stream, int64_t *tile_ptr,
                                  int32_t *tile_col, int64_t *tile_nnz, uint8_t *row_ptr,
                                  uint16_t *mask, uint8_t *idx, void *val);

/*
 * tsg_tiles_copy_to_host_async -- the same copies, stream-ordered and non-blocking: the host
 * buffers hold the result once `stream` has passed the call (the caller synchronizes, e.g. on an
 * event), and T must stay alive until then.  Lets a caller overlap the copy of one result with
 * the computation of the next (row blocks on two streams).  Host buffers should be pinned
 * (pageable memory makes the copies synchronous).
 */
TSG_API tsg_status tsg_tiles_copy_to_host_async(const tsg_tiles *T, void *stream, int64_t *tile_ptr,
                                        int32_t *tile_col, int64_t *tile_nnz, uint8_t *row_ptr,
                                        uint16_t *mask, uint8_t *idx, void *val);

/* Release a handle (stream-ordered frees through its allocator).  NULL is a no-op. */
TSG_API void tsg_tiles_destroy(tsg_tiles *T, void *stream);

/* Free an array returned by tsg_tiles_to_csr (same allocator; NULL al = cudaFreeAsync). */
TSG_API void tsg_free(void *ptr, size_t bytes, const tsg_allocator *al, void *stream);

/* Scratch workspace: with no user allocator, the temporary arrays of a call (step-1 pairs,
 * occupancy words, scans, ...) come from a per-thread, per-device cached arena that grows to the
 * largest call seen and is reused (so repeated calls do no device allocation besides C's arrays).
 * This releases the calling thread's arena on the current device (stream-ordered on `stream`).
 * Returns the bytes it held. */
TSG_API size_t tsg_workspace_release(void *stream);

TSG_API const char *tsg_status_string(tsg_status s);
TSG_API const char *tsg_last_error(void);
TSG_API int tsg_abi_version(void);

/* Number of kernels launched by this process through the library so far (evidence counter). */
TSG_API int64_t tsg_kernel_launch_count(void);

#ifdef __cplusplus
}
#endif
#endif /* TSG_H_ */
