// tsg_kernels.cuh -- parameter blocks and host launchers shared by the step translation units
// (tsg_step1.cu: a0/a1, tsg_step23.cu: a2/a4) and the orchestration in tsg_spgemm.cu.
#pragma once

#include "tsg_internal.cuh"

namespace tsg {

typedef unsigned long long u64c;

// device-side counters of one tsg_spgemm call (zeroed at the start)
struct DevCounters {
    u64c max_u_small;  // largest candidate count among shared-memory rows
    u64c nbig;         // rows sorted in global memory
    u64c big_u;        // their total candidate count
    u64c list_tiles;   // A tiles expanded through B row lists
    u64c pairs;        // contributing pairs
    u64c products;     // intermediate products (stats only)
    u64c n2light;      // step-2 class sizes
    u64c n2heavy;
    u64c n3small;      // step-3 class sizes
    u64c n3medium;
    u64c n3dense;
    u64c nmerge;       // tile rows of step 1 handled by the warp k-way merge
    u64c n2dense;      // C tiles with nnz >= t_nnz (step 2 counts them; step 3 launches the dense kernel iff > 0)
    u64c max_a_dense;  // row path: most A tiles in a tile row with dense C tiles
    u64c structural;   // |C'| (TSG_STATS_STRUCTURAL)
    u64c nsmall;       // rows sorted in shared memory (their list: smallList)
    u64c overflow;     // step 1's candidate scratch was too small (the call is redone with a larger arena)
    u64c next_small, next_big;  // work counters of the persistent step-1 kernels
    u64c q[5][16];     // work-queue counters of the step-2/3 kernels, one 128-byte line each
};

constexpr int ROW_T = 256;        // threads of a step-1 row CTA
constexpr int ROW_NW = ROW_T / 32;
#ifndef TSG_ROW_CAP
#define TSG_ROW_CAP 256
#endif
// max candidates of a wide row (> 32 A tiles) sorted in shared memory (k_row_small); wider rows take
// the bitmap rank.  Measured on C4 (25 K such rows, 52 M candidates): 4096 -> 92.1 ms per call,
// 1024 -> 91.0, 256 -> 90.8 (the rank kernel's two 1024-thread CTAs per SM beat the sort's
// 61 ps per candidate)
constexpr int ROW_CAP = TSG_ROW_CAP;
constexpr int LIGHT_WORK = 16;    // step-2 thread-per-tile class: (pair, c) items of the tile
constexpr int SMALL_NNZ = 8;      // step-3 lane-per-entry class (k_s3_small): C tile nnz (<= 16)
constexpr int64_t ROWPATH_SMALL_U = 1 << 20;  // step-1 candidates below which narrow calls take the row path
constexpr int MERGE_MAX_A = 32;   // step-1 warp-merge class: A tiles of the tile row (one lane each)

// ---------------- a0 for hypersparse operands: one 16-byte record per tile.
// A single-nonzero tile carries its entry and its value inline, so a pair of such tiles costs two
// 16-byte loads in steps 2-3 instead of a sector each for mask, transposed mask, row offsets, value
// offset and value (R-MAT tiles average 1.05 nonzeros).  As four 32-bit words:
//   x, y  single: the value's bits (its dtype, low bytes first); else: the tile's nonzero offset
//   z     tile column
//   w     bits 0-15 row occupancy, 16-23 (r << 4) | c of the single nonzero, bit 24 single
struct alignas(16) TileRec {
    uint64_t v;
    int32_t col;
    uint32_t w;
};
static_assert(sizeof(TileRec) == 16, "one 16-byte load per tile");
void launch_tile_records(int64_t nt, const int32_t *tile_col, const int64_t *tile_nnz, const uint16_t *mask,
                         const uint8_t *idx, const void *val, int32_t dtype, TileRec *rec, cudaStream_t s);

// ---------------- a1 row sort
struct S1Params {
    const int64_t *tpA;
    const int64_t *tnzA;      // A tile_nnz (for the per-C-tile work estimate)
    const uint16_t *colOccA;
    const int64_t *costOff;
    const int64_t *startA;
    const int32_t *tcB;
    const uint16_t *rowOccB;
    const uint32_t *list;
    const int32_t *listJ;     // tile column of each B row list entry (list mode)
    const int32_t *rowJlo;
    const int32_t *rowJhi;
    const uint8_t *rowClass;
    int64_t tnB;       // tile columns of B (the merge packs a tile column into 27 bits)
    int sort_only;     // TSG_STEP1_SORT_ONLY: wide rows use the global radix sort, not the bitmap rank
    uint64_t *pairs;   // [Utot]  (posA << 32) | posB, at costOff[a0] + i
    int32_t *tJ;       // [Utot]  C tile column of rank r, at costOff[a0] + r
    uint32_t *tStart;  // [Utot]  first pair (row-relative)
    uint32_t *tCnt;    // [Utot]  pair count
    uint32_t *tWork;   // [Utot]  (pair, c) items: sum over pairs of popc(colOcc(A) & rowOcc(B))
    int64_t *nC;       // [tm]    C tiles of the row
    const int32_t *bigList;
    const int64_t *bigOff;
    const int32_t *smallList;
    const int64_t *utot;   // the candidate total (costOff[ntA]), read on the device
    int64_t capU, capBig;  // capacity of the candidate-space and wide-row scratch (elements)
    uint64_t *bigKeysA, *bigKeysB;
    uint32_t *bigPosB, *bigKpos;
    DevCounters *cnt;
    // the row path's fused step 2 (k_sym_rows): masks and row offsets of each C tile at its
    // candidate-space slot, tile nnz in tWork, the row's nnz total
    const uint16_t *mA, *mB;
    uint16_t *sMaskC;   // [16 Utot]
    uint8_t *sRowPtrC;  // [16 Utot]
    int64_t *rowNnz;    // [tm]
    int dense_threshold;  // counts the dense C tiles into cnt->n2dense
};

// ---------------- compaction of step-1 results into per-C-tile arrays + step-2 classes
struct CompactParams {
    int64_t tm;
    const int64_t *tpA;
    const int64_t *costOff;
    const int64_t *tilePtrC;
    const int32_t *tJ;
    const uint32_t *tStart;
    const uint32_t *tCnt;
    const uint32_t *tWork;
    int32_t *tile_col;
    int64_t *pairBeg;
    uint32_t *pairCnt;
    uint32_t *work;   // (pair, c) items per C tile: the step-2 class split
};

// ---------------- a2 step 2 and a4 step 3: warps take groups of 32 consecutive C tiles
struct StepParams {
    int64_t ntC;
    const int64_t *pairBeg;
    const uint32_t *pairCnt;
    const uint64_t *pairs;
    // A
    const int64_t *tnzA;
    const uint8_t *rpA;
    const uint16_t *mA;
    const uint16_t *mTA;      // transposed masks
    const uint16_t *colOccA;
    const uint8_t *ixA;
    const void *vA;           // values: dtype_in (double / float / half)
    // B
    const int64_t *tnzB;
    const uint8_t *rpB;
    const uint16_t *mB;
    const uint16_t *rowOccB;
    const uint16_t *mTB;      // transposed masks (column j of B_KJ: bit c <=> B(c,j) != 0)
    const uint8_t *ixB;
    const void *vB;
    // C
    int64_t *tnzC;   // step 2: per-tile nnz; step 3: offsets
    uint8_t *rpC;
    uint16_t *mC;
    uint8_t *ixC;
    void *vC;              // values: double for F64 inputs, float for F32 and F16 inputs
    int dtype_in;          // tsg_dtype of A and B
    const uint32_t *work;  // step-2 class split
    // step-3 classes per group of 32 C tiles (bit i = tile 32g+i), written by step 2: medium / dense
    // tiles among the light tiles (k_s2_light) and among the heavy tiles (k_s2)
    uint32_t *medL, *medH, *denL, *denH;
    int qchunk[5];         // work-queue units per request (k_s2_light, k_s2, k_s3_small, k_s3, k_s3_dense)
    int qoverride;         // work distribution override (-1 automatic, 0 static, k > 0 queue chunk k)
    int dense_threshold;
    int small_max;         // step 3: tiles with nnz <= small_max take the lane-per-entry path
    int small_stage;       // step 3: k_s3_small stages B row metadata with cp.async (hypersparse B)
    const TileRec *recA, *recB;  // hypersparse operands: per-tile records (else nullptr)
    int64_t recA_voff;     // added to A records' value offsets (A a row slice inside B: B's offsets)
    DevCounters *cnt;
};

// launchers (tsg_step1.cu)
void launch_occupancy(const uint16_t *mask, int64_t nt, uint16_t *row_occ, uint16_t *col_occ, cudaStream_t s,
                      void *zero = nullptr, size_t zero_bytes = 0);  // also zeroes `zero` (the call's counters)
void launch_rowlist(int64_t tmB, const int64_t *tpB, const uint16_t *maskB, const int64_t *lptr, int32_t *lcnt,
                    uint32_t *list, const int32_t *tcB, int32_t *listJ, cudaStream_t s);
void launch_products(int64_t tmB, const int64_t *tpB, const uint16_t *maskB, int64_t ntA, const int32_t *tcA,
                     const uint16_t *maskA, int32_t *rnnz, DevCounters *cnt, cudaStream_t s);
void launch_atile_plan(int64_t ntA, const int32_t *tcA, const uint16_t *colOccA, const int64_t *tpB,
                       const int32_t *tcB, const int64_t *lptr, const uint32_t *list, const int32_t *listJ,
                       bool scan_only, int64_t *cost, int64_t *start, int32_t *jlo, int32_t *jhi, DevCounters *cnt,
                       cudaStream_t s);
void launch_row_plan(int64_t tmA, const int64_t *tpA, const int64_t *costOff, const int32_t *jloA,
                     const int32_t *jhiA, bool merge, int32_t *rowJlo, int32_t *rowJhi, uint8_t *rowClass,
                     int64_t *nC, int32_t *bigList, int64_t *bigOff, int32_t *smallList, DevCounters *cnt,
                     cudaStream_t s);
// step 1 of the per-C-tile path; the row-class counts are read on the device (persistent grids
// over the class lists), so no host read is needed before it
void launch_row_sort(const S1Params &P, int64_t tm, cudaStream_t s);
void launch_sym_rows(const S1Params &P, int64_t tm, cudaStream_t s);
void launch_row_products(int64_t tmA, const int64_t *tpA, const int32_t *tcA, const uint16_t *maskA, int64_t tmB,
                         const int64_t *tpB, const uint16_t *maskB, int32_t *rnnz, int64_t *w, cudaStream_t s);
void launch_cuts(const int64_t *pre, int64_t tm, int64_t parts, int64_t *cuts, cudaStream_t s);
bool launch_structural(int64_t tmA, const int64_t *tpA, const int32_t *tcA, const int64_t *tpB, const int32_t *tcB,
                       int64_t tnB, DevCounters *cnt, cudaStream_t s);
void launch_transpose(const uint16_t *mask, int64_t nt, uint16_t *maskT, cudaStream_t s);
void launch_compact(const CompactParams &P, int64_t ntC, cudaStream_t s);

// ---------------- a4 on the row path (tsg_rows.cu)
struct RowNumArgs {
    int64_t tm, ntC;
    const tsg_tiles *A, *B;
    tsg_tiles *C;                 // tile_ptr filled; the other arrays allocated
    const uint16_t *mTB, *rowOccB;
    const int64_t *costOff;
    const uint64_t *pairs;
    const int32_t *tJ;
    const uint32_t *tStart, *tCnt, *tNnz;
    const uint16_t *sMaskC;
    const uint8_t *sRowPtrC;
    const int64_t *rowOff;        // [tm+1] exclusive scan of the rows' nnz
    int dense_threshold, small_max;
    int64_t n_dense;              // dense C tiles (counted by k_sym_rows)
    int max_a_dense;              // most A tiles in a tile row with dense C tiles (k_sym_rows)
    const uint16_t *colOccA;      // column occupancy words of A's tiles
    void *small;                  // scratch for the small C tiles' records (32 B each, <= ntC)
    DevCounters *cnt;
};
constexpr int ROW_REC_BYTES = 32;
// k_num_rows / k_num_small on `s`; the dense class (independent of them) on `sd`
void launch_num_rows(const RowNumArgs &a, cudaStream_t s, cudaStream_t sd);

// launchers (tsg_step23.cu)
void launch_step2(const StepParams &P, cudaStream_t s);
void launch_step3(const StepParams &P, int64_t n_dense, cudaStream_t s);

}  // namespace tsg
