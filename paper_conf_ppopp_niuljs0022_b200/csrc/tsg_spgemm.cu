// tsg_spgemm.cu -- host orchestration of one tsg_spgemm call: the three steps of TileSpGEMM
// (Section 3.3) with the device prefix sums and the allocation between them.
//
//   a0  helper indices (tsg_step1.cu): occupancy words, transposed masks, optional B row lists
//   a1  plan: candidate count per A tile, prefix sum, per-row class       -> blocking read #1
//   Row path (every non-empty tile row has <= 32 A tiles: stencils, FEM, banded):
//     a1+a2  k_sym_rows: per tile row, the exact C tile set + pairs (warp merge) and each C
//            tile's masks / row offsets / nnz, at the row's candidate-space slots
//     a3     prefix sums of the rows' tile counts and nnz                -> blocking read #2
//            (C's tile count and nnz together), then C is allocated once
//     a4     k_num_rows: per tile row, C's tile records copied into place + the numeric phase
//   Per-C-tile path (wide tile rows: power-law graphs, hubs):
//     a1     merge / shared-memory sort / bitmap rank per row class; scan -> read #2 (tile count)
//     a2     k_s2_light / k_s2 per group of 32 C tiles; scan of tile nnz -> read #3 (nnz(C))
//     a4     k_s3_small / k_s3 / k_s3_dense per group of 32 C tiles
// Both paths give the same C bit for bit (tests/test_gpu_parity.py).
#include <algorithm>
#include <cstdlib>
#include <cstring>

#include <nvtx3/nvToolsExt.h>

#include "tsg_kernels.cuh"

namespace tsg {
namespace {
// NVTX ranges per step (one range per step of the method, visible in Nsight Systems /
// ncu --nvtx; header-only NVTX3, a no-op without an attached tool)
struct Range {
    bool on = false;
    void push(const char *name) {
        pop();
        nvtxRangePushA(name);
        on = true;
    }
    void pop() {
        if (on) nvtxRangePop();
        on = false;
    }
    ~Range() { pop(); }
};

struct Timer {
    bool on = false;
    cudaStream_t s{};
    cudaEvent_t ev[8]{};
    void init(bool enable, cudaStream_t st) {
        on = enable;
        s = st;
        if (on)
            for (auto &e : ev) TSG_CUDA(cudaEventCreate(&e));
    }
    void mark(int i) {
        if (on) TSG_CUDA(cudaEventRecord(ev[i], s));
    }
    float ms(int a, int b) {
        float x = 0.f;
        if (on) cudaEventElapsedTime(&x, ev[a], ev[b]);
        return x;
    }
    ~Timer() {
        if (on)
            for (auto &e : ev) cudaEventDestroy(e);
    }
};

// A side stream forked from `s` (one cached non-blocking stream and two events per host thread
// and device); join() makes `s` wait for the side work, and the destructor joins if nothing did
class SideStream {
   public:
    explicit SideStream(cudaStream_t s) : s_(s) {
        int dev = 0;
        cudaGetDevice(&dev);
        static thread_local Res res[16];
        r_ = &res[dev & 15];
        if (!r_->side) {
            TSG_CUDA(cudaStreamCreateWithFlags(&r_->side, cudaStreamNonBlocking));
            TSG_CUDA(cudaEventCreateWithFlags(&r_->fork, cudaEventDisableTiming));
            TSG_CUDA(cudaEventCreateWithFlags(&r_->joinev, cudaEventDisableTiming));
        }
        TSG_CUDA(cudaEventRecord(r_->fork, s_));
        TSG_CUDA(cudaStreamWaitEvent(r_->side, r_->fork, 0));
    }
    cudaStream_t stream() const { return r_->side; }
    void done() {
        TSG_CUDA(cudaEventRecord(r_->joinev, r_->side));
        recorded_ = true;
    }
    void join() {
        if (joined_) return;
        if (!recorded_) done();
        TSG_CUDA(cudaStreamWaitEvent(s_, r_->joinev, 0));
        joined_ = true;
    }
    ~SideStream() {
        if (joined_) return;
        if (!recorded_) cudaEventRecord(r_->joinev, r_->side);
        cudaStreamWaitEvent(s_, r_->joinev, 0);
    }

   private:
    struct Res {
        cudaStream_t side = nullptr;
        cudaEvent_t fork = nullptr, joinev = nullptr;
    };
    cudaStream_t s_;
    Res *r_;
    bool recorded_ = false, joined_ = false;
};
}  // namespace

void run_spgemm(const tsg_tiles *A, const tsg_tiles *B, uint32_t flags, const Allocator &al, cudaStream_t s,
                tsg_tiles *C, tsg_stats *st) {
    reset_call_launches();
    TSG_REQUIRE((flags & ~(uint32_t)TSG_SPGEMM_FLAGS) == 0, TSG_ERR_INVALID_ARG, "unknown tsg_spgemm flag");
    TSG_REQUIRE(A->nt < ((int64_t)1 << 31) && B->nt < ((int64_t)1 << 31), TSG_ERR_OVERFLOW, "input has >= 2^31 tiles");
    TSG_REQUIRE(A->tn == B->tm, TSG_ERR_SHAPE, "tile shapes disagree");
    TSG_REQUIRE(A->dtype == B->dtype, TSG_ERR_INVALID_ARG, "A and B value types differ");
    const int32_t dtC = A->dtype == TSG_F64 ? TSG_F64 : TSG_F32;  // F16 x F16 -> F32
    TSG_REQUIRE(((uintptr_t)A->mask & 15) == 0 && ((uintptr_t)B->mask & 15) == 0 && ((uintptr_t)A->row_ptr & 15) == 0 &&
                    ((uintptr_t)B->row_ptr & 15) == 0 && ((uintptr_t)A->val % A->vsize()) == 0 && ((uintptr_t)B->val % B->vsize()) == 0,
                TSG_ERR_INVALID_ARG, "mask and row_ptr arrays must be 16-byte aligned, val aligned to its type");
    int TH = (int)((flags >> TSG_DENSE_THRESHOLD_SHIFT) & 0x1ffu);
    if (TH == 0) TH = TSG_DENSE_NNZ;
    TSG_REQUIRE(TH <= 257, TSG_ERR_INVALID_ARG, "dense threshold > 257");
    const int qv = (int)((flags >> TSG_QUEUE_CHUNK_SHIFT) & 0xfu);
    // TSG_DEBUG_HIGH_OFFSETS: C's nonzero offsets carry +2^32 during step 3 (against shifted bases)
    const int64_t bias = (flags & TSG_DEBUG_HIGH_OFFSETS) ? ((int64_t)1 << 32) : 0;
    Timer tm_;
    tm_.init((flags & TSG_STATS_TIMING) && st, s);
    tm_.mark(0);

    Range nv;
    nv.push("tsg a0 helper indices");
    Buffers tmp(al, s, true), out(al, s);
    const int64_t ntA = A->nt, tmA = A->tm, tmB = B->tm;
    int syncs = 0;
    DevCounters *cnt = tmp.get<DevCounters>(1);  // zeroed by the first occupancy launch
    static_assert(sizeof(DevCounters) % 8 == 0, "counters are zeroed as 64-bit words");

    // ---------------- a0: occupancy words, optional B row lists, optional product count
    // A inside B's tile arrays (A^2, or a row slice of B: SURVEY 8(e)'s rank shards and row blocks):
    // A's tile t is B's tile t + off, so one pass over B gives A's helper words too
    const int64_t off = (int64_t)(A->mask - B->mask) / TILE;
    const bool inB = A->mask >= B->mask && (A->mask - B->mask) % TILE == 0 && off + ntA <= B->nt;
    uint16_t *rowOccB = tmp.get<uint16_t>(B->nt);
    uint16_t *colOccA;
    if (inB) {
        uint16_t *colOccB = tmp.get<uint16_t>(B->nt);
        launch_occupancy(B->mask, B->nt, rowOccB, colOccB, s, cnt, sizeof(DevCounters));
        colOccA = colOccB + off;
    } else {
        colOccA = tmp.get<uint16_t>(ntA);
        launch_occupancy(A->mask, ntA, nullptr, colOccA, s, cnt, sizeof(DevCounters));
        launch_occupancy(B->mask, B->nt, rowOccB, nullptr, s);
    }
    // transposed masks: first used by step 2 / 3, so they are computed on a side stream while
    // step 1 runs (joined before their first use, and on every exit path by the guard's destructor)
    uint16_t *mTB = tmp.get<uint16_t>(TILE * B->nt);
    uint16_t *mTA = inB ? mTB + TILE * off : tmp.get<uint16_t>(TILE * ntA);
    SideStream side(s);
    launch_transpose(B->mask, B->nt, mTB, side.stream());
    if (!inB) launch_transpose(A->mask, ntA, mTA, side.stream());
    side.done();
    const bool lists = !(flags & TSG_STEP1_SCAN_ONLY) &&
                       ((flags & TSG_STEP1_LIST_ALWAYS) || (B->nt > 0 && B->nnz < 2 * B->nt));
    int64_t *lptr = nullptr;
    uint32_t *list = nullptr;
    int32_t *listJ = nullptr;
    if (lists) {
        int32_t *lcnt = tmp.get<int32_t>(TILE * tmB);
        lptr = tmp.get<int64_t>(TILE * tmB + 1);
        list = tmp.get<uint32_t>(B->nnz);
        listJ = tmp.get<int32_t>(B->nnz);
        launch_rowlist(tmB, B->tile_ptr, B->mask, nullptr, lcnt, nullptr, nullptr, nullptr, s);
        exclusive_scan<int32_t>(lcnt, lptr, TILE * tmB, s, tmp);
        launch_rowlist(tmB, B->tile_ptr, B->mask, lptr, lcnt, list, B->tile_col, listJ, s);
    }
    // hypersparse operands (fewer than 4 nonzeros per B tile, no small-tile flag): 16-byte per-tile
    // records for step 1's wide rows and steps 2-3 (inB: A's are a slice of B's)
    TileRec *recA = nullptr, *recB = nullptr;
    if (!(flags & (TSG_SMALL_STAGE_ON | TSG_SMALL_STAGE_OFF)) && B->nt > 0 && B->nnz < 4 * B->nt) {
        recB = tmp.get<TileRec>(B->nt);
        launch_tile_records(B->nt, B->tile_col, B->tile_nnz, B->mask, B->idx, B->val, B->dtype, recB, s);
        // A's records are a slice of B's only if A's arrays are B's, shifted (a row slice of B):
        // the records carry values, so sharing masks alone is not enough
        const int64_t dz = (int64_t)(A->idx - B->idx);
        const bool slice = inB && A->tile_col == B->tile_col + off && dz >= 0 &&
                           static_cast<const uint8_t *>(A->val) ==
                               static_cast<const uint8_t *>(B->val) + dz * (int64_t)A->vsize();
        if (slice) {
            recA = recB + off;
        } else {
            recA = tmp.get<TileRec>(std::max<int64_t>(ntA, 1));
            launch_tile_records(ntA, A->tile_col, A->tile_nnz, A->mask, A->idx, A->val, A->dtype, recA, s);
        }
    }
    if (st && (flags & TSG_STATS_PRODUCTS)) {
        int32_t *rnnz = tmp.get<int32_t>(TILE * tmB);
        launch_products(tmB, B->tile_ptr, B->mask, ntA, A->tile_col, A->mask, rnnz, cnt, s);
    }
    bool structural = false;
    if (st && (flags & TSG_STATS_STRUCTURAL) && tmA > 0)
        structural = launch_structural(tmA, A->tile_ptr, A->tile_col, B->tile_ptr, B->tile_col, B->tn, cnt, s);
    tm_.mark(1);

    // ---------------- a1: plan
    nv.push("tsg a1 plan");
    int64_t *cost = tmp.get<int64_t>(ntA);
    int64_t *startA = tmp.get<int64_t>(ntA);
    int32_t *jloA = tmp.get<int32_t>(ntA);
    int32_t *jhiA = tmp.get<int32_t>(ntA);
    launch_atile_plan(ntA, A->tile_col, colOccA, B->tile_ptr, B->tile_col, lptr, list, listJ,
                      (bool)(flags & TSG_STEP1_SCAN_ONLY), cost, startA, jloA, jhiA, cnt, s);
    int64_t *costOff = tmp.get<int64_t>(ntA + 1);
    exclusive_scan<int64_t>(cost, costOff, ntA, s, tmp);
    int32_t *rowJlo = tmp.get<int32_t>(tmA);
    int32_t *rowJhi = tmp.get<int32_t>(tmA);
    uint8_t *rowClass = tmp.get<uint8_t>(tmA);
    int64_t *nC = tmp.get<int64_t>(tmA + 1);
    int32_t *bigList = tmp.get<int32_t>(tmA);
    int64_t *bigOff = tmp.get<int64_t>(tmA);
    int32_t *smallList = tmp.get<int32_t>(tmA);
    launch_row_plan(tmA, A->tile_ptr, costOff, jloA, jhiA, !(flags & TSG_STEP1_SORT_ONLY), rowJlo, rowJhi, rowClass,
                    nC, bigList, bigOff, smallList, cnt, s);
    tm_.mark(2);

    // ---------------- a1: step 1 (both paths): exact C tile layout + pairs, per row class
    // Its scratch (24 B per candidate in the candidate space, 24 B per candidate of the wide rows)
    // is sized from the free part of the call's cached arena: the candidate total is only read
    // with C's tile count afterwards (the paper's allocation points, are the two
    // reads).  The kernels check the true total on the device; if it did not fit -- the first
    // call of a larger problem -- the call is redone with the arena grown to the need.  A caller
    // allocator (no arena) reads the total first instead (one more blocking read).
    nv.push("tsg a1 step 1: tile layout + pairs");
    S1Params P1{};
    P1.tpA = A->tile_ptr;
    P1.tnzA = A->tile_nnz;
    P1.colOccA = colOccA;
    P1.costOff = costOff;
    P1.startA = startA;
    P1.tcB = B->tile_col;
    P1.rowOccB = rowOccB;
    P1.list = list;
    P1.listJ = listJ;
    P1.rowJlo = rowJlo;
    P1.rowJhi = rowJhi;
    P1.rowClass = rowClass;
    P1.tnB = B->tn;
    P1.sort_only = (flags & TSG_STEP1_SORT_ONLY) ? 1 : 0;
    P1.utot = costOff + ntA;
    int64_t capU;
    if (tmp.arena_backed()) {
        // reserve for the largest candidate total seen (not all of the free arena: the rest of
        // the call draws from it too)
        const size_t slack = 16 * 256;  // alignment of the nine arrays
        const size_t freeb = tmp.arena_free();
        const int64_t fit = freeb > slack ? (int64_t)((freeb - slack) / 48) : 0;
        capU = std::min<int64_t>(fit, std::max<int64_t>(*tmp.arena_hint(), 1 << 16));
    } else {
        int64_t u = 0;
        read_device({{&u, costOff + ntA, sizeof(int64_t)}}, s);
        syncs++;
        capU = u;
    }
    capU = std::max<int64_t>(capU, 1);
    P1.capU = P1.capBig = capU;
    P1.pairs = tmp.get<uint64_t>(capU);
    P1.tJ = tmp.get<int32_t>(capU);
    P1.tStart = tmp.get<uint32_t>(capU);
    P1.tCnt = tmp.get<uint32_t>(capU);
    P1.tWork = tmp.get<uint32_t>(capU);
    P1.bigKeysA = tmp.get<uint64_t>(capU);
    P1.bigKeysB = tmp.get<uint64_t>(capU);
    P1.bigPosB = tmp.get<uint32_t>(capU);
    P1.bigKpos = tmp.get<uint32_t>(capU);
    P1.nC = nC;
    P1.bigList = bigList;
    P1.bigOff = bigOff;
    P1.smallList = smallList;
    P1.cnt = cnt;
    P1.mA = A->mask;
    P1.mB = B->mask;
    launch_row_sort(P1, tmA, s);
    int64_t *tile_ptr = out.get<int64_t>(tmA + 1);
    // blocking read #1: C's tile count, the candidate total, the row classes (exported by the scan)
    DevCounters hc{};
    int64_t Utot = 0, ntC = 0, nnzC = 0;
    {
        const std::initializer_list<DevRead> segs = {{&ntC, tile_ptr + tmA, sizeof(int64_t)},
                                                     {&Utot, costOff + ntA, sizeof(int64_t)},
                                                     {&hc, cnt, sizeof(DevCounters)}};
        const ExportArgs ex = begin_read(segs);
        exclusive_scan<int64_t>(nC, tile_ptr, tmA, s, tmp, &ex);
        finish_read(ex, segs, s);
    }
    syncs++;
    TSG_REQUIRE(Utot < ((int64_t)1 << 40), TSG_ERR_OVERFLOW, "too many step-1 candidates");
    if (hc.overflow) {
        const int64_t need = (int64_t)std::max<u64c>((u64c)Utot, hc.big_u);
        *tmp.arena_hint() = std::max(*tmp.arena_hint(), need);
        tmp.arena_need((size_t)48 * (size_t)need + ((size_t)1 << 20));
        throw Retry{};
    }
    if (tmp.arena_backed()) *tmp.arena_hint() = std::max(*tmp.arena_hint(), Utot);
    TSG_REQUIRE(ntC < ((int64_t)1 << 32), TSG_ERR_OVERFLOW, "C has >= 2^32 tiles");
    tm_.mark(3);

    // the row path needs every non-empty tile row to be a merge row (<= 32 A tiles).  It wins where
    // the call is small (fewer launches: C1) or A's tiles are dense enough to make dense C tiles
    // common (C3: 0.89 vs 1.0 ms); on sparse-tile stencils (C2: 17 nnz per A tile) the per-C-tile
    // kernels run at higher occupancy and are faster
    const bool narrow = !(flags & (TSG_PATH_GENERAL | TSG_STEP1_SORT_ONLY)) && hc.nbig == 0 && hc.max_u_small == 0 &&
                        tmA > 0;
    const bool rowpath = narrow && ((flags & TSG_PATH_ROWS_FORCE) || A->nnz >= 32 * A->nt || Utot <= ROWPATH_SMALL_U);
    if (rowpath) {
        P1.sMaskC = tmp.get<uint16_t>(TILE * Utot);
        P1.sRowPtrC = tmp.get<uint8_t>(TILE * Utot);
        P1.rowNnz = tmp.get<int64_t>(tmA);
        P1.dense_threshold = TH;
        nv.push("tsg a2 row path: masks per tile row");
        launch_sym_rows(P1, tmA, s);
        // ---------------- a3: nonzero offsets of the rows; the one allocation of C
        nv.push("tsg a3 scan + allocation");
        int64_t *rowOff = tmp.get<int64_t>(tmA + 1);
        DevCounters hc2{};
        {
            const std::initializer_list<DevRead> segs = {{&nnzC, rowOff + tmA, sizeof(int64_t)},
                                                         {&hc2, cnt, sizeof(DevCounters)}};
            const ExportArgs ex = begin_read(segs);
            exclusive_scan<int64_t>(P1.rowNnz, rowOff, tmA, s, tmp, &ex);
            finish_read(ex, segs, s);
        }
        syncs++;
        C->tile_col = out.get<int32_t>(ntC);
        C->tile_nnz = out.get<int64_t>(ntC + 1);
        C->row_ptr = out.get<uint8_t>(TILE * ntC);
        C->mask = out.get<uint16_t>(TILE * ntC);
        C->idx = out.get<uint8_t>(nnzC);
        C->val = out.get<uint8_t>((int64_t)dtype_size(dtC) * nnzC);
        C->tile_ptr = tile_ptr;
        tm_.mark(4);
        side.join();
        // ---------------- a4: step 3
        nv.push("tsg a4 numeric");
        RowNumArgs R{};
        R.tm = tmA;
        R.ntC = ntC;
        R.A = A;
        R.B = B;
        R.C = C;
        R.mTB = mTB;
        R.rowOccB = rowOccB;
        R.costOff = costOff;
        R.pairs = P1.pairs;
        R.tJ = P1.tJ;
        R.tStart = P1.tStart;
        R.tCnt = P1.tCnt;
        R.tNnz = P1.tWork;
        R.sMaskC = P1.sMaskC;
        R.sRowPtrC = P1.sRowPtrC;
        R.rowOff = rowOff;
        R.dense_threshold = TH;
        R.small_max = SMALL_NNZ;
        R.n_dense = (int64_t)hc2.n2dense;
        R.max_a_dense = (int)hc2.max_a_dense;
        R.colOccA = colOccA;
        R.small = tmp.get<uint8_t>(ROW_REC_BYTES * ntC);
        R.cnt = cnt;
        if (bias) {
            launch_add_i64(rowOff, tmA + 1, bias, s);
            C->idx -= bias;
            C->val = static_cast<uint8_t *>(C->val) - bias * (int64_t)dtype_size(dtC);
        }
        {  // the dense class runs on a side stream next to k_num_rows / k_num_small (disjoint outputs)
            SideStream sd(s);
            launch_num_rows(R, s, sd.stream());
            sd.join();
        }
        if (bias) {
            launch_add_i64(C->tile_nnz, ntC + 1, -bias, s);
            C->idx += bias;
            C->val = static_cast<uint8_t *>(C->val) + bias * (int64_t)dtype_size(dtC);
        }
        tm_.mark(5);
    } else {
        // C's tile arrays, per-tile pair ranges
        int32_t *tile_col = out.get<int32_t>(ntC);
        int64_t *tile_nnz = out.get<int64_t>(ntC + 1);
        uint8_t *row_ptr = out.get<uint8_t>(TILE * ntC);
        uint16_t *mask = out.get<uint16_t>(TILE * ntC);
        int64_t *pairBeg = tmp.get<int64_t>(ntC);
        uint32_t *pairCnt = tmp.get<uint32_t>(ntC);
        uint32_t *work = tmp.get<uint32_t>(ntC);
        CompactParams PC{tmA, A->tile_ptr, costOff, tile_ptr, P1.tJ, P1.tStart, P1.tCnt, P1.tWork,
                         tile_col, pairBeg, pairCnt, work};
        launch_compact(PC, ntC, s);

        // ---------------- a2: step 2
        nv.push("tsg a2 step 2: masks");
        side.join();
        StepParams P{};
        P.ntC = ntC;
        P.pairBeg = pairBeg;
        P.pairCnt = pairCnt;
        P.pairs = P1.pairs;
        P.tnzA = A->tile_nnz;
        P.rpA = A->row_ptr;
        P.mA = A->mask;
        P.mTA = mTA;
        P.colOccA = colOccA;
        P.ixA = A->idx;
        P.vA = A->val;
        P.dtype_in = A->dtype;
        P.tnzB = B->tile_nnz;
        P.rpB = B->row_ptr;
        P.mB = B->mask;
        P.rowOccB = rowOccB;
        P.mTB = mTB;
        P.ixB = B->idx;
        P.vB = B->val;
        P.tnzC = tile_nnz;
        P.rpC = row_ptr;
        P.mC = mask;
        P.work = work;
        {
            const int64_t ng = (ntC + 31) / 32;
            P.medL = tmp.get<uint32_t>(ng);
            P.medH = tmp.get<uint32_t>(ng);
            P.denL = tmp.get<uint32_t>(ng);
            P.denH = tmp.get<uint32_t>(ng);
        }
        P.qoverride = qv == 0 ? -1 : qv - 1;
        P.dense_threshold = TH;
        P.small_max = SMALL_NNZ;
        // small-tile B staging pays where B's tile metadata misses in cache: hypersparse tiles
        // (fewer than 4 nonzeros per B tile on average, e.g. R-MAT); flags force either way
        P.small_stage = (flags & TSG_SMALL_STAGE_ON) ? 1 : (flags & TSG_SMALL_STAGE_OFF) ? 0 : (B->nnz < 4 * B->nt);
        P.recA = recA;
        P.recB = recB;
        // A's records are B's when A lies inside B: their value offsets count from B's values
        P.recA_voff = (recA && recB && recA >= recB && recA < recB + B->nt) ? -(int64_t)(A->idx - B->idx) : 0;
        P.cnt = cnt;
        launch_step2(P, s);
        // ---------------- a3: offsets of C's nonzeros, allocation
        nv.push("tsg a3 scan + allocation");
        DevCounters hc2{};
        {
            const std::initializer_list<DevRead> segs = {{&nnzC, tile_nnz + ntC, sizeof(int64_t)},
                                                         {&hc2, cnt, sizeof(DevCounters)}};
            const ExportArgs ex = begin_read(segs);
            exclusive_scan<int64_t>(tile_nnz, tile_nnz, ntC, s, tmp, &ex);
            finish_read(ex, segs, s);
        }
        syncs++;
        uint8_t *idx = out.get<uint8_t>(nnzC);
        void *val = out.get<uint8_t>((int64_t)dtype_size(dtC) * nnzC);
        tm_.mark(4);
        // ---------------- a4: step 3
        nv.push("tsg a4 step 3: numeric");
        P.ixC = idx - bias;
        P.vC = static_cast<uint8_t *>(val) - bias * (int64_t)dtype_size(dtC);
        if (bias) launch_add_i64(tile_nnz, ntC + 1, bias, s);
        launch_step3(P, (int64_t)hc2.n2dense, s);
        if (bias) launch_add_i64(tile_nnz, ntC + 1, -bias, s);
        tm_.mark(5);
        C->tile_ptr = tile_ptr;
        C->tile_col = tile_col;
        C->tile_nnz = tile_nnz;
        C->row_ptr = row_ptr;
        C->mask = mask;
        C->idx = idx;
        C->val = val;
    }

    // ---------------- the result handle
    C->m = A->m;
    C->n = B->n;
    C->tm = tmA;
    C->tn = B->tn;
    C->nt = ntC;
    C->nnz = nnzC;
    C->dtype = dtC;
    for (int k = 0; k < 7; k++) {
        C->bytes[k] = out.take(C->array(k));
        C->owns[k] = true;
    }
    C->al = al;
    if (st) {
        DevCounters fin{};
        read_device({{&fin, cnt, sizeof(DevCounters)}}, s);
        memset(st, 0, sizeof(*st));
        st->products = (flags & TSG_STATS_PRODUCTS) ? (int64_t)fin.products : -1;
        st->tiles_structural = structural ? (int64_t)fin.structural : ((flags & TSG_STATS_STRUCTURAL) && tmA == 0 ? 0 : -1);
        st->tiles_c = ntC;
        st->nnz_c = nnzC;
        st->candidates = Utot;
        st->pairs = (int64_t)fin.pairs;
        st->tiles_dense = (int64_t)fin.n3dense;
        st->tiles_sparse = ntC - (int64_t)fin.n3dense;
        st->path = rowpath ? TSG_PATH_ROWS : TSG_PATH_TILES;
        st->step1_big_rows = (int64_t)fin.nbig;
        st->step1_list_tiles = (int32_t)fin.list_tiles;
        st->step1_merge_rows = (int64_t)fin.nmerge;
        st->bytes_scratch = (int64_t)tmp.handed();
        st->bytes_out = 0;
        for (int k = 0; k < 7; k++) st->bytes_out += (int64_t)C->bytes[k];
        st->host_syncs = syncs;
        st->kernel_launches = call_launches();
        st->ms_host_sync = (float)t_host_sync_ms;
        st->ms_host_alloc = (float)t_host_alloc_ms;
        if (tm_.on) {
            st->ms_index = tm_.ms(0, 1);
            st->ms_step1 = tm_.ms(1, 3);  // plan + step 1 (+ blocking read #1)
            st->ms_step2 = tm_.ms(3, 4);  // step 2 (masks), the nonzero scan, read #2, allocation of C
            st->ms_alloc = 0.f;
            st->ms_step3 = tm_.ms(4, 5);
            st->ms_total = tm_.ms(0, 5);
        }
    }
}

}  // namespace tsg
