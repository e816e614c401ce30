// tsg_spgemm.cu -- host orchestration of one tsg_spgemm call: the three steps of TileSpGEMM
// (Section 3.3) with the device prefix sums and allocations between them.
//
//   a0  helper indices (tsg_step1.cu): occupancy words, optional B row lists
//   a1  step 1 (tsg_step1.cu): exact C tile layout + contributing pairs in ascending K
//   a2  step 2 (tsg_step23.cu): bit-mask symbolic phase, row offsets, tile nnz
//   a3  device prefix sums + allocation of C (tsg_scan.cu, stream-ordered pool)
//   a4  step 3 (tsg_step23.cu): numeric phase with the adaptive accumulator
//
// Blocking device->host reads: (0) candidate total and row classes, (1) number of C tiles,
// (2) nnz(C).  Everything else is stream-ordered.
#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "tsg_kernels.cuh"

namespace tsg {
namespace {
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
}  // namespace

namespace {
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
    void done() { TSG_CUDA(cudaEventRecord(r_->joinev, r_->side)); recorded_ = true; }
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
    TSG_REQUIRE(A->nt < ((int64_t)1 << 31) && B->nt < ((int64_t)1 << 31), TSG_ERR_OVERFLOW, "input has >= 2^31 tiles");
    TSG_REQUIRE(A->tn == B->tm, TSG_ERR_SHAPE, "tile shapes disagree");
    TSG_REQUIRE(A->dtype == B->dtype, TSG_ERR_INVALID_ARG, "A and B value types differ");
    const int32_t dtC = A->dtype == TSG_F64 ? TSG_F64 : TSG_F32;  // F16 x F16 -> F32
    TSG_REQUIRE(((uintptr_t)A->mask & 15) == 0 && ((uintptr_t)B->mask & 15) == 0 && ((uintptr_t)A->row_ptr & 15) == 0 &&
                    ((uintptr_t)B->row_ptr & 15) == 0 && ((uintptr_t)A->val % A->vsize()) == 0 && ((uintptr_t)B->val % B->vsize()) == 0,
                TSG_ERR_INVALID_ARG, "mask and row_ptr arrays must be 16-byte aligned, val aligned to its type");
    int TH = (int)((flags >> TSG_DENSE_THRESHOLD_SHIFT) & 0x1ffu);
    if (TH == 0) TH = TSG_DENSE_NNZ;
    if (const char *e = getenv("TSG_DENSE_THRESHOLD")) TH = std::max(1, std::min(257, atoi(e)));  // tuning only
    Timer tm_;
    tm_.init((flags & TSG_STATS_TIMING) && st, s);
    tm_.mark(0);

    Buffers tmp(al, s, true), out(al, s);
    const int64_t ntA = A->nt, tmA = A->tm, tmB = B->tm;
    int syncs = 0;
    DevCounters *cnt = tmp.get<DevCounters>(1);
    TSG_CUDA(cudaMemsetAsync(cnt, 0, sizeof(DevCounters), s));

    // ---------------- a0: occupancy words, optional B row lists, optional product count
    // A inside B's tile arrays (A^2, or a row slice of B: SURVEY 8(e)'s rank shards and row blocks):
    // A's tile t is B's tile t + off, so one pass over B gives A's helper words too
    const int64_t off = (int64_t)(A->mask - B->mask) / TILE;
    const bool inB = A->mask >= B->mask && (A->mask - B->mask) % TILE == 0 && off + ntA <= B->nt;
    uint16_t *rowOccB = tmp.get<uint16_t>(B->nt);
    uint16_t *colOccA;
    if (inB) {
        uint16_t *colOccB = tmp.get<uint16_t>(B->nt);
        launch_occupancy(B->mask, B->nt, rowOccB, colOccB, s);
        colOccA = colOccB + off;
    } else {
        colOccA = tmp.get<uint16_t>(ntA);
        launch_occupancy(A->mask, ntA, nullptr, colOccA, s);
        launch_occupancy(B->mask, B->nt, rowOccB, nullptr, s);
    }
    // transposed masks: first used by step 2, so they are computed on a side stream while step 1
    // runs (joined before step 2, and on every exit path by the guard's destructor)
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
    if (lists) {
        int32_t *lcnt = tmp.get<int32_t>(TILE * tmB);
        lptr = tmp.get<int64_t>(TILE * tmB + 1);
        list = tmp.get<uint32_t>(B->nnz);
        launch_rowlist(tmB, B->tile_ptr, B->mask, nullptr, lcnt, nullptr, s);
        exclusive_scan<int32_t>(lcnt, lptr, TILE * tmB, s, tmp);
        launch_rowlist(tmB, B->tile_ptr, B->mask, lptr, lcnt, list, s);
    }
    if (st && (flags & TSG_STATS_PRODUCTS)) {
        int32_t *rnnz = tmp.get<int32_t>(TILE * tmB);
        launch_products(tmB, B->tile_ptr, B->mask, ntA, A->tile_col, A->mask, rnnz, cnt, s);
    }
    tm_.mark(1);

    // ---------------- a1: step 1
    int64_t *cost = tmp.get<int64_t>(ntA);
    int64_t *startA = tmp.get<int64_t>(ntA);
    int32_t *jloA = tmp.get<int32_t>(ntA);
    int32_t *jhiA = tmp.get<int32_t>(ntA);
    launch_atile_plan(ntA, A->tile_col, colOccA, B->tile_ptr, B->tile_col, lptr, list,
                      (bool)(flags & TSG_STEP1_SCAN_ONLY), cost, startA, jloA, jhiA, cnt, s);
    int64_t *costOff = tmp.get<int64_t>(ntA + 1);
    exclusive_scan<int64_t>(cost, costOff, ntA, s, tmp);
    int32_t *rowJlo = tmp.get<int32_t>(tmA);
    int32_t *rowJhi = tmp.get<int32_t>(tmA);
    uint8_t *rowClass = tmp.get<uint8_t>(tmA);
    int64_t *nC = tmp.get<int64_t>(tmA + 1);
    int32_t *bigList = tmp.get<int32_t>(tmA);
    int64_t *bigOff = tmp.get<int64_t>(tmA);
    launch_row_plan(tmA, A->tile_ptr, costOff, jloA, jhiA, !(flags & TSG_STEP1_SORT_ONLY), rowJlo, rowJhi, rowClass,
                    nC, bigList, bigOff, cnt, s);
    // sync #0: candidate total and row classes
    DevCounters hc{};
    int64_t Utot = 0;
    read_device({{&Utot, costOff + ntA, sizeof(int64_t)}, {&hc, cnt, sizeof(DevCounters)}}, s);
    syncs++;
    TSG_REQUIRE(Utot < ((int64_t)1 << 40), TSG_ERR_OVERFLOW, "too many step-1 candidates");

    S1Params P1{};
    P1.tpA = A->tile_ptr;
    P1.tnzA = A->tile_nnz;
    P1.colOccA = colOccA;
    P1.costOff = costOff;
    P1.startA = startA;
    P1.tcB = B->tile_col;
    P1.rowOccB = rowOccB;
    P1.list = list;
    P1.rowJlo = rowJlo;
    P1.rowJhi = rowJhi;
    P1.rowClass = rowClass;
    P1.tnB = B->tn;
    P1.sort_only = (flags & TSG_STEP1_SORT_ONLY) ? 1 : 0;
    P1.pairs = tmp.get<uint64_t>(Utot);
    P1.tJ = tmp.get<int32_t>(Utot);
    P1.tStart = tmp.get<uint32_t>(Utot);
    P1.tCnt = tmp.get<uint32_t>(Utot);
    P1.tWork = tmp.get<uint32_t>(Utot);
    P1.nC = nC;
    P1.bigList = bigList;
    P1.bigOff = bigOff;
    P1.cnt = cnt;
    if (hc.nbig > 0) {
        P1.bigKeysA = tmp.get<uint64_t>(hc.big_u);
        P1.bigKeysB = tmp.get<uint64_t>(hc.big_u);
        P1.bigPosB = tmp.get<uint32_t>(hc.big_u);
        P1.bigKpos = tmp.get<uint32_t>(hc.big_u);
    }
    launch_row_sort(P1, tmA, (int64_t)hc.max_u_small, (int64_t)hc.nbig, (int64_t)hc.nmerge, s);
    int64_t *tile_ptr = out.get<int64_t>(tmA + 1);
    exclusive_scan<int64_t>(nC, tile_ptr, tmA, s, tmp);
    tm_.mark(2);
    // sync #1: number of C tiles
    const int64_t ntC = read_scalar(tile_ptr + tmA, s);
    syncs++;
    TSG_REQUIRE(ntC < ((int64_t)1 << 32), TSG_ERR_OVERFLOW, "C has >= 2^32 tiles");

    // ---------------- allocation of C's tile arrays, per-tile pair ranges, class lists
    int32_t *tile_col = out.get<int32_t>(ntC);
    int64_t *tile_nnz = out.get<int64_t>(ntC + 1);
    uint8_t *row_ptr = out.get<uint8_t>(TILE * ntC);
    uint16_t *mask = out.get<uint16_t>(TILE * ntC);
    int64_t *pairBeg = tmp.get<int64_t>(ntC);
    uint32_t *pairCnt = tmp.get<uint32_t>(ntC);
    uint32_t *work = tmp.get<uint32_t>(ntC);
    tm_.mark(3);
    CompactParams PC{tmA, A->tile_ptr, costOff, tile_ptr, P1.tJ, P1.tStart, P1.tCnt, P1.tWork,
                     tile_col, pairBeg, pairCnt, work};
    launch_compact(PC, s);

    // ---------------- a2: step 2
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
    P.dense_threshold = TH;
    P.small_max = SMALL_NNZ;
    P.dense_tc = ((flags & TSG_DENSE_TC) || getenv("TSG_DENSE_TC")) ? 1 : 0;  // env: tuning only
    // small-tile B staging pays where B's tile metadata misses in cache: hypersparse tiles
    // (fewer than 4 nonzeros per B tile on average, e.g. R-MAT); flags force either way
    P.small_stage = (flags & TSG_SMALL_STAGE_ON) ? 1 : (flags & TSG_SMALL_STAGE_OFF) ? 0 : (B->nnz < 4 * B->nt);
    if (const char *e = getenv("TSG_SMALL_NNZ")) P.small_max = std::max(0, std::min(16, atoi(e)));  // tuning only
    P.cnt = cnt;
    launch_step2(P, s);
    // ---------------- a3: offsets of C's nonzeros, allocation
    exclusive_scan<int64_t>(tile_nnz, tile_nnz, ntC, s, tmp);
    tm_.mark(4);
    // step-3 row classes: whole C tile rows for the row kernel, the rest per tile
    RowParams R{};
    R.tm = tmA;
    R.tpA = A->tile_ptr;
    R.tcA = A->tile_col;
    R.tnzA = A->tile_nnz;
    R.rpA = A->row_ptr;
    R.mA = A->mask;
    R.colOccA = colOccA;
    R.vA = static_cast<const double *>(A->val);
    R.tpB = B->tile_ptr;
    R.tnzB = B->tile_nnz;
    R.rpB = B->row_ptr;
    R.mB = B->mask;
    R.vB = static_cast<const double *>(B->val);
    R.pairs = P1.pairs;
    R.pairBeg = pairBeg;
    R.pairCnt = pairCnt;
    R.tpC = tile_ptr;
    R.tnzC = tile_nnz;
    R.rpC = row_ptr;
    R.mC = mask;
    R.dense_threshold = TH;
    R.cnt = cnt;
    const bool rowk = (flags & TSG_STEP3_ROWS) != 0 && A->dtype == TSG_F64;  // the row kernel is fp64 only
    if (rowk) {
        R.rowAcc = tmp.get<int32_t>(tmA);
        R.skip = tmp.get<uint8_t>(ntC);
        launch_step3_class(R, s);
    }
    int64_t nnzC = 0;
    DevCounters hc2{};
    read_device({{&nnzC, tile_nnz + ntC, sizeof(int64_t)}, {&hc2, cnt, sizeof(DevCounters)}}, s);
    syncs++;
    uint8_t *idx = out.get<uint8_t>(nnzC);
    void *val = out.get<uint8_t>((int64_t)dtype_size(dtC) * nnzC);
    tm_.mark(5);

    // ---------------- a4: step 3
    P.ixC = idx;
    P.vC = val;
    R.ixC = idx;
    R.vC = static_cast<double *>(val);
    if (rowk && hc2.n3rows > 0) launch_step3_rows(R, s);
    if (!rowk || hc2.n3fallback > 0) {
        P.skip = rowk ? R.skip : nullptr;
        launch_step3(P, (int64_t)hc2.n2dense, s);
    }
    tm_.mark(6);

    // ---------------- the result handle
    C->m = A->m;
    C->n = B->n;
    C->tm = tmA;
    C->tn = B->tn;
    C->nt = ntC;
    C->nnz = nnzC;
    C->tile_ptr = tile_ptr;
    C->tile_col = tile_col;
    C->tile_nnz = tile_nnz;
    C->row_ptr = row_ptr;
    C->mask = mask;
    C->idx = idx;
    C->val = val;
    C->dtype = dtC;
    void *arr[7] = {tile_ptr, tile_col, tile_nnz, row_ptr, mask, idx, val};
    for (int k = 0; k < 7; k++) {
        C->bytes[k] = out.take(arr[k]);
        C->owns[k] = true;
    }
    C->al = al;
    if (st) {
        DevCounters fin{};
        read_device({{&fin, cnt, sizeof(DevCounters)}}, s);
        memset(st, 0, sizeof(*st));
        st->products = (flags & TSG_STATS_PRODUCTS) ? (int64_t)fin.products : -1;
        st->tiles_structural = -1;
        st->tiles_c = ntC;
        st->nnz_c = nnzC;
        st->candidates = Utot;
        st->pairs = (int64_t)fin.pairs;
        st->tiles_dense = (int64_t)fin.n3dense;
        st->tiles_sparse = ntC - (int64_t)fin.n3dense;
        st->step3_rows = (int64_t)fin.n3rows;
        st->step3_row_tiles = rowk ? ntC - (int64_t)fin.n3fallback : 0;
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
            st->ms_step1 = tm_.ms(1, 2);
            st->ms_alloc = tm_.ms(2, 3) + tm_.ms(4, 5);
            st->ms_step2 = tm_.ms(3, 4);
            st->ms_step3 = tm_.ms(5, 6);
            st->ms_total = tm_.ms(0, 6);
        }
    }
}

}  // namespace tsg
