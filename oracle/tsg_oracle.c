/*
 * tsg_oracle.c -- plain, slow, single-threaded CPU oracle for TileSpGEMM (Niu et al., PPoPP'22).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference leg may load this library.  It shares no code, header, table or constant
 * generator with the CUDA path (paper_conf_ppopp_niuljs0022_b200/csrc) and never calls it.
 *
 * Citations are to /root/reference/PAPER.md lines ("P:a-b") and to the readings A1..A17 listed
 * in DESIGN.md §2 (taken from SURVEY.md §8(c)).  Everything is fp64; build with
 * -O2 -ffp-contract=off so that a*b+c is never silently fused (the fma mode asks for it).
 *
 *   O1 orc_gustavson_*      Gustavson row-row SpGEMM, Algorithm 1, dense accumulator
 *   O2 orc_csr_to_tiles_*   CSR -> sparse-tile format, Section 3.2
 *   O3 orc_tiles_to_csr     inverse of O2
 *   O4 orc_tile_structural_*, orc_step2_masks
 *                           Section 3.3 step 1 (C' = A'B') and Algorithm 2
 *                           (set intersection + bit-mask OR)
 *   O5 orc_products         number of intermediate products (Table 2 caption)
 *   -- orc_gustavson*_omp   O1 over contiguous row chunks on OpenMP threads (a baseline, same results)
 *   -- orc_spmv             y = A x, for the row-sum invariant C·1 = A·(B·1)
 *
 * Status codes: 0 ok, -1 bad argument, -2 out of memory, -3 inconsistent input.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define TILE 16 /* "our tile size is always set to 16-by-16" */

static int cmp_i64(const void *a, const void *b) {
    int64_t x = *(const int64_t *)a, y = *(const int64_t *)b;
    return (x > y) - (x < y);
}

/* ------------------------------------------------------------------------------------------
 * O5: products = sum_i sum_{k in A(i,:)} nnz(B(k,:))  (Table 2 caption: "the number of
 * intermediate products (i.e., half of the number of floating point operations)")
 * ------------------------------------------------------------------------------------------ */
int64_t orc_products(int64_t m, const int64_t *Arp, const int32_t *Aci, const int64_t *Brp) {
    int64_t total = 0;
    for (int64_t i = 0; i < m; i++)
        for (int64_t p = Arp[i]; p < Arp[i + 1]; p++) total += Brp[Aci[p] + 1] - Brp[Aci[p]];
    return total;
}

/* ------------------------------------------------------------------------------------------
 * O1: Gustavson row-row SpGEMM, Algorithm 1.
 *
 * For each row i of A (line 1), each nonzero a_ik (line 4), each nonzero b_kj of row k of B
 * (line 5): value = a_ik*b_kj (line 6); if c_ij is not yet in row i, insert it and set it to the
 * value (lines 7-9), else add the value (line 11).  The accumulator is dense (size n) with a
 * stamp array recording the first touch; the touched columns are sorted at the end of the row.
 * Every touched column is emitted, including exact zeros from cancellation (reading A11).
 * fma_mode=1 replaces line 11 by c = fma(a, b, c) (reading A16, bitwise comparison gate).
 * abs_out[e] = sum |a*b| over the products that formed entry e (tolerance bound).
 *
 * rows == NULL computes all m rows; otherwise rows[0..nrows) (any order) and the output is the
 * concatenation of those rows.  Two calls: orc_gustavson_rowcounts then orc_gustavson.
 * ------------------------------------------------------------------------------------------ */
int orc_gustavson_rowcounts(int64_t m, int64_t n, const int64_t *Arp, const int32_t *Aci,
                            const int64_t *Brp, const int32_t *Bci, const int64_t *rows,
                            int64_t nrows, int64_t *rowlen) {
    if (m < 0 || n < 0) return -1;
    int64_t *stamp = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    if (!stamp) return -2;
    for (int64_t j = 0; j < n; j++) stamp[j] = -1;
    int64_t R = rows ? nrows : m;
    for (int64_t t = 0; t < R; t++) {
        int64_t i = rows ? rows[t] : t;
        int64_t cnt = 0;
        for (int64_t p = Arp[i]; p < Arp[i + 1]; p++) {
            int64_t k = Aci[p];
            for (int64_t q = Brp[k]; q < Brp[k + 1]; q++) {
                int64_t j = Bci[q];
                if (stamp[j] != t) {
                    stamp[j] = t;
                    cnt++;
                }
            }
        }
        rowlen[t] = cnt;
    }
    free(stamp);
    return 0;
}

int orc_gustavson(int64_t m, int64_t n, const int64_t *Arp, const int32_t *Aci, const double *Aval,
                  const int64_t *Brp, const int32_t *Bci, const double *Bval, const int64_t *rows,
                  int64_t nrows, const int64_t *Crp, int32_t *Cci, double *Cval, double *Cabs,
                  int fma_mode) {
    if (m < 0 || n < 0) return -1;
    size_t nn = (size_t)(n > 0 ? n : 1);
    int64_t *stamp = (int64_t *)malloc(sizeof(int64_t) * nn);
    double *acc = (double *)malloc(sizeof(double) * nn);
    double *acc_abs = (double *)malloc(sizeof(double) * nn);
    int64_t *list = (int64_t *)malloc(sizeof(int64_t) * nn);
    if (!stamp || !acc || !acc_abs || !list) {
        free(stamp); free(acc); free(acc_abs); free(list);
        return -2;
    }
    for (int64_t j = 0; j < n; j++) stamp[j] = -1;
    int64_t R = rows ? nrows : m;
    for (int64_t t = 0; t < R; t++) {
        int64_t i = rows ? rows[t] : t;
        int64_t len = 0;
        for (int64_t p = Arp[i]; p < Arp[i + 1]; p++) {          /* line 4, ascending k */
            int64_t k = Aci[p];
            double a = Aval[p];
            for (int64_t q = Brp[k]; q < Brp[k + 1]; q++) {      /* line 5 */
                int64_t j = Bci[q];
                double b = Bval[q];
                double value = a * b;                            /* line 6 */
                if (stamp[j] != t) {                             /* lines 7-9: insert */
                    stamp[j] = t;
                    list[len++] = j;
                    acc[j] = value;
                    acc_abs[j] = fabs(value);
                } else {                                         /* line 11: accumulate */
                    acc[j] = fma_mode ? fma(a, b, acc[j]) : acc[j] + value;
                    acc_abs[j] += fabs(value);
                }
            }
        }
        if (Crp[t + 1] - Crp[t] != len) {
            free(stamp); free(acc); free(acc_abs); free(list);
            return -3;
        }
        qsort(list, (size_t)len, sizeof(int64_t), cmp_i64);
        for (int64_t e = 0; e < len; e++) {
            int64_t j = list[e];
            Cci[Crp[t] + e] = (int32_t)j;
            Cval[Crp[t] + e] = acc[j];
            if (Cabs) Cabs[Crp[t] + e] = acc_abs[j];
        }
    }
    free(stamp); free(acc); free(acc_abs); free(list);
    return 0;
}

/* O1 on all host cores (the oracle_omp baseline).  The row sample is split into
 * nthreads contiguous chunks and each chunk is computed by the unchanged single-threaded
 * orc_gustavson_rowcounts / orc_gustavson above on its own OpenMP thread (private accumulators).
 * The per-row arithmetic is identical, so the result equals the single-threaded one bit for bit
 * (tests/test_oracle_pins.py).  `rows` must be given (the row ids of the sample). */
int orc_gustavson_rowcounts_omp(int64_t m, int64_t n, const int64_t *Arp, const int32_t *Aci,
                                const int64_t *Brp, const int32_t *Bci, const int64_t *rows,
                                int64_t nrows, int64_t *rowlen, int nthreads) {
    if (!rows || nthreads < 1) return -1;
    int rc = 0;
#pragma omp parallel for num_threads(nthreads) schedule(static) reduction(min : rc)
    for (int c = 0; c < nthreads; c++) {
        const int64_t r0 = nrows * c / nthreads, r1 = nrows * (c + 1) / nthreads;
        const int e = orc_gustavson_rowcounts(m, n, Arp, Aci, Brp, Bci, rows + r0, r1 - r0, rowlen + r0);
        if (e < rc) rc = e;
    }
    return rc;
}

int orc_gustavson_omp(int64_t m, int64_t n, const int64_t *Arp, const int32_t *Aci, const double *Aval,
                      const int64_t *Brp, const int32_t *Bci, const double *Bval, const int64_t *rows,
                      int64_t nrows, const int64_t *Crp, int32_t *Cci, double *Cval, double *Cabs,
                      int fma_mode, int nthreads) {
    if (!rows || nthreads < 1) return -1;
    int rc = 0;
#pragma omp parallel for num_threads(nthreads) schedule(static) reduction(min : rc)
    for (int c = 0; c < nthreads; c++) {
        const int64_t r0 = nrows * c / nthreads, r1 = nrows * (c + 1) / nthreads;
        const int e = orc_gustavson(m, n, Arp, Aci, Aval, Brp, Bci, Bval, rows + r0, r1 - r0, Crp + r0, Cci, Cval,
                                    Cabs, fma_mode);
        if (e < rc) rc = e;
    }
    return rc;
}

/* O1 in single precision (the paper's Section 4.7 setup computes with half
 * inputs and single-precision output): the same Algorithm 1 loop with float
 * accumulators; inputs are floats (a half input is widened to float exactly before the call).
 * Cabs is the fp64 sum of |a*b| (exact products of floats). */
int orc_gustavson_f32(int64_t m, int64_t n, const int64_t *Arp, const int32_t *Aci, const float *Aval,
                      const int64_t *Brp, const int32_t *Bci, const float *Bval, const int64_t *rows,
                      int64_t nrows, const int64_t *Crp, int32_t *Cci, float *Cval, double *Cabs,
                      int fma_mode) {
    if (m < 0 || n < 0) return -1;
    size_t nn = (size_t)(n > 0 ? n : 1);
    int64_t *stamp = (int64_t *)malloc(sizeof(int64_t) * nn);
    float *acc = (float *)malloc(sizeof(float) * nn);
    double *acc_abs = (double *)malloc(sizeof(double) * nn);
    int64_t *list = (int64_t *)malloc(sizeof(int64_t) * nn);
    if (!stamp || !acc || !acc_abs || !list) {
        free(stamp); free(acc); free(acc_abs); free(list);
        return -2;
    }
    for (int64_t j = 0; j < n; j++) stamp[j] = -1;
    int64_t R = rows ? nrows : m;
    for (int64_t t = 0; t < R; t++) {
        int64_t i = rows ? rows[t] : t;
        int64_t len = 0;
        for (int64_t p = Arp[i]; p < Arp[i + 1]; p++) {          /* line 4, ascending k */
            int64_t k = Aci[p];
            float a = Aval[p];
            for (int64_t q = Brp[k]; q < Brp[k + 1]; q++) {      /* line 5 */
                int64_t j = Bci[q];
                float b = Bval[q];
                float value = a * b;                             /* line 6 */
                if (stamp[j] != t) {                             /* lines 7-9: insert */
                    stamp[j] = t;
                    list[len++] = j;
                    acc[j] = value;
                    acc_abs[j] = fabs((double)a * (double)b);
                } else {                                         /* line 11: accumulate */
                    acc[j] = fma_mode ? fmaf(a, b, acc[j]) : acc[j] + value;
                    acc_abs[j] += fabs((double)a * (double)b);
                }
            }
        }
        if (Crp[t + 1] - Crp[t] != len) {
            free(stamp); free(acc); free(acc_abs); free(list);
            return -3;
        }
        qsort(list, (size_t)len, sizeof(int64_t), cmp_i64);
        for (int64_t e = 0; e < len; e++) {
            int64_t j = list[e];
            Cci[Crp[t] + e] = (int32_t)j;
            Cval[Crp[t] + e] = acc[j];
            if (Cabs) Cabs[Crp[t] + e] = acc_abs[j];
        }
    }
    free(stamp); free(acc); free(acc_abs); free(list);
    return 0;
}

/* ------------------------------------------------------------------------------------------
 * O2: CSR -> sparse tiles, Section 3.2.
 *   tile_ptr[tm+1]   offsets of tiles per tile row
 *   tile_col[nt]     tile column index, ascending within a tile row
 *   tile_nnz[nt+1]   offsets of each tile's nonzeros (exclusive scan)
 *   val[nnz]         values in tile order, CSR order inside the tile
 *   idx[nnz]         (r<<4)|c, 4+4 bits "within an 8-bit unsigned char"  (reading A1)
 *   row_ptr[16*nt]   16 local row offsets, no 17th entry                 (reading A3)
 *   mask[16*nt]      bit c of row r set iff (r,c) is a nonzero           (reading A2)
 * tm = ceil(m/16), tn = ceil(n/16); padding rows/cols never carry bits (reading A5).
 * ------------------------------------------------------------------------------------------ */
int orc_csr_to_tiles_count(int64_t m, int64_t n, const int64_t *Arp, const int32_t *Aci,
                           int64_t *tile_ptr) {
    if (m < 0 || n < 0) return -1;
    int64_t tm = (m + TILE - 1) / TILE, tn = (n + TILE - 1) / TILE;
    int64_t *seen = (int64_t *)malloc(sizeof(int64_t) * (size_t)(tn > 0 ? tn : 1));
    if (!seen) return -2;
    for (int64_t J = 0; J < tn; J++) seen[J] = -1;
    tile_ptr[0] = 0;
    for (int64_t I = 0; I < tm; I++) {
        int64_t cnt = 0;
        for (int64_t i = I * TILE; i < (I + 1) * TILE && i < m; i++)
            for (int64_t p = Arp[i]; p < Arp[i + 1]; p++) {
                int64_t J = Aci[p] / TILE;
                if (seen[J] != I) {
                    seen[J] = I;
                    cnt++;
                }
            }
        tile_ptr[I + 1] = tile_ptr[I] + cnt;
    }
    free(seen);
    return 0;
}

int orc_csr_to_tiles_fill(int64_t m, int64_t n, const int64_t *Arp, const int32_t *Aci,
                          const double *Aval, const int64_t *tile_ptr, int32_t *tile_col,
                          int64_t *tile_nnz, uint8_t *row_ptr, uint16_t *mask, uint8_t *idx,
                          double *val) {
    if (m < 0 || n < 0) return -1;
    int64_t tm = (m + TILE - 1) / TILE, tn = (n + TILE - 1) / TILE;
    int64_t *seen = (int64_t *)malloc(sizeof(int64_t) * (size_t)(tn > 0 ? tn : 1));
    int64_t *cols = (int64_t *)malloc(sizeof(int64_t) * (size_t)(tn > 0 ? tn : 1));
    if (!seen || !cols) { free(seen); free(cols); return -2; }
    for (int64_t J = 0; J < tn; J++) seen[J] = -1;
    int64_t out = 0; /* running nonzero offset, tile order */
    tile_nnz[0] = 0;
    for (int64_t I = 0; I < tm; I++) {
        /* the set of non-empty tile columns of tile row I, ascending */
        int64_t cnt = 0;
        for (int64_t i = I * TILE; i < (I + 1) * TILE && i < m; i++)
            for (int64_t p = Arp[i]; p < Arp[i + 1]; p++) {
                int64_t J = Aci[p] / TILE;
                if (seen[J] != I) { seen[J] = I; cols[cnt++] = J; }
            }
        if (cnt != tile_ptr[I + 1] - tile_ptr[I]) { free(seen); free(cols); return -3; }
        qsort(cols, (size_t)cnt, sizeof(int64_t), cmp_i64);
        for (int64_t q = 0; q < cnt; q++) {
            int64_t t = tile_ptr[I] + q, J = cols[q];
            tile_col[t] = (int32_t)J;
            int64_t start = out;
            for (int r = 0; r < TILE; r++) {
                int64_t i = I * TILE + r;
                row_ptr[t * TILE + r] = (uint8_t)(out - start);  /* count of rows < r */
                uint16_t mk = 0;
                if (i < m)
                    for (int64_t p = Arp[i]; p < Arp[i + 1]; p++) {
                        int64_t j = Aci[p];
                        if (j / TILE != J) continue;
                        int c = (int)(j % TILE);
                        mk |= (uint16_t)(1u << c);
                        idx[out] = (uint8_t)((r << 4) | c);
                        val[out] = Aval[p];
                        out++;
                    }
                mask[t * TILE + r] = mk;
            }
            tile_nnz[t + 1] = out;
        }
    }
    free(seen); free(cols);
    return 0;
}

/* ------------------------------------------------------------------------------------------
 * O3: sparse tiles -> CSR (inverse of O2).  Row r of tile t spans
 * [tile_nnz[t] + row_ptr[16t+r], tile_nnz[t] + row_ptr[16t+r+1]) with the 17th offset taken
 * from tile_nnz[t+1].  Column = 16*tile_col[t] + (idx & 15).
 * Returns -3 if an idx row nibble disagrees with its row segment.
 * ------------------------------------------------------------------------------------------ */
int orc_tiles_to_csr(int64_t m, int64_t n, const int64_t *tile_ptr, const int32_t *tile_col,
                     const int64_t *tile_nnz, const uint8_t *row_ptr, const uint8_t *idx,
                     const double *val, int64_t *Crp, int32_t *Cci, double *Cval) {
    if (m < 0 || n < 0) return -1;
    int64_t tm = (m + TILE - 1) / TILE;
    int64_t out = 0;
    Crp[0] = 0;
    for (int64_t I = 0; I < tm; I++)
        for (int r = 0; r < TILE; r++) {
            int64_t i = I * TILE + r;
            if (i >= m) break;
            for (int64_t t = tile_ptr[I]; t < tile_ptr[I + 1]; t++) {
                int64_t b = tile_nnz[t] + row_ptr[t * TILE + r];
                int64_t e = (r < TILE - 1) ? tile_nnz[t] + row_ptr[t * TILE + r + 1] : tile_nnz[t + 1];
                for (int64_t p = b; p < e; p++) {
                    if ((idx[p] >> 4) != r) return -3;
                    Cci[out] = (int32_t)(tile_col[t] * TILE + (idx[p] & 15));
                    Cval[out] = val[p];
                    out++;
                }
            }
            Crp[i + 1] = out;
        }
    return 0;
}

/* ------------------------------------------------------------------------------------------
 * O4a: step 1 of Section 3.3, the structural tile product C' = A'B'.  A' and B'
 * are the tile layouts (tile_ptr/tile_col); "only sparsity structures of matrices A' and B' are
 * needed".  No tile-wise cancellation is considered, so C' may contain tiles that
 * turn out empty.  count: Cp_ptr[tm+1]; fill: Cp_col (ascending per tile row).
 * ------------------------------------------------------------------------------------------ */
static int structural(int64_t tmA, int64_t tnB, const int64_t *tpA, const int32_t *tcA,
                      const int64_t *tpB, const int32_t *tcB, int64_t *Cp_ptr, int32_t *Cp_col) {
    int64_t *seen = (int64_t *)malloc(sizeof(int64_t) * (size_t)(tnB > 0 ? tnB : 1));
    int64_t *cols = (int64_t *)malloc(sizeof(int64_t) * (size_t)(tnB > 0 ? tnB : 1));
    if (!seen || !cols) { free(seen); free(cols); return -2; }
    for (int64_t J = 0; J < tnB; J++) seen[J] = -1;
    Cp_ptr[0] = 0;
    for (int64_t I = 0; I < tmA; I++) {
        int64_t cnt = 0;
        for (int64_t p = tpA[I]; p < tpA[I + 1]; p++) {
            int64_t K = tcA[p];
            for (int64_t q = tpB[K]; q < tpB[K + 1]; q++) {
                int64_t J = tcB[q];
                if (seen[J] != I) { seen[J] = I; cols[cnt++] = J; }
            }
        }
        if (Cp_col) {
            if (cnt != Cp_ptr[I + 1] - Cp_ptr[I]) { free(seen); free(cols); return -3; }
            qsort(cols, (size_t)cnt, sizeof(int64_t), cmp_i64);
            for (int64_t q = 0; q < cnt; q++) Cp_col[Cp_ptr[I] + q] = (int32_t)cols[q];
        } else {
            Cp_ptr[I + 1] = Cp_ptr[I] + cnt;
        }
    }
    free(seen); free(cols);
    return 0;
}

int orc_tile_structural_count(int64_t tmA, int64_t tnB, const int64_t *tpA, const int32_t *tcA,
                              const int64_t *tpB, const int32_t *tcB, int64_t *Cp_ptr) {
    return structural(tmA, tnB, tpA, tcA, tpB, tcB, Cp_ptr, NULL);
}

int orc_tile_structural_fill(int64_t tmA, int64_t tnB, const int64_t *tpA, const int32_t *tcA,
                             const int64_t *tpB, const int32_t *tcB, const int64_t *Cp_ptr,
                             int32_t *Cp_col) {
    return structural(tmA, tnB, tpA, tcA, tpB, tcB, (int64_t *)Cp_ptr, Cp_col);
}

/* ------------------------------------------------------------------------------------------
 * O4b: step 2 of Section 3.3, Algorithm 2, for a list of C tiles (row I, col J):
 *   lines 4-18: the set intersection of tilecolidx_A(I,*) with tilerowidx_B(*,J).
 *     B's tile columns come from a tile-CSC of B built here (tileColPtr_B / tileRowidx_B,
 *     reading A9).  Any exact intersection gives the same sorted list (reading A13); a plain
 *     two-pointer merge is used.
 *   lines 19-25: for each matched pair (A_IK, B_KJ) and each nonzero (r,c) of A_IK,
 *     mask_C[r] |= mask_B_KJ[c] (Fig 5).
 *   nnz of the tile = sum of popcounts of mask_C.
 * Outputs per C tile: mask[16*nc], nnz[nc], matched[nc] (intersection size),
 * contributing[nc] (pairs whose A column set meets the B row set: colOcc(A)&rowOcc(B) != 0).
 * ------------------------------------------------------------------------------------------ */
int orc_step2_masks(int64_t tmB, int64_t tnB, const int64_t *tpA, const int32_t *tcA,
                    const uint16_t *maskA, const int64_t *tpB, const int32_t *tcB,
                    const uint16_t *maskB, int64_t nc, const int64_t *cI, const int32_t *cJ,
                    uint16_t *mask_out, int64_t *nnz_out, int64_t *matched_out,
                    int64_t *contrib_out) {
    int64_t ntB = tpB[tmB];
    /* tile-CSC of B: for each tile column J, the (tile row K, tile position) pairs ascending K */
    int64_t *cptr = (int64_t *)calloc((size_t)tnB + 1, sizeof(int64_t));
    int64_t *crow = (int64_t *)malloc(sizeof(int64_t) * (size_t)(ntB > 0 ? ntB : 1));
    int64_t *cpos = (int64_t *)malloc(sizeof(int64_t) * (size_t)(ntB > 0 ? ntB : 1));
    int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)(tnB > 0 ? tnB : 1));
    if (!cptr || !crow || !cpos || !fill) { free(cptr); free(crow); free(cpos); free(fill); return -2; }
    for (int64_t q = 0; q < ntB; q++) cptr[tcB[q] + 1]++;
    for (int64_t J = 0; J < tnB; J++) cptr[J + 1] += cptr[J];
    for (int64_t J = 0; J < tnB; J++) fill[J] = cptr[J];
    for (int64_t K = 0; K < tmB; K++)
        for (int64_t q = tpB[K]; q < tpB[K + 1]; q++) {
            int64_t J = tcB[q];
            crow[fill[J]] = K;
            cpos[fill[J]] = q;
            fill[J]++;
        }
    for (int64_t t = 0; t < nc; t++) {
        int64_t I = cI[t], J = cJ[t];
        uint16_t mc[TILE];
        memset(mc, 0, sizeof(mc));
        int64_t pa = tpA[I], ea = tpA[I + 1], pb = cptr[J], eb = cptr[J + 1];
        int64_t matched = 0, contrib = 0;
        while (pa < ea && pb < eb) {
            int64_t ka = tcA[pa], kb = crow[pb];
            if (ka < kb) { pa++; continue; }
            if (kb < ka) { pb++; continue; }
            /* matched pair (A_IK, B_KJ) */
            matched++;
            const uint16_t *mA = maskA + pa * TILE, *mB = maskB + cpos[pb] * TILE;
            uint16_t colA = 0, rowB = 0;
            for (int r = 0; r < TILE; r++) {
                colA |= mA[r];
                if (mB[r]) rowB |= (uint16_t)(1u << r);
            }
            if (colA & rowB) contrib++;
            for (int r = 0; r < TILE; r++)
                for (int c = 0; c < TILE; c++)
                    if (mA[r] >> c & 1) mc[r] |= mB[c]; /* AtomicOr(mask_c, mask_b), line 23 */
            pa++;
            pb++;
        }
        int64_t nz = 0;
        for (int r = 0; r < TILE; r++) {
            mask_out[t * TILE + r] = mc[r];
            nz += __builtin_popcount(mc[r]);
        }
        nnz_out[t] = nz;
        if (matched_out) matched_out[t] = matched;
        if (contrib_out) contrib_out[t] = contrib;
    }
    free(cptr); free(crow); free(cpos); free(fill);
    return 0;
}

/* y = A x (plain CSR SpMV; used for the invariant C·1 = A·(B·1)) */
int orc_spmv(int64_t m, const int64_t *Arp, const int32_t *Aci, const double *Aval, const double *x,
             double *y) {
    for (int64_t i = 0; i < m; i++) {
        double s = 0.0;
        for (int64_t p = Arp[i]; p < Arp[i + 1]; p++) s = s + Aval[p] * x[Aci[p]];
        y[i] = s;
    }
    return 0;
}
