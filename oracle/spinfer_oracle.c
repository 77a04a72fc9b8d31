/*
 * spinfer_oracle.c — CPU ORACLE for the TCA-BME SpMM hot path.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load or call this library. The
 * product path (paper_conf_eurosys_fanydlgww025_b200/) never does, and shares
 * no code, header, table or constant generator with it.
 *
 * Plain, single-threaded, slow, obviously correct C. Floating point in fp64.
 * Every function cites the PAPER.md passage (P:<line>) it follows; readings of
 * silent/garbled points are DESIGN.md §"Readings of the paper" (A1..A16).
 *
 * Format (§4.2):
 *   BitmapTile (BT) 8x8, one uint64 bitmap, set bit = non-zero
 *   TCTile (TT) 16x16 = 2x2 BTs, column-major: TL,BL,TR,BR = Ra0..Ra3
 *   GroupTile (GT) GT_H x GT_W = 64x64 (reading A1); TTs column-major
 *   inside a GT; GTs row-major
 *   GTileOffset[NGT+1] int32, Values fp16 in nested GT->TT->BT order,
 *   Bitmap uint64 per BT (same nested order, reading A5)
 *   bit b of a BT <-> (row b/8, col b%8), LSB = (0,0)   (reading A2)
 *   values inside a BT in ascending bit order           (reading A3)
 *   each GT's value segment padded with +0.0 to a multiple of 8 halves
 *   (16 B) (reading A6); GTileOffset counts fp16 elements incl. padding
 *   non-zero <=> (bits & 0x7FFF) != 0 (reading A7)
 *
 * Parity pins: tests/test_oracle.py (brute-force index, round trip, counts,
 * eq. (9), checkerboard worked example, PTX m16n8k16 A-fragment layout,
 * dense-GEMM definition, integer exactness, identity).
 */
#include <stdint.h>
#include <stddef.h>
#include <string.h>
#include <stdlib.h>

#define O_GT 64   /* GT_H = GT_W = 64 (reading A1) */
#define O_TT 16   /* TCTile 16x16 */
#define O_BT 8    /* BitmapTile 8x8 */

enum { O_OK = 0, O_EINVAL = -1, O_EOVERFLOW = -3 };

/* ---- fp16 <-> fp64 (IEEE binary16), exact / round-to-nearest-even ---- */

double oracle_f16_to_f64(uint16_t h) {
    int s = (h >> 15) & 1, e = (h >> 10) & 0x1F, m = h & 0x3FF;
    double v;
    if (e == 0) v = (double)m * (1.0 / 16777216.0);                 /* m * 2^-24 */
    else if (e == 31) v = m ? (0.0 / 0.0) : (1.0 / 0.0);
    else { v = (double)(m | 0x400); int p = e - 25; while (p > 0) { v *= 2; --p; } while (p < 0) { v *= 0.5; ++p; } }
    return s ? -v : v;
}

/* RNE conversion by exhaustive nearest search over the finite halves
 * (obviously correct; used only for the integer-exact pins). */
uint16_t oracle_f64_to_f16(double d) {
    if (d != d) return 0x7E00;
    uint16_t best = 0; double bestd = -1.0;
    uint16_t sign = (d < 0) ? 0x8000 : 0;
    double a = d < 0 ? -d : d;
    if (a >= 65520.0) return (uint16_t)(sign | 0x7C00);
    for (uint32_t h = 0; h < 0x7C00; ++h) {
        double diff = oracle_f16_to_f64((uint16_t)h) - a;
        if (diff < 0) diff = -diff;
        if (bestd < 0 || diff < bestd || (diff == bestd && (h & 1) == 0)) { bestd = diff; best = (uint16_t)h; }
    }
    return (uint16_t)(sign | best);
}

static int nonzero16(uint16_t bits) { return (bits & 0x7FFF) != 0; }   /* reading A7 */

/* ---- sizes, eq. (9) ---- */

/* Reading A8: a shape that is not a multiple of the GT is zero-padded to the next multiple of 64
 * in both dimensions (elements outside M x K are zeros: no bit set, no value stored). */
static int cdiv(int a, int b) { return (a + b - 1) / b; }
int64_t oracle_ngt(int M, int K) { return (int64_t)cdiv(M, O_GT) * cdiv(K, O_GT); }   /* NGT */
int64_t oracle_nbt(int M, int K) { return oracle_ngt(M, K) * 64; }                      /* NBT */

/* Stor_TCA-BME = 4B(NGT+1) + 8B*NBT + 2B*NNZ, eq. (9) P:210. Pass n_values
 * (padded count) to get the buffer size actually allocated, nnz for eq. (9). */
int64_t oracle_storage_bytes(int M, int K, int64_t n_values) {
    return 4 * (oracle_ngt(M, K) + 1) + 8 * oracle_nbt(M, K) + 2 * n_values;
}

/* CR = 2B*M*K / Stor, eq. (1) P:109. */
double oracle_compression_ratio(int M, int K, int64_t n_values) {
    return 2.0 * (double)M * (double)K / (double)oracle_storage_bytes(M, K, n_values);
}

static int valid_shape(int M, int K) {
    return M > 0 && K > 0;   /* any shape, zero-padded to whole GroupTiles (reading A8) */
}

/* W[r][c] of the zero-padded matrix (reading A8) */
static uint16_t w_at(const uint16_t *W, int M, int K, int r, int c) {
    return (r < M && c < K) ? W[(size_t)r * K + c] : (uint16_t)0;
}

/* Element (r, c) of BT number `bt` (0..3, column-major in the TT) of
 * TCTile number `tt` (column-major in the GT) of GT (gr, gc), bit b. */
static void bt_elem(int gr, int gc, int tt, int bt, int b, int *r, int *c) {
    int tr = tt % 4, tc = tt / 4;          /* TCTiles column-major inside the GT */
    int br = bt % 2, bc = bt / 2;          /* BTs column-major inside the TT: TL,BL,TR,BR */
    *r = gr * O_GT + tr * O_TT + br * O_BT + b / 8;   /* bit b <-> (b/8, b%8) (reading A2) */
    *c = gc * O_GT + tc * O_TT + bc * O_BT + b % 8;
}

/* ---- C1: encode, step by step ---- */

/* Counts only: nnz and padded n_values. */
int oracle_encode_count(const uint16_t *W, int M, int K, int64_t *nnz, int64_t *n_values, int32_t *max_gt_values) {
    if (!W || !valid_shape(M, K)) return O_EINVAL;
    int64_t running = 0, z = 0; int32_t mx = 0;
    for (int gr = 0; gr < cdiv(M, O_GT); ++gr)
        for (int gc = 0; gc < cdiv(K, O_GT); ++gc) {      /* GTs row-major */
            int64_t start = running;
            for (int tt = 0; tt < 16; ++tt)
                for (int bt = 0; bt < 4; ++bt)
                    for (int b = 0; b < 64; ++b) {
                        int r, c; bt_elem(gr, gc, tt, bt, b, &r, &c);
                        if (nonzero16(w_at(W, M, K, r, c))) { ++running; ++z; }
                    }
            while (running % 8 != 0) ++running;           /* 16-B padding (reading A6) */
            if (running - start > mx) mx = (int32_t)(running - start);
        }
    if (running >= ((int64_t)1 << 31)) return O_EOVERFLOW;           /* reading A9 */
    if (nnz) *nnz = z;
    if (n_values) *n_values = running;
    if (max_gt_values) *max_gt_values = mx;
    return O_OK;
}

/* Full encode into caller buffers: gtile_offset[NGT+1], bitmap[NBT], values[n_values]. */
int oracle_encode(const uint16_t *W, int M, int K, int32_t *gtile_offset, uint64_t *bitmap, uint16_t *values) {
    if (!W || !gtile_offset || !bitmap || !valid_shape(M, K)) return O_EINVAL;
    int64_t running = 0;
    int KG = cdiv(K, O_GT);
    for (int gr = 0; gr < cdiv(M, O_GT); ++gr)
        for (int gc = 0; gc < KG; ++gc) {                 /* GTs row-major */
            int64_t g = (int64_t)gr * KG + gc;
            gtile_offset[g] = (int32_t)running;           /* start of GT g's values */
            for (int tt = 0; tt < 16; ++tt)               /* TCTiles column-major */
                for (int bt = 0; bt < 4; ++bt) {          /* BTs column-major: Ra0..Ra3 */
                    uint64_t bm = 0;
                    for (int b = 0; b < 64; ++b) {
                        int r, c; bt_elem(gr, gc, tt, bt, b, &r, &c);
                        uint16_t v = w_at(W, M, K, r, c);
                        if (nonzero16(v)) {
                            bm |= (uint64_t)1 << b;                  /* set bit = non-zero */
                            values[running++] = v;                   /* nested order */
                        }
                    }
                    bitmap[(g * 16 + tt) * 4 + bt] = bm;             /* reading A5 */
                }
            while (running % 8 != 0) values[running++] = 0x0000;     /* reading A6 */
        }
    gtile_offset[oracle_ngt(M, K)] = (int32_t)running;
    return O_OK;
}

/* ---- C2: decode (inverse of C1); unset bits become +0.0 ---- */
int oracle_decode(const int32_t *gtile_offset, const uint64_t *bitmap, const uint16_t *values,
                  int M, int K, uint16_t *W_out) {
    if (!gtile_offset || !bitmap || !W_out || !valid_shape(M, K)) return O_EINVAL;
    int KG = cdiv(K, O_GT);
    for (int gr = 0; gr < cdiv(M, O_GT); ++gr)
        for (int gc = 0; gc < KG; ++gc) {
            int64_t g = (int64_t)gr * KG + gc;
            int64_t pos = gtile_offset[g];
            for (int tt = 0; tt < 16; ++tt)
                for (int bt = 0; bt < 4; ++bt) {
                    uint64_t bm = bitmap[(g * 16 + tt) * 4 + bt];
                    for (int b = 0; b < 64; ++b) {
                        int r, c; bt_elem(gr, gc, tt, bt, b, &r, &c);
                        uint16_t v = ((bm >> b) & 1) ? values[pos++] : 0x0000;
                        if (r < M && c < K) W_out[(size_t)r * K + c] = v;   /* padding dropped (A8) */
                    }
                }
        }
    return O_OK;
}

/* ---- C3: SpMM ---- */

/* The plain definition Y = W x X, fp64: Y[i][n] = sum_k W[i][k] X[k][n]. */
void oracle_gemm_f64(const uint16_t *W, const uint16_t *X, int M, int K, int N, double *Y) {
    for (int i = 0; i < M; ++i)
        for (int n = 0; n < N; ++n) {
            double acc = 0.0;
            for (int k = 0; k < K; ++k)
                acc += oracle_f16_to_f64(W[(size_t)i * K + k]) * oracle_f16_to_f64(X[(size_t)k * N + n]);
            Y[(size_t)i * N + n] = acc;
        }
}

/* SpMM that walks the TCA-BME arrays directly: for every GT (row-major),
 * TCTile, BitmapTile in storage order, each set bit b contributes
 * value * X[col][:] to Y[row][:]. Y [M][N] fp64 is overwritten. */
int oracle_spmm_tca_f64(const int32_t *gtile_offset, const uint64_t *bitmap, const uint16_t *values,
                        const uint16_t *X, int M, int K, int N, double *Y) {
    if (!gtile_offset || !bitmap || !X || !Y || !valid_shape(M, K) || N <= 0) return O_EINVAL;
    memset(Y, 0, sizeof(double) * (size_t)M * N);
    int KG = cdiv(K, O_GT);
    double *xrow = (double *)malloc(sizeof(double) * (size_t)N);
    for (int gr = 0; gr < cdiv(M, O_GT); ++gr)
        for (int gc = 0; gc < KG; ++gc) {
            int64_t g = (int64_t)gr * KG + gc;
            int64_t pos = gtile_offset[g];
            for (int tt = 0; tt < 16; ++tt)
                for (int bt = 0; bt < 4; ++bt) {
                    uint64_t bm = bitmap[(g * 16 + tt) * 4 + bt];
                    for (int b = 0; b < 64; ++b) {
                        if (!((bm >> b) & 1)) continue;
                        int r, c; bt_elem(gr, gc, tt, bt, b, &r, &c);
                        double w = oracle_f16_to_f64(values[pos++]);
                        if (r >= M || c >= K) return O_EINVAL;   /* a bit in the padding: not an encoding */
                        for (int n = 0; n < N; ++n) xrow[n] = oracle_f16_to_f64(X[(size_t)c * N + n]);
                        for (int n = 0; n < N; ++n) Y[(size_t)r * N + n] += w * xrow[n];
                    }
                }
        }
    free(xrow);
    return O_OK;
}

/* Same walk restricted to a list of output rows (for sampled parity at full size).
 * Yrows [nrows][N]. For each requested row: locate its GT row, walk each GT of
 * that row in storage order, advancing the value cursor over every set bit and
 * accumulating only the bits that fall on the requested row. */
int oracle_spmm_tca_rows_f64(const int32_t *gtile_offset, const uint64_t *bitmap, const uint16_t *values,
                             const uint16_t *X, int M, int K, int N,
                             const int32_t *rows, int nrows, double *Yrows) {
    if (!gtile_offset || !bitmap || !X || !Yrows || !rows || !valid_shape(M, K) || N <= 0) return O_EINVAL;
    int KG = cdiv(K, O_GT);
    for (int q = 0; q < nrows; ++q) {
        int row = rows[q];
        if (row < 0 || row >= M) return O_EINVAL;
        double *y = Yrows + (size_t)q * N;
        for (int n = 0; n < N; ++n) y[n] = 0.0;
        int gr = row / O_GT;
        for (int gc = 0; gc < KG; ++gc) {
            int64_t g = (int64_t)gr * KG + gc;
            int64_t pos = gtile_offset[g];
            for (int tt = 0; tt < 16; ++tt)
                for (int bt = 0; bt < 4; ++bt) {
                    uint64_t bm = bitmap[(g * 16 + tt) * 4 + bt];
                    for (int b = 0; b < 64; ++b) {
                        if (!((bm >> b) & 1)) continue;
                        int r, c; bt_elem(gr, gc, tt, bt, b, &r, &c);
                        uint16_t v = values[pos++];
                        if (r != row) continue;
                        if (c >= K) return O_EINVAL;              /* a bit in the padding */
                        double w = oracle_f16_to_f64(v);
                        for (int n = 0; n < N; ++n) y[n] += w * oracle_f16_to_f64(X[(size_t)c * N + n]);
                    }
                }
        }
    }
    return O_OK;
}

/* ---- C4: SMBD lane emulator (Alg. 2) ----
 * For one BitmapTile `bitmap` whose non-zeros start at `bt_values`, lane l
 * (0..31) decodes its two halves a0, a1 of the .f16x2 register:
 *   Phase I : bit 2l set -> a0 = V[MaskedPopCount(b, l)], else 0
 *   Phase II: bit 2l+1 set -> a1 = V[count + (a0 was non-zero)], else 0
 * MaskedPopCount(b, l) = PopCount(b & ((1 << 2l) - 1)), 64-bit shift (A4). */
int oracle_masked_popcount(uint64_t b, int lane) {
    int offset = lane * 2;                                  /* Alg. 2 line 1 */
    uint64_t mask = ((uint64_t)1 << offset) - 1;            /* line 2 (64-bit, A4) */
    uint64_t x = b & mask; int cnt = 0;                     /* line 3: PopCount */
    while (x) { cnt += (int)(x & 1); x >>= 1; }
    return cnt;                                             /* line 4 */
}

void oracle_smbd_lane(uint64_t bitmap, const uint16_t *bt_values, int lane, uint16_t *a0, uint16_t *a1) {
    int count = oracle_masked_popcount(bitmap, lane);
    int b0 = (int)((bitmap >> (2 * lane)) & 1), b1 = (int)((bitmap >> (2 * lane + 1)) & 1);
    *a0 = b0 ? bt_values[count] : 0;                        /* Phase I */
    *a1 = b1 ? bt_values[count + b0] : 0;                   /* Phase II: reuse count (+1 if a0 loaded) */
}

/* One TCTile (4 BTs in storage order, Ra0..Ra3 = TL,BL,TR,BR) whose
 * values start at tt_values: BT j's values begin after PopCount of BTs < j
 * (P:274). Lane's 4 registers, each (a1 << 16) | a0 (.f16x2, low half = a0). */
void oracle_smbd_tctile(const uint64_t bm[4], const uint16_t *tt_values, int lane, uint32_t ra[4]) {
    int base = 0;
    for (int j = 0; j < 4; ++j) {
        uint16_t a0, a1;
        oracle_smbd_lane(bm[j], tt_values + base, lane, &a0, &a1);
        ra[j] = ((uint32_t)a1 << 16) | a0;
        uint64_t x = bm[j];                                 /* PopCount of the whole BT */
        while (x) { base += (int)(x & 1); x >>= 1; }
    }
}

/* ---- C6: tensor-parallel row partition ----
 * Rank r of `world` owns GT rows [r*q + min(r, rem), ...) with q = MG / world,
 * rem = MG % world: contiguous, multiples of 64 rows, sizes differ by <= 1 GT row. */
int oracle_tp_rows(int M, int world, int rank, int *row_begin, int *row_count) {
    if (M <= 0 || world <= 0 || rank < 0 || rank >= world || !row_begin || !row_count) return O_EINVAL;
    int MG = cdiv(M, O_GT), q = MG / world, rem = MG % world;
    int gb = rank * q + (rank < rem ? rank : rem);
    int gn = q + (rank < rem ? 1 : 0);
    *row_begin = gb * O_GT;
    *row_count = gn * O_GT;
    if (*row_begin > M) *row_begin = M;                    /* A8: the ragged tail belongs to the */
    if (*row_begin + *row_count > M) *row_count = M - *row_begin;   /* rank owning the last GT row */
    return O_OK;
}

/* ---- C7: fused FC epilogue (the OPT FC1 layers run bias + ReLU after the
 * SpMM): Y[i][n] = act(Y[i][n] + bias[i]) in fp64, act 0 = identity, 1 = ReLU
 * (max(v, 0)). bias may be NULL (no bias). Applied to the exact fp64 product of C3. */
int oracle_bias_act_f64(double *Y, int M, int N, const uint16_t *bias, int act) {
    if (!Y || M < 0 || N < 0 || (act != 0 && act != 1)) return O_EINVAL;
    for (int i = 0; i < M; ++i) {
        const double b = bias ? oracle_f16_to_f64(bias[i]) : 0.0;
        for (int n = 0; n < N; ++n) {
            double v = Y[(size_t)i * N + n] + b;
            if (act == 1 && v < 0.0) v = 0.0;
            Y[(size_t)i * N + n] = v;
        }
    }
    return O_OK;
}
