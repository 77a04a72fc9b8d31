/*
 * spinfer.h — C ABI of the B200 (sm_100a) TCA-BME SpMM library (libspinfer.so).
 *
 * The operation (§2.1, §2.3): Y = W x X with
 *   W in R^{M x K}  — an fp16 weight matrix, unstructured-sparse (30-70% zeros,
 *                     P:13), stored in TCA-BME (§4.2);
 *   X in R^{K x N}  — fp16 activations, N = decode tokens;
 *   Y in R^{M x N}  — fp16 output, fp32 accumulation (Listing 1).
 *
 * TCA-BME: 8x8 BitmapTiles (one uint64 bitmap each) grouped
 * 2x2 column-major into 16x16 TCTiles, TCTiles column-major inside
 * 64x64 GroupTiles, GroupTiles row-major. Three arrays:
 *   gtile_offset int32[NGT+1], NGT = ceil(M/64) ceil(K/64): start (in fp16 elements) of
 *                each GroupTile's values, gtile_offset[0] = 0,
 *                gtile_offset[NGT] = n_values;
 *   bitmap       uint64[NBT], NBT = 64 NGT, in GroupTile -> TCTile -> BitmapTile
 *                order; bit b <-> (row b/8, col b%8) of the BitmapTile;
 *   values       fp16[n_values], non-zeros in the same nested order, ascending
 *                bit order inside a BitmapTile; each GroupTile's
 *                segment is padded with +0.0 to a multiple of 8 halves (16 B,
 *                P:266). Storage = eq. (9) + padding (<= 7 halves/GT).
 * "Non-zero" means (bits & 0x7FFF) != 0: -0.0 is dropped, NaN/Inf are kept.
 * M and K need not be multiples of 64: the matrix is zero-padded to whole
 * GroupTiles (no bit set and no value stored in the padding, A8).
 * All readings of silent/garbled points are listed in DESIGN.md.
 *
 * Conventions for every call:
 *  - Pointers are DEVICE pointers unless marked (host). fp16 is passed as
 *    uint16_t bit patterns. Matrices are row-major and contiguous.
 *  - Device pointers must be 16-byte aligned (cp.async.bulk requirement).
 *  - All buffers are owned and allocated by the CALLER; the library keeps no
 *    state and allocates no persistent memory (encode_count uses one 64-byte
 *    stream-ordered temporary). Calls are stream-ordered and asynchronous
 *    except spinfer_encode_count, which synchronizes `stream`.
 *  - Every function returns a spinfer_status; nothing aborts, no exception
 *    crosses the ABI. Asynchronous device faults surface at the caller's next
 *    synchronization (as a CUDA error there).
 *  - `stream` is a cudaStream_t passed as void* (0 = legacy default stream).
 *  - Requires an sm_100 device (SPINFER_ENODEV otherwise).
 */
#ifndef SPINFER_H_
#define SPINFER_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    SPINFER_OK = 0,
    SPINFER_EINVAL = -1,     /* null pointer, bad shape (M or K <= 0, N not in [1, 65536]),
                                misaligned pointer, struct/call mismatch, unknown activation */
    SPINFER_ENOSPC = -2,     /* workspace too small */
    SPINFER_EOVERFLOW = -3,  /* n_values would reach 2^31 (gtile_offset is int32) */
    SPINFER_ECUDA = -4,      /* CUDA launch/runtime error */
    SPINFER_ENODEV = -5      /* current device is not sm_100 */
} spinfer_status;

#if defined(__GNUC__)
#define SPINFER_API __attribute__((visibility("default")))
#else
#define SPINFER_API
#endif

#define SPINFER_GT 64        /* GroupTile edge GT_H = GT_W (paper silent; reading A1) */

/* Host-side descriptor of one TCA-BME matrix. The three device arrays are
 * caller-owned (e.g. torch tensors). */
typedef struct {
    int32_t M, K;             /* > 0 (not necessarily multiples of 64: zero-padded GroupTiles) */
    int32_t gt_h, gt_w;       /* must be 64, 64 */
    int64_t nnz;              /* true non-zeros (informational) */
    int64_t n_values;         /* == gtile_offset[NGT] (padded count), < 2^31 */
    int32_t max_gt_values;    /* max_g (gtile_offset[g+1]-gtile_offset[g]) — sizes the SpMM
                                 pipeline stages; <= 0 means unknown (assume 4096, dense) */
    int32_t reserved;
    int32_t *gtile_offset;    /* device [NGT+1] */
    uint64_t *bitmap;         /* device [NBT] */
    uint16_t *values;         /* device [max(n_values,8)] fp16 bits */
} spinfer_tca;

/* Encode, phase 1 (P:196 sizes; GPU encoder, not described by the paper).
 * W: device fp16 [M][K]. Writes gtile_offset[0..NGT] (device, caller-allocated
 * NGT+1 int32) and returns to the HOST n_values (padded), nnz and max_gt_values.
 * Synchronizes `stream`. SPINFER_EOVERFLOW if n_values >= 2^31. */
SPINFER_API int spinfer_encode_count(const uint16_t *W, int M, int K, int32_t *gtile_offset,
                         int64_t *n_values /* host */, int64_t *nnz /* host */,
                         int32_t *max_gt_values /* host, may be NULL */, void *stream);

/* Encode, phase 2: fills T->bitmap (NBT uint64) and T->values (n_values fp16,
 * padding written as +0.0) from W, using T->gtile_offset from phase 1.
 * T (host struct) must carry M, K, gt_h = gt_w = 64 and the three device pointers. */
SPINFER_API int spinfer_encode_fill(const uint16_t *W, const spinfer_tca *T, void *stream);

/* Decode TCA-BME -> dense fp16 W_out [M][K] (device); unset bits give +0.0. */
SPINFER_API int spinfer_decode(const spinfer_tca *T, uint16_t *W_out, void *stream);

/* Bytes of device workspace spinfer_spmm needs for this shape: a fixed 64 KiB
 * region of split-K fix-up counters (one int32 per GT row; ceil(M/64) < 16383)
 * whose last int32 (byte offset 65532) is the ERROR WORD, followed by fp32
 * split-K partials and, when N is not a multiple of 8, a zero-padded copy of X
 * (K x roundup(N, 8) fp16). 0 for an invalid shape. The workspace must be
 * ZERO-FILLED before its first use; every spinfer_spmm call leaves the counter
 * region zero again, so one zeroed workspace (sized for the largest shape) can
 * be reused by successive calls of any shape on ONE stream — never by two calls
 * that may run concurrently. The grid (and so the partials' size) depends on
 * the device's SM count and SPINFER_OPT_MAX_CTAS: query after setting options. */
SPINFER_API size_t spinfer_spmm_workspace_bytes(int M, int K, int N);

/* Y = W x X with fp32 accumulation and one round-to-nearest-even to
 * fp16 per output. X: device fp16 [K][N] row-major; Y: device fp16
 * [M][N] row-major (fully overwritten). 1 <= N <= 65536. One persistent kernel launch:
 *   N <= 16  (decode batch): mma.sync SMBD kernel, stream-K over GroupTiles with an
 *            in-kernel split-K fix-up (P:216 / Alg. 1);
 *   N 17-32: the same decomposition on tcgen05 with the accumulators in TMEM;
 *   N > 32   (prefill): tcgen05 with W decoded into shared memory, 128-row x
 *            (up to) 512-column output tiles, no split-K.
 * N not a multiple of 8 costs the same as the next multiple of 8 plus a zero-padded copy of
 * X in the workspace. For N <= 32, K <= 4,194,240 (at most 65535 GroupTile columns: the stage
 * headers pack the column index in 16 bits) and ceil(M/64) < 16383; SPINFER_EINVAL otherwise. */
SPINFER_API int spinfer_spmm(const spinfer_tca *T, const uint16_t *X, uint16_t *Y, int M, int K, int N,
                 void *workspace, size_t ws_bytes, void *stream);

/* Y = act(W x X + bias) with the epilogue fused into the SpMM kernels (SURVEY §8(f) rank 4:
 * the FC1 layers of the paper's OPT models run bias + ReLU after the SpMM).
 * bias: device fp16 [M] (one value per output row) or NULL (no bias). act: SPINFER_ACT_NONE or
 * SPINFER_ACT_RELU. The bias is added to the fp32 accumulator, the activation applied in fp32,
 * then one RNE to fp16 per output. Everything else as spinfer_spmm (which is this call with
 * bias = NULL, act = SPINFER_ACT_NONE). SPINFER_EINVAL for an unknown act or a bias not 2-byte
 * aligned. */
#define SPINFER_ACT_NONE 0
#define SPINFER_ACT_RELU 1
SPINFER_API int spinfer_spmm_ex(const spinfer_tca *T, const uint16_t *X, uint16_t *Y, int M, int K, int N,
                                const uint16_t *bias, int act, void *workspace, size_t ws_bytes, void *stream);

/* Tensor-parallel row partition: rank `rank` of `world` owns rows
 * [*row_begin, *row_begin + *row_count) — contiguous, whole GroupTile rows (multiples of 64;
 * the ragged tail of an M that is not a multiple of 64 goes to the rank owning the last GT
 * row), sizes differ by at most 64; ranks beyond the GT-row count get 0 rows (host only). */
SPINFER_API int spinfer_tp_rows(int M, int world, int rank, int *row_begin /* host */, int *row_count /* host */);

/* Zero-copy row shard of a TCA-BME matrix (P:196 — GroupTiles are stored
 * row-major, so the GT rows [row_begin/64, ceil((row_begin+row_count)/64)) are one contiguous
 * slice of all three arrays). row_begin must be a multiple of 64, row_count a multiple of 64
 * unless the shard ends at T->M (the ragged tail, A8); typically the span
 * spinfer_tp_rows returns. Writes the shard's GTileOffset, rebased to start at 0, into
 * offset_out (caller-allocated DEVICE int32[ceil(row_count/64) * ceil(K/64) + 1], 16-byte
 * aligned) and fills *out (host): M = row_count, K, n_values and max_gt_values (T's, an upper
 * bound) set, nnz = -1 (unknown), bitmap and values pointing INTO T's arrays (aligned: every
 * GroupTile's values start at a multiple of 8 halves). T's buffers must outlive *out.
 * Synchronizes `stream` (the shard's value count is read back). */
SPINFER_API int spinfer_tca_shard(const spinfer_tca *T, int row_begin, int row_count, int32_t *offset_out,
                                  spinfer_tca *out /* host */, void *stream);

/* Row-partitioned SpMM: T_shard encodes W[row_begin : row_begin+row_count, :]
 * (as returned by spinfer_tp_rows(M_full, world, rank)); writes ONLY those rows
 * of Y_full [M_full][N]. Performs no communication: the caller gathers Y_full
 * (e.g. NCCL all-gather) when the next layer needs it. */
SPINFER_API int spinfer_spmm_tp(const spinfer_tca *T_shard, const uint16_t *X, uint16_t *Y_full, int M_full,
                    int K, int N, int world, int rank, void *workspace, size_t ws_bytes, void *stream);

/* Fused all-gather epilogue (the exchange the paper blames for its shrinking
 * multi-GPU gains): spinfer_spmm_tp whose kernel also stores this rank's rows of Y
 * directly into every rank's Y_full (peer stores over NVLink / NVSwitch, no NCCL), followed by one
 * release increment of every rank's completion counter.
 *   Y_full_peers: HOST array [world] of DEVICE pointers: rank r's Y_full [M_full][N] as mapped in
 *                 this process (CUDA IPC / torch symmetric memory; on one device, plain pointers);
 *   flag_peers:   HOST array [world] of DEVICE pointers to each rank's uint32 counter (zeroed once).
 * world <= 8, N <= 16 (the decode regime; SPINFER_EINVAL otherwise), no bias / activation. Rank r's
 * Y_full holds every rank's rows once its spinfer_gather_wait has returned (on its stream). */
SPINFER_API int spinfer_spmm_tp_gather(const spinfer_tca *T_shard, const uint16_t *X, uint16_t *const *Y_full_peers,
                                       int M_full, int K, int N, int world, int rank, uint32_t *const *flag_peers,
                                       void *workspace, size_t ws_bytes, void *stream);

/* Stream-ordered wait (one device thread) until every rank's signal of the current exchange reached
 * this rank's counter `flag` (device). `state` (device uint32, zeroed together with the counter)
 * holds the expected count, so a captured CUDA graph replays the exchange correctly. timeout_us > 0
 * bounds the wait: on expiry flag 4 is OR-ed into the workspace's error word (if workspace is not
 * NULL) and the wait returns. */
SPINFER_API int spinfer_gather_wait(uint32_t *flag, uint32_t *state, int world, void *workspace, uint32_t timeout_us,
                                    void *stream);

/* Corrupt-input report. The kernels check every stage they load against the TCA-BME
 * invariants (gtile_offset non-decreasing and <= n_values, a GroupTile's popcount equal to
 * its padded value count rounded down by < 8, at most max_gt_values values per GroupTile):
 * a violating stage is not copied / decoded (its rows' contribution is zero, so Y is NOT
 * valid) and a flag is OR-ed into the workspace's error word — 1: gtile_offset out of range
 * or larger than max_gt_values; 2: bitmaps inconsistent with gtile_offset; 4: a
 * spinfer_gather_wait timed out. No out-of-bounds
 * access happens either way. This call copies the error word to *flags (host), resets it to
 * 0 and synchronizes `stream`. */
SPINFER_API int spinfer_spmm_check(void *workspace, int32_t *flags /* host */, void *stream);

/* Process-wide options (tests, ablation, tuning). 0 is every option's default. Not
 * synchronized with calls running on other host threads: set them before launching work.
 *   SPINFER_OPT_KERNEL    0 auto (N <= 16: the mma.sync decoupled-warp kernel, else tcgen05),
 *                         1 force the decoupled-warp kernel (N <= 32; N 17-32 run its half-GroupTile
 *                         mode: X padded to 32 columns, two warps per GroupTile), 2 force tcgen05;
 *   SPINFER_OPT_MAX_CTAS  cap on the persistent grid (0: one CTA per SM);
 *   SPINFER_OPT_STAGE_G   cap on GroupTile columns per pipeline stage (0: the kernel's max);
 *   SPINFER_OPT_STAGE_S   cap on pipeline stages (0: as many as shared memory holds);
 *   SPINFER_OPT_WIDE_BN   N > 32 kernel: cap on the MMA N of a sub-tile (multiple of 16; 0: 256);
 *   SPINFER_OPT_PDL       1: launch the N <= 32 kernels (decoupled-warp and tcgen05) with programmatic dependent
 *                         launch (cudaLaunchAttributeProgrammaticStreamSerialization): its CTAs start
 *                         as the previous kernel's CTAs retire and stream the first stages' weights
 *                         (GTileOffset, bitmaps, values) while that kernel finishes; X, the workspace
 *                         and Y are touched only after griddepcontrol.wait, i.e. after the previous
 *                         grid completed. For chains of SpMMs on one stream (a layer stack). The
 *                         weights must not be written by the immediately preceding kernel unless that
 *                         kernel is one of this library's encoders (they never trigger early).
 * SPINFER_EINVAL for an unknown key or an out-of-range value. */
#define SPINFER_OPT_KERNEL 0
#define SPINFER_OPT_MAX_CTAS 1
#define SPINFER_OPT_STAGE_G 2
#define SPINFER_OPT_STAGE_S 3
#define SPINFER_OPT_WIDE_BN 4
#define SPINFER_OPT_PDL 5
#define SPINFER_OPT_COUNT 6
#define SPINFER_KERNEL_AUTO 0
#define SPINFER_KERNEL_DW 1
#define SPINFER_KERNEL_TC 2
SPINFER_API int spinfer_set_option(int key, int value);
SPINFER_API int spinfer_get_option(int key);

/* Static string for a status code. */
SPINFER_API const char *spinfer_status_str(int status);

/* Library build/version info (host string). */
SPINFER_API const char *spinfer_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SPINFER_H_ */
