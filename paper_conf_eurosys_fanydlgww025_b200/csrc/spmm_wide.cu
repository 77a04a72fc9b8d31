// spmm_wide.cu — TCA-BME SpMM Y = W x X for wide X (N > 32: prefill; the
// paper's large-N comparison, §5.5) on the tcgen05 tensor cores.
//
// At large N the product is compute-bound and W's decode cost is amortised over the N columns a
// CTA multiplies: the SMBD decode (MaskedPopCount, Alg. 2, with warp-scanned PopCount
// bases as in spmm_dw.cu) writes each 128 x 64 W tile densely into SHARED memory in the UMMA
// canonical K-major SWIZZLE_128B layout, and one thread issues tcgen05.mma (M = 128, N = bn <= 256,
// K = 16, A and B from shared-memory descriptors, fp32 D in TMEM) for up to two N sub-tiles.
// One persistent CTA per SM walks output tiles (128 rows x nsub * bn columns) in a grouped order
// (16 rowblocks x the column tiles) so that the rowblocks' compressed W and the X column tiles in
// flight stay in L2. Warp roles (one CTA, 16 warps):
//   0      W producer: per K-step (one GroupTile column) the two GT rows' packed values and bitmaps
//          (bulk copies from different lanes of one instruction) into a W ring;
//   1      X producer: the X tile rows [64 gc, 64 gc + 64) x the tile's columns (tensor TMA, 64 x 64
//          boxes, SWIZZLE_128B = the UMMA MN-major canonical layout); owns the TMEM allocation;
//   2      MMA issuer (one thread): 4 K-steps of 16 per stage and sub-tile, commits release the
//          A / X slots and, after a tile's last K-step, hand the accumulator to the epilogue;
//   4-7,   epilogue: TMEM lane quarter q = warp & 3 -> fp16 (+ bias / ReLU) -> Y; warps 4-7 the
//   24-27  even 32-column chunks of each sub-tile, 24-27 the odd ones;
//   8-23   decode: warp d decodes TCTile column (d >> 1) & 3 of GT row d & 1 in the K-steps of parity
//          d >> 3 (its own PopCount scan of the GT, 16 BitmapTiles), two K-steps in flight.
// Tile rows past M and columns past N are computed on zero-filled / garbage operands and never
// stored; K past the matrix is zero (bitmaps of the padding are empty, X rows are TMA-zero-filled).
#include <cuda.h>
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include "internal.cuh"
#include "ptx.cuh"

namespace spinfer {
namespace {

constexpr int kWThreads = 28 * 32;
constexpr int kWWProd = 0, kWXProd = 1, kWMma = 2, kWEpi0 = 4, kWDec0 = 8, kWEpi1 = 24;
constexpr int kWDecWarps = 16;
constexpr int kWMaxSA = 4, kWMaxSX = 4, kWMaxSW = 8;
constexpr uint32_t kWABytes = 128 * 128;         // decoded A tile: 128 rows x 64 K fp16
constexpr uint32_t kWBox = 64 * 64 * 2;          // one X box: 64 K rows x 64 N (128 B rows)
constexpr uint32_t kWTblBytes = 256;             // a decode warp's SMBD table: 16 BTs x 2 halves x 8 B
constexpr uint32_t kWHdr = 16;                   // per W stage: value count of each GT row (halves)
// barrier region (bytes from the 1024-aligned smem base)
constexpr uint32_t kWBarWFull = 0, kWBarWEmpty = 64, kWBarXFull = 128, kWBarXEmpty = 160, kWBarAFull = 192,
                   kWBarAEmpty = 224, kWBarDFull = 256, kWBarDEmpty = 264, kWTmemSlot = 272, kWHdrOff = 512;
constexpr uint32_t kSelAw = 0x7f62u, kSelBw = 0x4cbfu, kSelCw = 0x2333u;   // SMBD selector (spmm_dw.cu)

struct WParams {
    CUtensorMap tmap_x;          // X [K][Np] fp16, box {64, 64}, SWIZZLE_128B
    const int32_t *off;
    const uint64_t *bm;
    const uint16_t *vals;
    uint16_t *Y;
    const uint16_t *bias;        // fp16 [M] or null
    int act;
    int32_t *ws_err;
    int M, N, KG, MG, RB;        // RB = rowblocks of 128 rows
    int nsub, bn, bps;           // MMA sub-tiles per tile, MMA N, X boxes per sub-tile
    int ntn, tiles, group;       // column tiles, tiles, rowblocks per raster group
    int SA, SX, SW;              // ring depths
    uint32_t o_a, o_x, o_w, o_tbl;
    uint32_t x_bytes, w_stage, w_v1, vcap;   // X stage bytes; W stage bytes, row-1 values offset, value bytes per row
    int n_values;
    uint32_t idesc;
    long long *prof;             // experiments only (SPINFER_INSTRUMENT): [CTA][warp][4] cycle counters
};

#ifndef SPINFER_INSTRUMENT
#define SPINFER_INSTRUMENT 0
#endif
// Per-warp cycle accounting (instrumented build only): k0 waiting on the input barrier, k1 waiting
// on the output slot, k2 working, k3 total.
struct WProf {
#if SPINFER_INSTRUMENT
    long long c[4] = {0, 0, 0, 0}, t = 0, t0 = 0;
    __device__ __forceinline__ void start() { t0 = t = clock64(); }
    __device__ __forceinline__ void lap(int k) { const long long n = clock64(); c[k] += n - t; t = n; }
    __device__ __forceinline__ void dump(long long *p, int cta, int w, int lane) {
        c[3] = clock64() - t0;
        if (p && lane == 0) for (int k = 0; k < 4; ++k) p[((size_t)cta * 32 + w) * 4 + k] = c[k];
    }
#else
    __device__ __forceinline__ void start() {}
    __device__ __forceinline__ void lap(int) {}
    __device__ __forceinline__ void dump(long long *, int, int, int) {}
#endif
};

__device__ __forceinline__ void tile_coords(const WParams &q, int t, int &rb, int &nt) {
    const int per_group = q.group * q.ntn;
    const int g = t / per_group, idx = t - g * per_group;
    const int rows = min(q.group, q.RB - g * q.group);
    rb = g * q.group + idx % rows;
    nt = idx / rows;
}

// UMMA shared-memory descriptors (SM100 format: start >> 4 [0,14), LBO >> 4 [16,30), SBO >> 4
// [32,46), version 1 at bit 46, layout type [61,64): 2 = SWIZZLE_128B)
__device__ __forceinline__ uint64_t desc_sw128(uint32_t start, uint32_t lbo, uint32_t sbo) {
    return (uint64_t)((start >> 4) & 0x3FFFu) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46) | (2ull << 61);
}

__global__ void __launch_bounds__(kWThreads, 1) k_spmm_wide(const __grid_constant__ WParams q) {
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *const smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    const uint32_t sbase = smem_u32(smem);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int KG = q.KG;
    const uint32_t bwf = sbase + kWBarWFull, bwe = sbase + kWBarWEmpty, bxf = sbase + kWBarXFull,
                   bxe = sbase + kWBarXEmpty, baf = sbase + kWBarAFull, bae = sbase + kWBarAEmpty,
                   bdf = sbase + kWBarDFull, bde = sbase + kWBarDEmpty;
    if (threadIdx.x == 0) {
        for (int s = 0; s < q.SW; ++s) {
            mbar_init(bwf + 8 * s, 32);                      // producer lanes (lane 0: expect_tx) + bytes
            mbar_init(bwe + 8 * s, 256);                     // the K-step's eight decode warps (every lane)
        }
        for (int s = 0; s < q.SX; ++s) {
            mbar_init(bxf + 8 * s, 1);
            mbar_init(bxe + 8 * s, 1);                       // MMA commit
        }
        for (int s = 0; s < q.SA; ++s) {
            mbar_init(baf + 8 * s, 256);                     // the K-step's eight decode warps (after their proxy fences)
            mbar_init(bae + 8 * s, 1);                       // MMA commit
        }
        mbar_init(bdf, 1);
        mbar_init(bde, 256);                                 // every epilogue lane
        fence_barrier_init();
    }
    if (warp == kWXProd) tm_alloc(sbase + kWTmemSlot, 512);
    tm_fence_before();
    __syncthreads();
    tm_fence_after();
    const uint32_t tmem = *reinterpret_cast<volatile uint32_t *>(smem + kWTmemSlot);
    const int t0 = blockIdx.x, tstep = gridDim.x;
    WProf pf;
    pf.start();

    if (warp == kWWProd) {
        // ------------------------------------------------------------ W producer
        // GTileOffset windows of 16 K-steps: lane l <= 16 holds off[row start + gc0 + l] of both GT rows,
        // loaded one window ahead (the copies of a K-step never wait for a global load)
        const uint64_t pol = policy_evict_first();
        int kk = 0;
        for (int t = t0; t < q.tiles; t += tstep) {
            int rb, nt;
            tile_coords(q, t, rb, nt);
            const int rows = min(2, q.MG - 2 * rb);
            const long long base0 = (long long)(2 * rb) * KG, base1 = base0 + KG;
            auto window = [&](int gc0, int &a, int &b) {
                const bool in = lane <= 16 && gc0 + lane <= KG;
                a = in ? __ldg(q.off + base0 + gc0 + lane) : 0;
                b = (in && rows > 1) ? __ldg(q.off + base1 + gc0 + lane) : 0;
            };
            int ca, cb, na, nb;
            window(0, ca, cb);
            window(16, na, nb);
            for (int gc = 0; gc < KG; ++gc, ++kk) {
                const int j = gc & 15;
                if (j == 0 && gc > 0) {
                    ca = na; cb = nb;
                    window(gc + 16, na, nb);
                }
                const int s = kk % q.SW;
                pf.lap(2);
                if (kk >= q.SW) mbar_wait_sleep(bwe + 8 * s, ((kk / q.SW) & 1) ^ 1);
                pf.lap(1);
                const uint32_t st = sbase + q.o_w + (uint32_t)s * q.w_stage;
                // lanes 0 / 1: the value range of GT row lane (validated: never trust the offsets)
                const int a0 = __shfl_sync(0xffffffffu, ca, j), a1 = __shfl_sync(0xffffffffu, ca, j + 1);
                const int b0 = __shfl_sync(0xffffffffu, cb, j), b1 = __shfl_sync(0xffffffffu, cb, j + 1);
                const int o0 = lane == 0 ? a0 : lane == 1 ? b0 : 0, o1 = lane == 0 ? a1 : lane == 1 ? b1 : 0;
                uint32_t vb = lane < rows ? 2u * (uint32_t)(o1 - o0) : 0u;
                bool bad = false;
                if (lane < rows && (o0 < 0 || o1 < o0 || o1 > q.n_values || (o0 & 7) || vb > q.vcap)) {
                    vb = 0;
                    bad = true;              // poison: the decode warps skip the GT
                    atomicOr(q.ws_err, 1);
                }
                if (lane < 2) sts_u32(sbase + kWHdrOff + (uint32_t)s * kWHdr + 4u * lane, bad ? 0xFFFFFFFFu : (uint32_t)(o1 - o0));
                const uint32_t v0 = __shfl_sync(0xffffffffu, vb, 0), v1 = __shfl_sync(0xffffffffu, vb, 1);
                const uint32_t bmb = 512u * (uint32_t)rows;
                if (lane == 0) mbar_arrive_expect_tx(bwf + 8 * s, v0 + v1 + bmb);
                else mbar_arrive(bwf + 8 * s);
                __syncwarp();
                if (lane < rows && vb) bulk_g2s(st + 1024u + (lane ? q.w_v1 : 0u), q.vals + o0, vb, bwf + 8 * s, pol);
                if (lane >= 2 && lane - 2 < rows)
                    bulk_g2s(st + 512u * (uint32_t)(lane - 2), q.bm + ((size_t)(2 * rb + lane - 2) * KG + gc) * 64, 512u,
                             bwf + 8 * s, pol);
            }
        }
    } else if (warp == kWXProd) {
        // ------------------------------------------------------------ X producer
        // lane j issues box j of the stage (sub-tile j / bps, 64-column chunk j % bps): one TMA
        // instruction for all boxes (a thread's successive copies serialise at ~310 ns each)
        if (lane == 0) prefetch_tmap(&q.tmap_x);
        const int nbox = q.nsub * q.bps;
        const int bsub = lane / q.bps, bj = lane - bsub * q.bps;
        int kk = 0;
        for (int t = t0; t < q.tiles; t += tstep) {
            int rb, nt;
            tile_coords(q, t, rb, nt);
            const int n0 = nt * q.nsub * q.bn;
            for (int gc = 0; gc < KG; ++gc, ++kk) {
                const int s = kk % q.SX;
                if (kk >= q.SX) mbar_wait_sleep(bxe + 8 * s, ((kk / q.SX) & 1) ^ 1);
                const uint32_t st = sbase + q.o_x + (uint32_t)s * q.x_bytes;
                if (lane == 0) mbar_arrive_expect_tx(bxf + 8 * s, q.x_bytes);
                __syncwarp();
                if (lane < nbox)
                    tma_2d_g2s(st + (uint32_t)lane * kWBox, &q.tmap_x, n0 + bsub * q.bn + 64 * bj, 64 * gc, bxf + 8 * s);
            }
        }
    } else if (warp == kWMma) {
        // ------------------------------------------------------------ MMA issuer
        if (lane == 0) {
            int kk = 0, ti = 0;
            for (int t = t0; t < q.tiles; t += tstep, ++ti) {
                if (ti > 0) {   // the epilogue has drained the previous tile's accumulators
                    mbar_wait(bde, (ti - 1) & 1);
                    tm_fence_after();
                }
                for (int gc = 0; gc < KG; ++gc, ++kk) {
                    const int sa = kk % q.SA, sx = kk % q.SX;
                    pf.lap(2);
                    mbar_wait_sleep(baf + 8 * sa, (kk / q.SA) & 1);
                    pf.lap(0);
                    mbar_wait_sleep(bxf + 8 * sx, (kk / q.SX) & 1);
                    pf.lap(1);
                    tm_fence_after();
                    const uint32_t a0 = sbase + q.o_a + (uint32_t)sa * kWABytes;
                    const uint32_t x0 = sbase + q.o_x + (uint32_t)sx * q.x_bytes;
#pragma unroll 1
                    for (int sub = 0; sub < q.nsub; ++sub) {
#pragma unroll
                        for (int k16 = 0; k16 < 4; ++k16) {
                            const uint64_t ad = desc_sw128(a0 + 32u * k16, 16u, 1024u);
                            const uint64_t bd = desc_sw128(x0 + (uint32_t)(sub * q.bps) * kWBox + 2048u * k16, kWBox, 1024u);
                            umma_f16_ss(tmem + (uint32_t)(sub * q.bn), ad, bd, q.idesc, (gc | k16) != 0);
                        }
                    }
                    umma_commit(bae + 8 * sa);
                    umma_commit(bxe + 8 * sx);
                }
                umma_commit(bdf);
            }
        }
        __syncwarp();
    } else if ((warp >= kWEpi0 && warp < kWEpi0 + 4) || warp >= kWEpi1) {
        // ------------------------------------------------------------ epilogue
        const int qd = warp & 3, es = warp >= kWEpi1 ? 1 : 0;
        const uint32_t tq = tmem + ((uint32_t)(32 * qd) << 16);
        int ti = 0;
        for (int t = t0; t < q.tiles; t += tstep, ++ti) {
            int rb, nt;
            tile_coords(q, t, rb, nt);
            pf.lap(2);
            mbar_wait_sleep(bdf, ti & 1);
            pf.lap(0);
            tm_fence_after();
            const int row = rb * 128 + 32 * qd + lane;
            const bool live = row < q.M;
            const float b = (live && q.bias) ? __half2float(__ushort_as_half(q.bias[row])) : 0.f;
            uint16_t *yrow = q.Y + (size_t)(live ? row : 0) * q.N;
            for (int sub = 0; sub < q.nsub; ++sub) {
                for (int c = 32 * es; c < q.bn; c += 64) {
                    float v[2][16];
                    tm_ld_32x32b_x16(tq + (uint32_t)(sub * q.bn + c), v[0]);
                    tm_ld_32x32b_x16(tq + (uint32_t)(sub * q.bn + c + 16), v[1]);
                    tm_wait_ld();
                    const int n = nt * q.nsub * q.bn + sub * q.bn + c;   // first column of the chunk
                    if (!live || n >= q.N) continue;
                    const int lim = min(q.N - n, q.bn - c);   // columns of this sub-tile and of Y
#pragma unroll
                    for (int h = 0; h < 2; ++h)
#pragma unroll
                        for (int j = 0; j < 16; ++j) {
                            float x = v[h][j] + b;
                            v[h][j] = q.act == SPINFER_ACT_RELU ? fmaxf(x, 0.f) : x;
                        }
                    if (lim >= 32 && (q.N & 7) == 0) {
#pragma unroll
                        for (int h = 0; h < 2; ++h)
#pragma unroll
                            for (int c8 = 0; c8 < 2; ++c8) {
                                __half2 p0 = __floats2half2_rn(v[h][8 * c8 + 0], v[h][8 * c8 + 1]);   // one RNE (A11)
                                __half2 p1 = __floats2half2_rn(v[h][8 * c8 + 2], v[h][8 * c8 + 3]);
                                __half2 p2 = __floats2half2_rn(v[h][8 * c8 + 4], v[h][8 * c8 + 5]);
                                __half2 p3 = __floats2half2_rn(v[h][8 * c8 + 6], v[h][8 * c8 + 7]);
                                *reinterpret_cast<uint4 *>(yrow + n + 16 * h + 8 * c8) =
                                    make_uint4(*reinterpret_cast<uint32_t *>(&p0), *reinterpret_cast<uint32_t *>(&p1),
                                               *reinterpret_cast<uint32_t *>(&p2), *reinterpret_cast<uint32_t *>(&p3));
                            }
                    } else {
                        __half *y = reinterpret_cast<__half *>(yrow);
#pragma unroll
                        for (int h = 0; h < 2; ++h)
#pragma unroll
                            for (int j = 0; j < 16; ++j)
                                if (16 * h + j < lim) y[n + 16 * h + j] = __float2half_rn(v[h][j]);
                    }
                }
            }
            tm_fence_before();
            mbar_arrive(bde);
        }
    } else if (warp >= kWDec0 && warp < kWDec0 + kWDecWarps) {
        // ------------------------------------------------------------ decode
        // Warp d decodes TCTile column qc = (d >> 1) & 3 (BitmapTiles 16 qc .. 16 qc + 15) of GT row
        // r = d & 1 in the K-steps of parity ph = d >> 3: two K-steps in flight, 4 decode warps per
        // SM sub-partition. (Every ring the decode warps wait on has an even depth, so a slot is
        // always reused by the same phase: a waiter can never be two barrier generations ahead.)
        const int d = warp - kWDec0, r = d & 1, qc = (d >> 1) & 3, ph = d >> 3;
        const uint32_t mulc = opaque_u32(1u << (30u - 2u * (uint32_t)(lane & 15)));
        const uint32_t tbl = sbase + q.o_tbl + (uint32_t)d * kWTblBytes;
        const uint32_t tbl_lane = tbl + (uint32_t)(lane >> 4) * 128u;
        // the lane's byte offset in the 128 x 64 SWIZZLE_128B K-major A tile for K chunk 2 qc + bc
        // (8 K each): row (lane >> 2) of an 8-row atom, 16-byte chunk XOR row, 4-byte pair (lane & 3)
        uint32_t lb[2];
#pragma unroll
        for (int bc = 0; bc < 2; ++bc)
            lb[bc] = (uint32_t)r * 8192u + (uint32_t)(lane >> 2) * 128u +
                     ((((uint32_t)(2 * qc + bc)) ^ (uint32_t)(lane >> 2)) & 7u) * 16u + (uint32_t)(lane & 3) * 4u;
        int kk = 0;
        for (int t = t0; t < q.tiles; t += tstep) {
            int rb, nt;
            tile_coords(q, t, rb, nt);
            const int rows = min(2, q.MG - 2 * rb);
            for (int gc = 0; gc < KG; ++gc, ++kk) {
                if ((kk & 1) != ph) continue;
                const int sw = kk % q.SW, sa = kk % q.SA;
                pf.lap(2);
                mbar_wait_sleep(bwf + 8 * sw, (kk / q.SW) & 1);
                pf.lap(0);
                if (kk >= q.SA) mbar_wait_sleep(bae + 8 * sa, ((kk / q.SA) & 1) ^ 1);
                pf.lap(1);
                const uint32_t wst = sbase + q.o_w + (uint32_t)sw * q.w_stage;
                const uint32_t ast = sbase + q.o_a + (uint32_t)sa * kWABytes;
                if (r < rows) {
                    const int nv = (int)lds_u32(sbase + kWHdrOff + (uint32_t)sw * kWHdr + 4u * r);
                    const uint32_t bms = wst + 512u * (uint32_t)r;
                    const uint32_t vsm = wst + 1024u + (r ? q.w_v1 : 0u);
                    const uint2 ba = lds_v2(bms + 8u * lane), bb = lds_v2(bms + 256u + 8u * lane);
                    // PopCount prefix over the GT's 64 BitmapTiles: lane l holds BTs l, l + 32
                    const uint32_t pax = __popc(ba.x), pbx = __popc(bb.x);
                    const uint32_t packed = (pax + __popc(ba.y)) | ((pbx + __popc(bb.y)) << 16);
                    uint32_t incl = packed;
#pragma unroll
                    for (int o = 1; o < 32; o <<= 1) {
                        const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
                        incl += (lane >= o) ? y : 0u;
                    }
                    const uint32_t tot = __shfl_sync(0xffffffffu, incl, 31);
                    const uint32_t tot_a = tot & 0xFFFFu, tot_all = tot_a + (tot >> 16);
                    // the GT's padded value count must match its popcount (corrupt input: skip the GT)
                    const bool ok = nv >= 0 && (int)((tot_all + 7u) & ~7u) == nv;
                    if (ok) {
                        // table [word half][BT 16 qc + j] x {bitmap half-word, smem address of its first value - 4}:
                        // BT 16 qc + j is held by lane 16 qc + j (qc < 2, part a) or 16 (qc - 2) + j (part b)
                        if ((lane >> 4) == (qc & 1)) {
                            const uint32_t excl = incl - packed;
                            const bool hb = qc >= 2;
                            const uint32_t A = hb ? vsm + 2u * (tot_a + (excl >> 16)) - 4u : vsm + 2u * (excl & 0xFFFFu) - 4u;
                            const uint2 bw = hb ? bb : ba;
                            const uint32_t te = tbl + 8u * (uint32_t)(lane & 15);
                            sts_v2(te, bw.x, A);
                            sts_v2(te + 128u, bw.y, A + 2u * (hb ? pbx : pax));
                        }
                    } else if (lane == 0) {
                        atomicOr(q.ws_err, 2);
                    }
                    __syncwarp();
                    if (ok) {
#pragma unroll
                        for (int g8 = 0; g8 < 2; ++g8) {   // BTs 16 qc + 8 g8 .. + 7: TCTile rows 2 g8, 2 g8 + 1
                            uint4 E[4];
#pragma unroll
                            for (int k = 0; k < 4; ++k) E[k] = lds_v4(tbl_lane + 64u * g8 + 16u * k);
#pragma unroll
                            for (int k = 0; k < 8; ++k) {
                                const uint32_t w = (k & 1) ? E[k >> 1].z : E[k >> 1].x;
                                const uint32_t A = (k & 1) ? E[k >> 1].w : E[k >> 1].y;
                                const uint32_t z = w * mulc;
                                const uint32_t a = A + 2u * __popc(z);
                                const uint32_t yy = z >> 30;
                                const uint32_t sel = yy * (yy * kSelBw + kSelAw) + kSelCw;
                                const uint32_t v = prmt(lds_u16(a), lds_u16(a + 2u), sel);
                                // BT 16 qc + j, j = 8 g8 + k: TCTile row tr = j >> 2; BT q = j & 3 in the TCTile
                                // (br = q & 1, bc = q >> 1)
                                const int j = 8 * g8 + k, tr = j >> 2, br = j & 1, bc = (j >> 1) & 1;
                                sts_u32(ast + lb[bc] + (uint32_t)(tr * 2 + br) * 1024u, v);
                            }
                        }
                    }
                    __syncwarp();   // table reads done before the next K-step rewrites it
                }
                fence_proxy_async_smem();   // the A tile stores, visible to the tensor core
                mbar_arrive(baf + 8 * sa);
                mbar_arrive(bwe + 8 * sw);
            }
        }
    }
    pf.lap(2);
    pf.dump(q.prof, blockIdx.x, warp, lane);
    tm_fence_before();
    __syncthreads();
    if (warp == kWXProd) {
        tm_fence_after();
        tm_dealloc(tmem, 512);
    }
}

inline uint32_t al_w(uint32_t x, uint32_t a) { return (x + a - 1) / a * a; }

struct WPlan {
    int P;
    size_t smem;
    WParams prm;
};

bool make_wplan(int M, int K, int N, int max_gt_values, WPlan *pl) {
    const int MG = (M + kGT - 1) / kGT, KG = (K + kGT - 1) / kGT;
    const int RB = (MG + 1) / 2;
    WParams &q = pl->prm;
    const int n16 = (N + 15) & ~15;
    const int ob = option(SPINFER_OPT_WIDE_BN);
    const int bnmax = ob >= 16 ? std::min(256, ob & ~15) : 256;
    if (n16 <= bnmax) { q.nsub = 1; q.bn = n16; }
    else if (n16 <= 2 * bnmax) { q.nsub = 2; q.bn = (((N + 1) / 2) + 15) & ~15; }
    else { q.nsub = 2; q.bn = bnmax; }
    q.bps = (q.bn + 63) / 64;
    q.ntn = (N + q.nsub * q.bn - 1) / (q.nsub * q.bn);
    q.RB = RB; q.MG = MG; q.KG = KG; q.M = M; q.N = N;
    const long long tiles = (long long)RB * q.ntn;
    if (tiles >= (1LL << 31)) return false;
    q.tiles = (int)tiles;
    q.group = std::min(RB, 16);
    int maxv = max_gt_values > 0 ? max_gt_values : 4096;
    maxv = std::min(4096, (maxv + 7) & ~7);
    q.vcap = al_w((uint32_t)maxv * 2u, 128);
    q.w_v1 = q.vcap;
    q.w_stage = al_w(1024u + 2u * q.vcap, 128);
    q.x_bytes = (uint32_t)(q.nsub * q.bps) * kWBox;
    const int smem_max = smem_optin();
    const uint32_t fixed = 1024u /* barriers, header */ + kWDecWarps * kWTblBytes + 1024u /* base alignment */;
    // ring depths: 2 X stages, then A slots and W stages in pairs (even depths: each slot is always
    // refilled for the same decode phase), then more X stages
    int SX = 2, SA = 2, SW = 2;
    auto total = [&](int sx, int sa, int sw) {
        return (long long)fixed + (long long)sx * q.x_bytes + (long long)sa * kWABytes + (long long)sw * q.w_stage;
    };
    if (total(SX, SA, SW) > smem_max) return false;
    while (SW + 2 <= kWMaxSW && SW < 4 && total(SX, SA, SW + 2) <= smem_max) SW += 2;
    while (SA + 2 <= kWMaxSA && total(SX, SA + 2, SW) <= smem_max) SA += 2;
    while (SW + 2 <= kWMaxSW && total(SX, SA, SW + 2) <= smem_max) SW += 2;
    while (SX < kWMaxSX && total(SX + 1, SA, SW) <= smem_max) ++SX;
    q.SX = SX; q.SA = SA; q.SW = SW;
    q.o_tbl = 1024u;
    q.o_a = al_w(q.o_tbl + kWDecWarps * kWTblBytes, 1024);
    q.o_x = q.o_a + (uint32_t)SA * kWABytes;
    q.o_w = q.o_x + (uint32_t)SX * q.x_bytes;
    pl->smem = (size_t)q.o_w + (size_t)SW * q.w_stage + 1024;
    q.idesc = (1u << 4) | (1u << 16) | ((uint32_t)(q.bn >> 3) << 17) | ((128u >> 4) << 24);   // f16 x f16 -> f32, A K-major, B MN-major
    pl->P = std::min(q.tiles, sm_count());
    return true;
}

}  // namespace

// Workspace of the wide kernel: [error word region][zero-padded X when N % 8 != 0].
size_t spmm_wide_workspace_bytes(int M, int K, int N) {
    (void)M;
    const int Np = (N + 7) & ~7;
    return kCounterRegion + ((N % 8) ? ((size_t)K * Np * 2 + 255) / 256 * 256 : 0);
}

int launch_spmm_wide(const spinfer_tca *T, const uint16_t *X, uint16_t *Y, int M, int K, int N, const uint16_t *bias,
                     int act, void *ws, size_t ws_bytes, cudaStream_t st) {
    WPlan pl;
    if (!make_wplan(M, K, N, T->max_gt_values, &pl)) return SPINFER_EINVAL;
    if (ws == nullptr || ws_bytes < spmm_wide_workspace_bytes(M, K, N)) return SPINFER_ENOSPC;
    WParams &q = pl.prm;
    uint8_t *w8 = reinterpret_cast<uint8_t *>(ws);
    const int Np = (N + 7) & ~7;
    const uint16_t *Xk = X;
    if (N % 8) {
        uint16_t *Xp = reinterpret_cast<uint16_t *>(w8 + kCounterRegion);
        if (int rc = launch_pad_x(X, Xp, K, N, Np, st)) return rc;
        Xk = Xp;
    }
    if (int rc = make_x_tmap_box(&q.tmap_x, Xk, K, Np, 64, 64, CU_TENSOR_MAP_SWIZZLE_128B)) return rc;
    q.off = T->gtile_offset;
    q.bm = T->bitmap;
    q.vals = T->values;
    q.Y = Y;
    q.bias = bias;
    q.act = act;
    q.ws_err = reinterpret_cast<int32_t *>(w8) + kErrWord;
    q.n_values = (int)T->n_values;
    q.prof = nullptr;
#if SPINFER_INSTRUMENT
    static long long *prof_buf = nullptr;
    const size_t nprof = (size_t)1024 * 32 * 4;
    if (!prof_buf && cudaMalloc(&prof_buf, nprof * 8) != cudaSuccess) return SPINFER_ECUDA;
    cudaMemsetAsync(prof_buf, 0, nprof * 8, st);
    q.prof = prof_buf;
#endif
    static int configured[64] = {0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    if ((int)pl.smem > configured[dev]) {
        if (cudaFuncSetAttribute(k_spmm_wide, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)pl.smem) != cudaSuccess)
            return SPINFER_ECUDA;
        configured[dev] = (int)pl.smem;
    }
    k_spmm_wide<<<pl.P, kWThreads, pl.smem, st>>>(q);
#if SPINFER_INSTRUMENT
    if (const char *path = getenv("SPINFER_PROF")) {   // experiments: dump the per-warp counters
        long long *host = (long long *)malloc(nprof * 8);
        cudaMemcpyAsync(host, q.prof, nprof * 8, cudaMemcpyDeviceToHost, st);
        cudaStreamSynchronize(st);
        if (FILE *f = fopen(path, "wb")) { fwrite(host, 8, nprof, f); fclose(f); }
        free(host);
    }
#endif
    return cudaGetLastError() == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
}

}  // namespace spinfer
