// spmm_tc.cu — TCA-BME SpMM Y = W x X on the tcgen05 tensor cores, the library's kernel for
// 24 <= N <= 32 (sm_100a; §4.3). One persistent CTA per SM, stream-K over
// GroupTile columns (replacing the paper's split-K grid, Alg. 1 lines 1-3), rowblocks
// split across CTAs combined by an in-kernel "last contributor sums" fix-up (the paper's
// ReductionWorkspace).
#include <cuda.h>
#include <algorithm>
#include <cstdlib>
#include "internal.cuh"
#include "ptx.cuh"

namespace spinfer {
namespace {

constexpr int kR = 2;               // GT rows per rowblock (128 output rows)
constexpr int kMaxG = 4;            // max GroupTile columns per stage
constexpr int kMaxStages = 8;
constexpr int kConstWord = 48;      // smem word index (byte 192) of the SMBD selector constants

struct Params {
    CUtensorMap tmap_x;          // X [K][N] fp16, box {NB, 64 G}, swizzle 32B (NB = 16) / 64B (NB = 32)
    const int32_t *off;
    const uint64_t *bm;
    const uint16_t *vals;
    uint16_t *Y;
    float *ws_part;              // [P][2 split segments][128 rows][Nw] fp32 CTA partials
    const uint16_t *bias;        // fused epilogue (spinfer_spmm_ex): fp16 [M] or null
    int act;                     // SPINFER_ACT_NONE / SPINFER_ACT_RELU
    int32_t *ws_cnt;             // [4 x rowblocks] split-K counters (zero between calls)
    int32_t *ws_err;             // error word: non-zero when corrupt TCA-BME input was skipped
    int n_values;                // gtile_offset bound
    uint32_t vcap;               // value bytes a stage slot holds per GT row
    int KG, MG;
    int N;                       // real N (X padded to NB by the TMA's out-of-bounds fill)
    uint32_t U;                  // units (rowblock x GT column); U * P < 2^32
    int P;
    int G, S;
    uint32_t stage_bytes, st_v0, st_v1;   // stage slot size; offsets in a slot (X slab at 0)
    uint32_t tbl_bytes;
    uint32_t o_desc, o_tbl, o_stage;      // region offsets from the smem base
    int M;                       // real rows of Y (M need not be a multiple of 64: rows >= M are padding, A8)
};

// Stream-K partition in 32-bit arithmetic (the host guarantees U * P < 2^32).
__device__ __forceinline__ int unit_start(int p, uint32_t U, int P) { return (int)((uint32_t)p * U / (uint32_t)P); }
__device__ __forceinline__ int unit_owner(int u, uint32_t U, int P) {
    return (int)(((uint32_t)(u + 1) * (uint32_t)P - 1u) / U);
}

// Stage iterator: every role walks the same deterministic stage sequence. A CTA's unit
// range [u0, u1) is processed in the order: A = the tail of the rowblock it starts inside
// (split with the previous CTA), C = the head of the rowblock it ends inside (split with
// the next CTA), then the full rowblocks in between. The split segments, whose results need
// the cross-CTA fix-up, are therefore finished early and their fix-up latency hides behind
// the full rowblocks; every CTA ends on a complete rowblock (plain Y stores).
// Per-stage bookkeeping is incremental 32-bit arithmetic (a division per part switch).
struct StageIter {
    int u, ue, us;           // current unit, end and start of the current part
    int ns0, ne0, ns1, ne1;  // remaining parts, in order (empty: start == end)
    int rb, gc, g, rows;     // current stage: rowblock, first GT column, #units, #GT rows
    int i, slot;             // stage index within the CTA, smem ring slot
    uint32_t ph;             // ring parity ((i / S) & 1)
    __device__ __forceinline__ void init(int u0, int u1, const Params &prm) {
        const int KG = prm.KG;
        const int a_end = (u0 % KG) ? min(u1, (u0 / KG + 1) * KG) : u0;          // A = [u0, a_end)
        const int c_beg = (u1 % KG) ? max(a_end, (u1 / KG) * KG) : u1;           // C = [c_beg, u1)
        // parts in order A, C, M = [a_end, c_beg); empty ones dropped (no arrays: no local memory)
        int q0s = u1, q0e = u1, q1s = u1, q1e = u1, q2s = u1, q2e = u1, k = 0;
        auto push = [&](int s_, int e_) {
            if (s_ >= e_) return;
            if (k == 0) { q0s = s_; q0e = e_; } else if (k == 1) { q1s = s_; q1e = e_; } else { q2s = s_; q2e = e_; }
            ++k;
        };
        push(u0, a_end);
        push(c_beg, u1);
        push(a_end, c_beg);
        ns0 = q1s; ne0 = q1e; ns1 = q2s; ne1 = q2e;
        i = 0; slot = 0; ph = 0;
        part(q0s, q0e, prm);
    }
    __device__ __forceinline__ void part(int s0, int e0, const Params &prm) {
        u = s0; us = s0; ue = e0;
        rb = (int)((uint32_t)u / (uint32_t)prm.KG);
        gc = u - rb * prm.KG;
        shape(prm);
    }
    __device__ __forceinline__ void shape(const Params &prm) {
        g = min(min(prm.G, prm.KG - gc), ue - u);
        rows = min(kR, prm.MG - kR * rb);
    }
    __device__ __forceinline__ bool valid() const { return u < ue; }
    __device__ __forceinline__ uint32_t par() const { return ph; }
    __device__ __forceinline__ bool seg_first() const { return u == us || gc == 0; }
    __device__ __forceinline__ bool seg_last(const Params &prm) const { return gc + g == prm.KG || u + g == ue; }
    __device__ __forceinline__ void next(const Params &prm) {
        u += g;
        gc += g;
        if (gc == prm.KG) { gc = 0; ++rb; }
        ++i;
        if (++slot == prm.S) { slot = 0; ph ^= 1u; }
        if (u == ue && ns0 < ne0) {
            const int s0 = ns0, e0 = ne0;
            ns0 = ns1; ne0 = ne1; ns1 = ne1;
            part(s0, e0, prm);
        } else {
            shape(prm);
        }
    }
};

// Per-CTA stage descriptor (built once in shared memory by scan warp 0): the consumer
// loop then carries only the stage index across its decode loop. (Keeping the StageIter
// live in registers made ptxas spill it; local memory goes to L2 here because the
// shared-memory carve-out leaves almost no L1, so each stage paid ~800-cycle reloads.)
//   w0: rb [0,20) | slot [20,24) | parity 24 | zero-acc 25 | segment end 26 | complete 27 | rows-1 28
//   w1: gc [0,16) | g [16,24);  tbl, stg: the slot's table and stage region offsets
struct StageDesc {
    uint32_t w0, w1, tbl, stg;   // tbl / stg: smem offsets (from the aligned base) of the slot's table / stage
    __device__ __forceinline__ int rb() const { return (int)(w0 & 0xFFFFFu); }
    __device__ __forceinline__ int slot() const { return (int)((w0 >> 20) & 15u); }
    __device__ __forceinline__ uint32_t par() const { return (w0 >> 24) & 1u; }
    __device__ __forceinline__ bool zero() const { return (w0 >> 25) & 1u; }
    __device__ __forceinline__ bool seg_end() const { return (w0 >> 26) & 1u; }
    __device__ __forceinline__ bool complete() const { return (w0 >> 27) & 1u; }
    __device__ __forceinline__ int rows() const { return 1 + (int)((w0 >> 28) & 1u); }
    __device__ __forceinline__ int g() const { return (int)((w1 >> 16) & 0xFFu); }
};

// SMBD selector (see spmm_dw.cu): PRMT of the two zero-extended u16 loads {V[c2-2], V[c2-1]},
// selector = y (kSelA + kSelB y) + kSelC for the lane's bit pair y
constexpr uint32_t kSelA = 0x7f62u, kSelB = 0x4cbfu, kSelC = 0x2333u;

// Fused epilogue of one output (spinfer_spmm_ex): + bias[row] and the activation, in fp32.
__device__ __forceinline__ float epi_act(float v, float b, int act) {
    v += b;
    return act == SPINFER_ACT_RELU ? fmaxf(v, 0.f) : v;
}

// ================================================================ tcgen05 path
// The library's kernel for N >= 24: the stream-K stage walk of the SMBD path with
// the accumulators in TMEM and the MMA on the 5th-generation tensor cores:
//   * 16 decode warps: warp w owns TMEM lane quarter q = w & 3 (TCTile rows 2q, 2q+1 of the
//     128-row rowblock; a warp may only touch its own lane quarter) and k-team kt = w >> 2
//     (GroupTile column kt of the stage). Per stage it
//       - builds the SMBD table for its GroupTile (PopCount prefix over the GT's 64 BTs)
//         from bitmaps it loaded into registers one stage earlier (no TMA, no scan warps):
//         {bitmap half-word, smem address of that half's first value - 4} per (BT, half);
//       - decodes its 8 TCTiles (32 BitmapTiles, MaskedPopCount Alg. 2) into
//         A-fragment registers and writes each TCTile to TMEM with one tcgen05.st.16x128b.x2.
//   * the k-team multiplies its own GroupTile column: once its 4 lane-quarter warps have written
//     their A tiles (named barrier), one elected lane of the team's warp 0 issues 4 x tcgen05.mma
//     kind::f16, M = 128, N = NB, K = 16, A from TMEM, B = the TMA-staged X slab (MN-major,
//     32B/64B swizzle), into the team's own fp32 accumulator in TMEM (2 per team: segment parity).
//     Four issuers in parallel (a single MMA warp issuing 16 tiny MMAs per stage was the
//     pipeline's slowest link); the epilogue sums the team accumulators in team order.
//   * 1 producer warp: per stage two 1-D bulk copies (the packed values of the two GT rows,
//     contiguous along K) and one 2-D tensor TMA (X rows [64 gc, 64 (gc + G)), box {NB, 64 G}).
//     Measured on B200 (tools/tma_sweep.sh): a bulk copy occupies the SM's TMA unit >= ~310 ns
//     however small, so a stage issues as few copies as possible.
//   * rowblock epilogue: segment s is finished by k-team s & 3 one stage after its last stage:
//     tcgen05.ld of D, one RNE to fp16 and the Y store, or (split rowblock) the fp32 partial,
//     counted and summed by the fix-up warp off the decode path.
// Every role walks the same StageIter sequence itself (no descriptor table, no start-up wait).
struct CfgTC {
    static constexpr int CW = 16;
    static constexpr int ProducerWarp = 16;
    static constexpr int ScanWarp = 17;      // 17, 18, 19: SMBD tables of the stages i % 3 == 0, 1, 2
    static constexpr int NScan = 3;          // (the scan warps bound the kernel: their throughput, not latency)
    static constexpr int Threads = 20 * 32;  // 5 warps per SM sub-partition: 96 registers each
    static constexpr uint32_t TmemCols = 512;
};
// TMEM columns: A buffers [k-team][ABufs] x 32 columns, then D [k-team][segment parity] x NB
template <int NB>
struct TmemTC {
    static constexpr int ABufs = NB == 16 ? 3 : 2;
    static constexpr uint32_t DCol = 4u * ABufs * 32u;
    static_assert(DCol + 8u * NB <= CfgTC::TmemCols, "TMEM budget");
};
// barrier / scalar region (bytes from the aligned smem base); per-warp tables from 1024
constexpr uint32_t kTcFull = 0, kTcEmpty = 64, kTcEmptyX = 128, kTcTmemSlot = 208;
constexpr uint32_t kTcAEmpty = 256, kTcDFull = 352, kTcDEmpty = 368, kTcFix = 384;   // aempty [4][3]
constexpr uint32_t kTcAFull = 400;     // [k-team][A buffer]: the team's 4 lane-quarter warps wrote their A tiles
constexpr uint32_t kTcScan = 512;      // [S]: the slot's SMBD table is written
constexpr uint32_t kTcTeamCnt = 960;   // int [k-team][A buffer]: A tiles written (last of 4 writers issues the MMA)
// ring position of a multi-buffer: index and phase parity, advanced once per use
template <int NBUF>
struct Ring {
    uint32_t b = 0, ph = 0;
    __device__ __forceinline__ void next() { if (++b == NBUF) { b = 0; ph ^= 1u; } }
};

template <int NB>
__device__ __forceinline__ void store_y_row(const Params &prm, size_t grow, float (&v)[NB]) {
    uint16_t *const Y = prm.Y;
    const int N = prm.N;
    if (grow >= (size_t)prm.M) return;   // padding row of a ragged M (A8)
    if (prm.bias || prm.act) {   // fused epilogue (spinfer_spmm_ex)
        const float b = prm.bias ? __half2float(__ushort_as_half(prm.bias[grow])) : 0.f;
#pragma unroll
        for (int j = 0; j < NB; ++j) v[j] = epi_act(v[j], b, prm.act);
    }
    if (N % 8) {   // N not a multiple of 8 (X was zero-padded): rows are not 16-byte aligned
        __half *y = reinterpret_cast<__half *>(Y + grow * (size_t)N);
#pragma unroll
        for (int j = 0; j < NB; ++j)
            if (j < N) y[j] = __float2half_rn(v[j]);   // one RNE per output (A11)
        return;
    }
    uint4 *yp = reinterpret_cast<uint4 *>(Y + grow * (size_t)N);
#pragma unroll
    for (int c8 = 0; c8 < NB / 8; ++c8)
        if (c8 * 8 < N) {
            __half2 h0 = __floats2half2_rn(v[8 * c8 + 0], v[8 * c8 + 1]);   // one RNE per output (A11)
            __half2 h1 = __floats2half2_rn(v[8 * c8 + 2], v[8 * c8 + 3]);
            __half2 h2 = __floats2half2_rn(v[8 * c8 + 4], v[8 * c8 + 5]);
            __half2 h3 = __floats2half2_rn(v[8 * c8 + 6], v[8 * c8 + 7]);
            yp[c8] = make_uint4(*reinterpret_cast<uint32_t *>(&h0), *reinterpret_cast<uint32_t *>(&h1),
                                *reinterpret_cast<uint32_t *>(&h2), *reinterpret_cast<uint32_t *>(&h3));
        }
}

template <int NB>
__global__ void __launch_bounds__(CfgTC::Threads, 1) k_spmm_tc(const __grid_constant__ Params prm) {
    constexpr int kCW = CfgTC::CW;
    constexpr int ABufs = TmemTC<NB>::ABufs;
    constexpr uint32_t DCol = TmemTC<NB>::DCol;
    constexpr uint32_t kEndBar = 1, kTeamBar = 2;   // named barriers: decode warps at the end; 2 + kt: k-team kt
    constexpr uint32_t kDescBarTC = 6;              // stage descriptors written (scan warp 1 -> decode warps)
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *const smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    const uint32_t sbase = smem_u32(smem);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int p = blockIdx.x;
    const uint32_t U = prm.U;
    const int KG = prm.KG, G = prm.G, S = prm.S;
    const int u0 = unit_start(p, U, prm.P), u1 = unit_start(p + 1, U, prm.P);
    // ring barriers per slot: full (values + X landed), empty (every decode warp is done with the
    // slot's values), emptyx (the MMA has read the slot's X slab)
    const uint32_t bar_full = sbase + kTcFull, bar_empty = sbase + kTcEmpty, bar_emptyx = sbase + kTcEmptyX;
    const uint32_t bar_ae = sbase + kTcAEmpty, bar_df = sbase + kTcDFull, bar_de = sbase + kTcDEmpty,
                   bar_scan = sbase + kTcScan;

    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(bar_full + 8 * s, 1);
            mbar_init(bar_empty + 8 * s, 32 * kCW);        // every lane of every decode warp (its table reads)
            mbar_init(bar_emptyx + 8 * s, 4);              // the 4 k-teams' MMA commits
            mbar_init(bar_scan + 8 * s, 32);               // the stage's scan warp (every lane: its table stores)
        }
        for (int k = 0; k < 4 * ABufs; ++k) mbar_init(bar_ae + 8 * k, 1);   // [k-team][buffer]: team MMA commit
        for (int k = 0; k < 4 * ABufs; ++k) mbar_init(sbase + kTcAFull + 8 * k, 4);   // [k-team][buffer]: A written
        for (int k = 0; k < 2; ++k) {
            mbar_init(bar_df + 8 * k, 4);                  // [segment parity]: the 4 k-teams' commits
            mbar_init(bar_de + 8 * k, 4);                  // the 4 warps of the finishing k-team
        }
        for (int k = 0; k < 2; ++k) mbar_init(sbase + kTcFix + 8 * k, 4);   // split segment A / C parked
        for (int k = 0; k < 12; ++k) reinterpret_cast<int *>(smem + kTcTeamCnt)[k] = 0;
        fence_barrier_init();
        reinterpret_cast<uint32_t *>(smem)[kConstWord] = kSelA;
        reinterpret_cast<uint32_t *>(smem)[kConstWord + 1] = kSelB;
        reinterpret_cast<uint32_t *>(smem)[kConstWord + 2] = kSelC;
    }
    if (warp == CfgTC::ProducerWarp && lane == 0) prefetch_tmap(&prm.tmap_x);
    if (warp == 0) tm_alloc(sbase + kTcTmemSlot, CfgTC::TmemCols);
    tm_fence_before();
    __syncthreads();
    tm_fence_after();
    if (threadIdx.x == 0) grid_dep_launch();   // SPINFER_OPT_PDL: the next kernel may be scheduled
    const uint32_t tmem = *reinterpret_cast<volatile uint32_t *>(smem + kTcTmemSlot);
    if (u0 >= u1) {   // no work (more CTAs than units)
        if (warp == 0) tm_dealloc(tmem, CfgTC::TmemCols);
        return;
    }

    if (warp == CfgTC::ProducerWarp) {
        // ------------------------------------------------------------ producer
        // Lanes 0 / 1 prefetch the value range of GT row 0 / 1 one stage ahead and issue its bulk
        // copy (one instruction for both rows); lane 0 issues the X tensor TMA.
        const uint64_t pol_w = policy_evict_first();
        const uint32_t xbytes = 64u * NB * 2u;         // one GroupTile column of X
        int2 poff = make_int2(0, 0);
        auto load_off = [&](const StageIter &sg) {
            int2 v = make_int2(0, 0);
            if (lane < sg.rows) {
                const int g0 = (kR * sg.rb + lane) * KG + sg.gc;
                v.x = __ldg(prm.off + g0);
                v.y = __ldg(prm.off + g0 + sg.g);
            }
            return v;
        };
        StageIter pit;
        pit.init(u0, u1, prm);
        poff = load_off(pit);
        for (; pit.valid();) {
            const StageIter sg = pit;
            const int i = sg.i, slot = sg.slot;
            if (i >= S) mbar_wait_sleep(bar_empty + 8 * slot, sg.par() ^ 1u);
            const uint32_t st = sbase + prm.o_stage + slot * prm.stage_bytes;
            uint32_t vb = 2u * (uint32_t)(poff.y - poff.x);   // lanes 0, 1: value bytes of their GT row
            // corrupt offsets (decreasing, past n_values, or more values than max_gt_values sized the
            // slot for): copy nothing; the scan warp zeroes the stage's tables and flags the error
            if (lane < sg.rows && (poff.x < 0 || poff.y < poff.x || poff.y > prm.n_values || vb > prm.vcap)) {
                vb = 0;
                atomicOr(prm.ws_err, 1);
            }
            const uint32_t vtot = __shfl_sync(0xffffffffu, vb, 0) + __shfl_sync(0xffffffffu, vb, 1);
            if (lane == 0) mbar_arrive_expect_tx(bar_full + 8 * slot, (uint32_t)G * xbytes + vtot);
            __syncwarp();
            if (lane < sg.rows && vb)
                bulk_g2s(st + (lane ? prm.st_v1 : prm.st_v0), prm.vals + poff.x, vb, bar_full + 8 * slot, pol_w);
            // the X slab region is free once the MMA of stage i - S has completed
            if (i >= S) mbar_wait(bar_emptyx + 8 * slot, sg.par() ^ 1u);
            // X may be the previous kernel's output (SPINFER_OPT_PDL): the first stage waits for that
            // grid with its weight copies in flight; everything else follows from this stage's data
            if (i == 0) grid_dep_wait();
            if (lane == 0) tma_2d_g2s(st, &prm.tmap_x, 0, 64 * sg.gc, bar_full + 8 * slot);   // box {NB, 64 G}
            pit.next(prm);
            if (pit.valid()) poff = load_off(pit);
        }
        return;
    }

    if (warp >= CfgTC::ScanWarp) {
        // ------------------------------------------------------------ scan
        // Scan warp s builds the SMBD tables of the stages i = s (mod 2), both GT rows: per
        // staged GroupTile the popcounts of its 64 BTs, a shuffle scan (the PopCount prefix,
        // P:274) and a table {bitmap half-word, smem address of that half's first value - 4}
        // per (BT, lane half), layout [GT (r, j)][half][BT] x 8 B. The bitmaps come from global
        // memory straight into registers, prefetched two stages ahead (no TMA copy: a bulk copy
        // costs the SM's TMA unit >= ~310 ns however small, tools/tma_sweep.sh). A table waits
        // only for its slot to be free, so its latency (shuffle round trips through the loaded
        // MIO queue) is hidden; three warps (stages i % 3) share the throughput the kernel is bound by.
        constexpr int Q = 2 * kMaxG;
        const int sw = warp - CfgTC::ScanWarp;
        struct Bm { uint2 a[Q], b[Q]; int o; };   // o: lane 8 rr + j holds gtile_offset of GT j of row rr
        auto fetch = [&](const StageIter &sg, Bm &f) {
            f.o = ((lane >> 3) < sg.rows && (lane & 7) <= sg.g && lane < 16)
                      ? __ldg(prm.off + (kR * sg.rb + (lane >> 3)) * KG + sg.gc + (lane & 7)) : 0;
#pragma unroll
            for (int qq = 0; qq < Q; ++qq) {
                const int rr = qq / kMaxG, j = qq % kMaxG;
                if (rr < sg.rows && j < sg.g) {
                    const uint64_t *gp = prm.bm + ((size_t)(kR * sg.rb + rr) * KG + sg.gc + j) * 64;
                    f.a[qq] = ldg_nc_v2(gp + lane);
                    f.b[qq] = ldg_nc_v2(gp + 32 + lane);
                } else {
                    f.a[qq] = make_uint2(0u, 0u);
                    f.b[qq] = make_uint2(0u, 0u);
                }
            }
        };
        if (sw == 1) {
            // stage descriptors for the decode warps (same encoding as k_spmm's StageDesc)
            if (lane == 0) {
                StageIter d;
                int n = 0;
                bool full_start = false;
                for (d.init(u0, u1, prm); d.valid(); d.next(prm), ++n) {
                    const bool zero = d.seg_first();
                    if (zero) full_start = (d.gc == 0);
                    const bool seg_end = d.seg_last(prm);
                    const bool complete = seg_end && full_start && (d.gc + d.g == KG);
                    const uint32_t w0 = (uint32_t)d.rb | ((uint32_t)d.slot << 20) | (d.ph << 24) | ((uint32_t)zero << 25) |
                                        ((uint32_t)seg_end << 26) | ((uint32_t)complete << 27) |
                                        ((uint32_t)(d.rows - 1) << 28);
                    sts_v4(sbase + prm.o_desc + 16u * (uint32_t)n,
                           make_uint4(w0, (uint32_t)d.gc | ((uint32_t)d.g << 16), 0u, 0u));
                }
                reinterpret_cast<volatile uint32_t *>(smem)[kConstWord + 3] = (uint32_t)n;
            }
            __syncwarp();
            named_bar_arrive(6u, 32u * (CfgTC::CW + 1));
        }
        StageIter it;
        it.init(u0, u1, prm);
        for (int k = 0; k < sw && it.valid(); ++k) it.next(prm);
        auto skip2 = [&](StageIter &x) {   // this warp's next stage: NScan stages on
            for (int k = 0; k < CfgTC::NScan && x.valid(); ++k) x.next(prm);
        };
        Bm F;   // one register set: the next stage's loads are issued right after a table is
                // published and complete while the warp waits for that stage's slot
        if (it.valid()) fetch(it, F);
        auto one = [&](Bm &cur) -> bool {
            if (!it.valid()) return false;
            const StageIter sg = it;
            const int slot = sg.slot;
            if (sg.i >= S) mbar_wait_sleep(bar_empty + 8 * slot, sg.par() ^ 1u);   // the slot's table is free
            const uint32_t st = sbase + prm.o_stage + slot * prm.stage_bytes;
            const uint32_t tb = sbase + prm.o_tbl + slot * prm.tbl_bytes;
            uint32_t packed[Q], incl[Q];
#pragma unroll
            for (int qq = 0; qq < Q; ++qq) {
                packed[qq] = (__popc(cur.a[qq].x) + __popc(cur.a[qq].y)) |
                             ((__popc(cur.b[qq].x) + __popc(cur.b[qq].y)) << 16);
                incl[qq] = packed[qq];
            }
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                uint32_t y[Q];
#pragma unroll
                for (int qq = 0; qq < Q; ++qq) y[qq] = __shfl_up_sync(0xffffffffu, incl[qq], o);
#pragma unroll
                for (int qq = 0; qq < Q; ++qq) incl[qq] += (lane >= o) ? y[qq] : 0u;
            }
            int rel[kR] = {0, 0};
            bool bad = false;
#pragma unroll
            for (int qq = 0; qq < Q; ++qq) {
                const int rr = qq / kMaxG, j = qq % kMaxG;
                const uint32_t t = __shfl_sync(0xffffffffu, incl[qq], 31);
                if (rr < sg.rows && j < sg.g) {
                    const uint32_t vsm = st + (rr ? prm.st_v1 : prm.st_v0);
                    const uint32_t excl = incl[qq] - packed[qq];
                    const uint32_t ea = excl & 0xFFFFu, eb = (t & 0xFFFFu) + (excl >> 16);
                    const uint32_t Aa = vsm + 2u * (uint32_t)(rel[rr] + (int)ea);
                    const uint32_t Ab = vsm + 2u * (uint32_t)(rel[rr] + (int)eb);
                    const uint32_t te = tb + (uint32_t)(rr * G + j) * 1024u + 8u * lane;
                    sts_v2(te, cur.a[qq].x, Aa - 4u);
                    sts_v2(te + 512u, cur.a[qq].y, Aa - 4u + 2u * __popc(cur.a[qq].x));
                    sts_v2(te + 256u, cur.b[qq].x, Ab - 4u);
                    sts_v2(te + 768u, cur.b[qq].y, Ab - 4u + 2u * __popc(cur.b[qq].x));
                }
                // GT j's first value within the row's chunk: earlier GTs' counts, each padded to
                // a multiple of 8 values (the GTileOffset rule, encode.cu)
                rel[rr] += (int)(((t & 0xFFFFu) + (t >> 16) + 7u) & ~7u);
            }
            // memory safety first: the tables address the row's values by popcount (rel), so a row
            // whose bitmaps claim more values than a slot holds (corrupt input) decodes as zeros,
            // reading only inside its slot
#pragma unroll
            for (int rr = 0; rr < kR; ++rr)
                if (rr < sg.rows) bad |= 2u * (uint32_t)rel[rr] > prm.vcap;
            if (bad) {
#pragma unroll
                for (int qq = 0; qq < Q; ++qq) {
                    const int rr = qq / kMaxG, j = qq % kMaxG;
                    if (rr < sg.rows && j < sg.g) {
                        const uint32_t a0 = st + (rr ? prm.st_v1 : prm.st_v0) - 4u;
                        const uint32_t te = tb + (uint32_t)(rr * G + j) * 1024u + 8u * lane;
                        sts_v2(te, 0u, a0);
                        sts_v2(te + 256u, 0u, a0);
                        sts_v2(te + 512u, 0u, a0);
                        sts_v2(te + 768u, 0u, a0);
                    }
                }
                if (lane == 0) atomicOr(prm.ws_err, 2);
            }
            __syncwarp();
            // publish the table only once the slot's values and X have landed too, so the decode
            // warps wait on one barrier per stage
            mbar_wait_sleep(bar_full + 8 * slot, sg.par());
            mbar_arrive(bar_scan + 8 * slot);
            // a GT row's GTileOffset range must equal its padded popcounts (the encoding rule): a
            // mismatch (corrupt input) is reported after the tables are published, off the decode's
            // critical path (the range checks of the copies are the producer's). Lane 8 rr + g holds
            // the row's end offset and receives its start from lane 8 rr: one shuffle per stage (the
            // scan warps bound this kernel: a per-GT check before the publish cost 6 % at N = 32)
            {
                const int ob = __shfl_up_sync(0xffffffffu, cur.o, (unsigned)sg.g);
                const int rr_l = lane >> 3;
                const bool chk = lane < 16 && rr_l < sg.rows && (lane & 7) == sg.g;
                if (__any_sync(0xffffffffu, chk && cur.o - ob != (rr_l ? rel[1] : rel[0])) && lane == 0)
                    atomicOr(prm.ws_err, 2);
            }
            skip2(it);
            if (it.valid()) fetch(it, cur);   // this warp's next stage
            return true;
        };
        while (one(F)) {
        }
        return;
    }

    // ---------------------------------------------------------------- decode warps
    const int q = warp & 3, kt = warp >> 2, r = q >> 1;
    const uint32_t mulc = opaque_u32(1u << (30u - 2u * (uint32_t)(lane & 15)));
    const uint32_t t_q = tmem + ((uint32_t)(32 * q) << 16);
    const uint32_t selA = reinterpret_cast<volatile uint32_t *>(smem)[kConstWord];
    const uint32_t selB = reinterpret_cast<volatile uint32_t *>(smem)[kConstWord + 1];
    const uint32_t selC = reinterpret_cast<volatile uint32_t *>(smem)[kConstWord + 2];
    const int N = prm.N;
    const int Nw = (N + 7) & ~7;   // partial row stride (X was padded to a multiple of 8)
    const int row_in = 32 * q + lane;               // row within the 128-row rowblock (= TMEM lane)
    const uint32_t tbl_lane = (uint32_t)(lane >> 4) * 512u + (uint32_t)(q & 1) * 64u;   // + GT * 1024 + tc * 128

    // rowblock epilogue of a segment (D parity db): run by the 4 warps of k-team seg & 3 one stage
    // after the segment's last stage. Sums the k-teams' accumulators in team order
    // (deterministic; nteams = the teams that issued MMAs in the segment).
    auto epilogue = [&](uint32_t db, uint32_t dph_, int rb, int rows, bool complete, int nteams) {
        mbar_wait(bar_df + 8u * db, dph_);
        tm_fence_after();
        float v[NB];
#pragma unroll
        for (int j = 0; j < NB; ++j) v[j] = 0.f;
#pragma unroll
        // NB = 32: a team's two x16 loads in flight per wait (measured -0.5 %); NB = 16: one load and
        // wait per team (batching two teams measured +1.8 %). Summed in team order: deterministic.
#pragma unroll
        for (int tt = 0; tt < 4; ++tt) {
            if (tt < nteams) {
                float x[NB / 16][16];
#pragma unroll
                for (int h = 0; h < NB / 16; ++h)
                    tm_ld_32x32b_x16(t_q + DCol + ((uint32_t)tt * 2u + db) * NB + 16u * h, x[h]);
                tm_wait_ld();
#pragma unroll
                for (int h = 0; h < NB / 16; ++h)
#pragma unroll
                    for (int j = 0; j < 16; ++j) v[16 * h + j] += x[h][j];
            }
        }
        tm_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(bar_de + 8u * db);
        const bool valid = row_in < 64 * rows;
        if (complete) {
            if (valid) store_y_row<NB>(prm, (size_t)rb * 128 + (size_t)row_in, v);
            return;
        }
        // split rowblock: park this CTA's fp32 partial; the last contributor sums (below)
        const int myslot = (rb == u0 / KG) ? 0 : 1;
        if (valid) {
            float4 *pp = reinterpret_cast<float4 *>(prm.ws_part + (((size_t)p * 2 + myslot) * 128 + row_in) * Nw);
#pragma unroll
            for (int c4 = 0; c4 < NB / 4; ++c4)
                if (c4 * 4 < Nw) pp[c4] = make_float4(v[4 * c4], v[4 * c4 + 1], v[4 * c4 + 2], v[4 * c4 + 3]);
        }
        // split-K fix-up per lane quarter, by the warp that parked it (one counter per rowblock
        // and quarter): the last contributor sums every contributor's partial of its 32 rows in
        // CTA order (deterministic), writes Y and re-zeroes the counter. A lane owns one
        // row, so all partials' loads of a row are in flight together (the single producer lane
        // group serving it measured a 10-20 us tail on CTAs whose last segment is split).
        __threadfence();
        __syncwarp();
        const int pf = unit_owner(rb * KG, U, prm.P);
        const int pl = unit_owner((rb + 1) * KG - 1, U, prm.P);
        int old = 0;
        if (lane == 0) old = atomicAdd(prm.ws_cnt + 4 * rb + q, 1);
        old = __shfl_sync(0xffffffffu, old, 0);
        if (old != pl - pf) return;
        __threadfence();
        if (valid) {
            // v (this CTA's partial, parked above) is re-used as the sum
#pragma unroll
            for (int j = 0; j < NB; ++j) v[j] = 0.f;
            for (int qq = pf; qq <= pl; ++qq) {
                const int sl = (rb == unit_start(qq, U, prm.P) / KG) ? 0 : 1;
                const float4 *pp = reinterpret_cast<const float4 *>(prm.ws_part + (((size_t)qq * 2 + sl) * 128 + row_in) * Nw);
#pragma unroll
                for (int c4 = 0; c4 < NB / 4; ++c4)
                    if (c4 * 4 < Nw) {
                        const float4 x = ldg_cg_f4(pp + c4);
                        v[4 * c4] += x.x; v[4 * c4 + 1] += x.y; v[4 * c4 + 2] += x.z; v[4 * c4 + 3] += x.w;
                    }
            }
            store_y_row<NB>(prm, (size_t)rb * 128 + (size_t)row_in, v);
        }
        if (lane == 0) prm.ws_cnt[4 * rb + q] = 0;   // leave the workspace zeroed
    };

    uint4 E[4];
    uint32_t tA0[8], tA1[8], sA[8], tB0[8], tB1[8], sB[8];
    auto load_E = [&](uint32_t tb, int tc) {
#pragma unroll
        for (int k = 0; k < 4; ++k) E[k] = lds_v4(tb + (uint32_t)tc * 128u + 16u * k);
    };
    auto issue = [&](uint32_t (&t0)[8], uint32_t (&t1)[8], uint32_t (&s1)[8]) {
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const uint32_t w = (k & 1) ? E[k >> 1].z : E[k >> 1].x;
            const uint32_t A = (k & 1) ? E[k >> 1].w : E[k >> 1].y;
            const uint32_t z = w * mulc;
            const uint32_t a = A + 2u * __popc(z);
            const uint32_t y = z >> 30;
            s1[k] = y * (y * selB + selA) + selC;
            t0[k] = lds_u16(a);
            t1[k] = lds_u16(a + 2u);
        }
    };
    auto assemble = [&](const uint32_t (&t0)[8], const uint32_t (&t1)[8], const uint32_t (&s1)[8], uint32_t tcol) {
        uint32_t a[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) a[k] = prmt(t0[k], t1[k], s1[k]);
        tm_st_16x128b_x2(t_q + tcol, a[0], a[1], a[2], a[3]);                    // TCTile row 2q
        tm_st_16x128b_x2(t_q + (16u << 16) + tcol, a[4], a[5], a[6], a[7]);      // TCTile row 2q + 1
    };

    // k-team MMA issue (warp q = 0 of the team, one elected lane): tcgen05.mma kind::f16,
    // M = 128, N = NB, K = 16; A = the team's TMEM buffer, B = the TMA-staged X slab (MN-major
    // canonical layout, 32B / 64B swizzle, SBO = 8 k-rows, version 1; verified by
    // tools/tc_probe.cu), D = the team's accumulator of the segment's parity.
    constexpr uint32_t idesc = (1u << 4) | (1u << 16) | ((uint32_t)(NB >> 3) << 17) | ((128u >> 4) << 24);
    constexpr uint64_t kDescHi = ((uint64_t)((8 * NB * 2) >> 4) << 32) | (1ull << 46) |
                                 ((uint64_t)(NB == 16 ? 6 : 4) << 61) | (1ull << 16);
    auto tc_rd = [&](int si) {
        const uint4 v = lds_v4(sbase + prm.o_desc + 16u * (uint32_t)si);
        return StageDesc{v.x, v.y, v.z, v.w};
    };
    Ring<ABufs> ar;
    int seg = -1;
    uint32_t dpar = 1, dph = 1;     // D parity of the current segment and its phase (advanced at segment start)
    bool first = false;             // team: the next MMA starts the segment's accumulation
    int maxg = 0;                   // GT columns of the segment's widest stage (teams kt < maxg multiply)
    bool pend = false;              // pending epilogue of this k-team: run at the end of the stage after its segment
    uint32_t pend_db = 0, pend_dph = 0;
    int pend_rb = 0, pend_rows = 0, pend_nt = 0;
    bool pend_complete = false;
    // per-stage descriptors (built once by scan warp 1): one 16-byte shared load per stage instead
    // of every warp walking the StageIter and the segment flags
    named_bar_sync(kDescBarTC, 32u * (kCW + 1));
    const int nst = (int)reinterpret_cast<volatile uint32_t *>(smem)[kConstWord + 3];
    for (int i = 0; i < nst; ++i, ar.next()) {
        const StageDesc d = tc_rd(i);
        const int slot = d.slot();
        struct { bool zero, seg_end, complete; } sf = {d.zero(), d.seg_end(), d.complete()};
        if (sf.zero) {
            ++seg;
            dpar ^= 1u;
            if (dpar == 0) dph ^= 1u;
            first = true;
            maxg = 0;
        }
        maxg = max(maxg, d.g());
        mbar_wait_sleep(bar_scan + 8 * slot, d.par());   // table written (the scan runs ahead)
        const uint32_t ab = (uint32_t)(kt * ABufs) + ar.b;
        if (i >= ABufs) mbar_wait(bar_ae + 8u * ab, ar.ph ^ 1u);
        tm_fence_after();
        if (r < d.rows() && kt < d.g()) {
            const uint32_t tb = sbase + prm.o_tbl + (uint32_t)slot * prm.tbl_bytes +
                                (uint32_t)(r * G + kt) * 1024u + tbl_lane;
            const uint32_t acol = ab * 32u;
            load_E(tb, 0);
            issue(tA0, tA1, sA);
            load_E(tb, 1);
            issue(tB0, tB1, sB);
            load_E(tb, 2);
            assemble(tA0, tA1, sA, acol + 0u);
            issue(tA0, tA1, sA);
            load_E(tb, 3);
            assemble(tB0, tB1, sB, acol + 8u);
            issue(tB0, tB1, sB);
            assemble(tA0, tA1, sA, acol + 16u);
            assemble(tB0, tB1, sB, acol + 24u);
            tm_wait_st();
        }
        tm_fence_before();
        __syncwarp();
        mbar_arrive(bar_empty + 8 * slot);   // this lane is done with the slot's values/table
        const bool mm = kt < d.g();
        // the team's 4 lane-quarter warps have written their A tiles: the team leader multiplies
        named_bar_sync(kTeamBar + (uint32_t)kt, 128);
        const bool issuer = (q == 0);
        if (issuer) {
            tm_fence_after();
            if (sf.zero && seg >= 2) {   // the D buffer's previous segment has been read out
                mbar_wait(bar_de + 8u * dpar, dph ^ 1u);
                tm_fence_after();
            }
            const uint32_t d_t = tmem + DCol + ((uint32_t)kt * 2u + dpar) * NB;
            const uint32_t a_t = tmem + ab * 32u;
            const uint32_t x_lo = (sbase + prm.o_stage + (uint32_t)slot * prm.stage_bytes) >> 4;
            const uint32_t acc0 = first ? 0u : 1u;
            if (elect_one()) {
                if (mm) {
#pragma unroll
                    for (int tc = 0; tc < 4; ++tc) {
                        const uint64_t bdesc = kDescHi | (uint64_t)((x_lo + (uint32_t)(kt * 4 + tc) * (16u * NB * 2u / 16u)) & 0x3FFFu);
                        umma_f16_ts(d_t, a_t + 8u * (uint32_t)tc, bdesc, idesc, tc == 0 ? acc0 : 1u);
                    }
                }
                umma_commit(bar_ae + 8u * ab);
                umma_commit(bar_emptyx + 8 * slot);
                if (sf.seg_end) umma_commit(bar_df + 8u * dpar);
            }
            __syncwarp();
        }
        if (mm) first = false;
        if (pend) {
            epilogue(pend_db, pend_dph, pend_rb, pend_rows, pend_complete, pend_nt);
            pend = false;
        }
        if (sf.seg_end && (seg & 3) == kt) {
            pend = true;
            pend_db = dpar; pend_dph = dph; pend_rb = d.rb(); pend_rows = d.rows(); pend_complete = sf.complete;
            pend_nt = min(maxg, 4);
        }
    }
    if (pend) epilogue(pend_db, pend_dph, pend_rb, pend_rows, pend_complete, pend_nt);
    tm_fence_before();
    named_bar_sync(kEndBar, 32u * kCW);   // every MMA has completed (the last epilogues waited on them)
    tm_fence_after();
    if (warp == 0) tm_dealloc(tmem, CfgTC::TmemCols);
}
inline uint32_t align_up(uint32_t x, uint32_t a) { return (x + a - 1) / a * a; }

struct Plan {
    int P, G, S;
    size_t smem;
    Params prm;
};

// Ring sizing: a slot holds the X slab (1024-aligned: the TMA swizzle is a function of the smem
// address) and both GT rows' value capacity G * max_gt_values; each slot carries its SMBD table.
bool make_plan(int M, int K, int NB, int max_gt_values, Plan *pl) {
    const int MG = (M + kGT - 1) / kGT, KG = (K + kGT - 1) / kGT;   // zero-padded to whole GTs (A8)
    if (KG > 65535) return false;                                      // StageDesc packs gc in 16 bits
    const long long U = (long long)((MG + kR - 1) / kR) * KG;
    pl->P = choose_grid_rb((MG + kR - 1) / kR, KG);
    if ((unsigned long long)U * (unsigned long long)pl->P >= (1ull << 32)) return false;   // 32-bit unit math
    const long long upc = (U + pl->P - 1) / pl->P;
    const int smem_max = smem_optin();
    int maxv = max_gt_values > 0 ? max_gt_values : 4096;
    maxv = std::min(4096, (maxv + 7) & ~7);
    int gmax = kMaxG, smax = kMaxStages;
    if (option(SPINFER_OPT_STAGE_G) > 0) gmax = std::max(1, std::min(kMaxG, option(SPINFER_OPT_STAGE_G)));
    if (option(SPINFER_OPT_STAGE_S) > 0) smax = std::max(2, std::min(kMaxStages, option(SPINFER_OPT_STAGE_S)));
    // stage descriptors: at most one per unit, and no more than ceil(units / G) + rowblock splits
    for (int G = gmax; G >= 1; --G) {
        const uint32_t tbl = (uint32_t)kR * G * 64 * 16;
        const uint32_t st_v0 = (uint32_t)G * 64 * NB * 2;   // X slab first
        const uint32_t vcap = align_up((uint32_t)G * maxv * 2, 16);
        const uint32_t st_v1 = st_v0 + vcap;
        const uint32_t stage = align_up(st_v1 + vcap, 1024);
        const uint32_t desc_bytes = align_up((uint32_t)(16 * std::min<long long>(upc, upc / G + upc / KG + 3)), 1024);
        const uint32_t fixed = 1024 + desc_bytes + 128 + 1024;
        if ((long long)fixed + 2LL * (stage + tbl) > smem_max) continue;
        const int S = (int)std::min<long long>(smax, ((long long)smem_max - fixed) / (stage + tbl));
        if (S < 3 && G > 1) continue;
        pl->G = G;
        pl->S = S;
        Params &q = pl->prm;
        q.KG = KG; q.MG = MG; q.U = (uint32_t)U; q.P = pl->P; q.G = G; q.S = S;
        q.stage_bytes = stage; q.st_v0 = st_v0; q.st_v1 = st_v1; q.vcap = vcap;
        q.tbl_bytes = tbl;
        q.o_desc = 1024;
        q.o_tbl = q.o_desc + desc_bytes;
        q.o_stage = align_up(q.o_tbl + (uint32_t)S * tbl, 1024);
        pl->smem = (size_t)q.o_stage + (size_t)S * stage + 128 + 1024;   // +1024: runtime base alignment
        return true;
    }
    return false;
}

template <int NB>
int launch_tc(const Plan &pl, cudaStream_t st) {
    static int configured_smem[64] = {0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    if ((int)pl.smem > configured_smem[dev]) {
        if (cudaFuncSetAttribute(k_spmm_tc<NB>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)pl.smem) != cudaSuccess)
            return SPINFER_ECUDA;
        configured_smem[dev] = (int)pl.smem;
    }
    if (option(SPINFER_OPT_PDL)) {   // programmatic dependent launch (layer stacks), see spmm_dw.cu
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3((unsigned)pl.P);
        cfg.blockDim = dim3((unsigned)CfgTC::Threads);
        cfg.dynamicSmemBytes = pl.smem;
        cfg.stream = st;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[0].val.programmaticStreamSerializationAllowed = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        return cudaLaunchKernelEx(&cfg, k_spmm_tc<NB>, pl.prm) == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
    }
    k_spmm_tc<NB><<<pl.P, CfgTC::Threads, pl.smem, st>>>(pl.prm);
    return cudaGetLastError() == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
}

}  // namespace

// Workspace of the tcgen05 kernel: [counters + error word][CTA partials of split rowblocks]
// [zero-padded X].
size_t spmm_tc_workspace_bytes(int M, int K, int N) {
    const int MG = (M + kGT - 1) / kGT, KG = (K + kGT - 1) / kGT;
    const long long U = (long long)((MG + kR - 1) / kR) * KG;
    if (4LL * ((MG + kR - 1) / kR) >= kErrWord) return 0;   // one counter per rowblock and TMEM lane quarter
    const int P = choose_grid_rb((MG + kR - 1) / kR, KG);
    const int Np = (N + 7) & ~7;
    const size_t part = (size_t)P * 2 * 128 * Np * 4;
    const size_t xpad = (N % 8) ? ((size_t)K * Np * 2 + 255) / 256 * 256 : 0;
    return kCounterRegion + part + xpad;
}

int launch_spmm_tc(const spinfer_tca *T, const uint16_t *X, uint16_t *Y, int M, int K, int N, const uint16_t *bias,
                   int act, void *ws, size_t ws_bytes, cudaStream_t st) {
    const int Np = (N + 7) & ~7;
    const int NB = Np <= 16 ? 16 : 32;   // MMA N (X padded by the TMA's out-of-bounds fill)
    Plan pl;
    if (!make_plan(M, K, NB, T->max_gt_values, &pl)) return SPINFER_EINVAL;
    const size_t need = spmm_tc_workspace_bytes(M, K, N);
    if (need == 0) return SPINFER_EINVAL;
    if (ws == nullptr || ws_bytes < need) return SPINFER_ENOSPC;
    Params &q = pl.prm;
    uint8_t *w8 = reinterpret_cast<uint8_t *>(ws);
    const uint16_t *Xk = X;
    if (N % 8) {   // rows of a zero-padded X copy are 16-byte aligned (the tensor map's stride rule)
        uint16_t *Xp = reinterpret_cast<uint16_t *>(w8 + kCounterRegion + (size_t)pl.P * 2 * 128 * Np * 4);
        if (int rc = launch_pad_x(X, Xp, K, N, Np, st)) return rc;
        Xk = Xp;
    }
    if (int rc = make_x_tmap(&q.tmap_x, Xk, K, Np, NB, 64 * pl.G, true)) return rc;
    q.N = N;
    q.off = T->gtile_offset;
    q.bm = T->bitmap;
    q.vals = T->values;
    q.Y = Y;
    q.bias = bias;
    q.act = act;
    q.ws_cnt = reinterpret_cast<int32_t *>(w8);
    q.ws_part = reinterpret_cast<float *>(w8 + kCounterRegion);
    q.ws_err = reinterpret_cast<int32_t *>(w8) + kErrWord;
    q.n_values = (int)T->n_values;
    q.M = M;
    return NB == 16 ? launch_tc<16>(pl, st) : launch_tc<32>(pl, st);
}

}  // namespace spinfer
