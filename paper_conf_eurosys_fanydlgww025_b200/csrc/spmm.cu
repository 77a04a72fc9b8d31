// spmm.cu — TCA-BME SpMM Y = W x X for sm_100a (§4.3).
//
// One persistent kernel, one CTA per SM. Work = "units": a unit is the column
// of R = 2 GroupTiles (one per GT row of a 128-row "rowblock") at GT column gc,
// linearised u = rb * KG + gc. CTA p owns units [floor(pU/P), floor((p+1)U/P))
// (stream-K: perfect balance in GroupTiles, each CTA reads one contiguous byte
// range per GT row). This replaces the paper's split-K grid mapping (Alg. 1
// lines 1-3); rowblocks split across CTAs are combined by an
// in-kernel "last arriver sums" fix-up (the paper's ReductionWorkspace).
// A "stage" = up to G consecutive units of one rowblock.
//
// Warp roles (11 warps; ids chosen for scheduler priority, see kProducerWarp):
//   top warp  producer: one lane issues, per stage, one cp.async.bulk (1-D TMA) per
//             GT row for the packed values and one for the bitmaps (both contiguous
//             per GT row), and one 2-D tensor TMA per GroupTile column for the X slab
//             (hardware 32B/64B swizzle = the ldmatrix bank-conflict-free layout),
//             all completing on the slot's full mbarrier. S-stage smem ring,
//             full/empty mbarriers (replaces the paper's LDGSTS.128 double buffer,
//             P:224; measured: issuing the bitmaps and X as 16-byte
//             cp.async cost the producer ~1.6K cycles per stage).
//   warps 8,9 scan (one per GT row): for each staged GroupTile computes every BitmapTile's base
//             (PopCount prefix over earlier BTs) and writes a table
//             {bitmap half-word, smem address of that half's first value}.
//   warps 0-7 consumers (GT row r = w/4, TCTile column c = w%4): SMBD decode
//             (MaskedPopCount, Alg. 2, two-phase a0/a1 P:287) into
//             mma.m16n8k16 A fragments, X via ldmatrix.trans, mma.sync with
//             fp32 accumulators (Listing 1).
#include <cuda.h>   // CUtensorMap (type + enums only; the encoder comes via cudaGetDriverEntryPoint)
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include "internal.cuh"
#include "ptx.cuh"

// experiments: force the 8-consumer-warp variant for N <= 16
#ifndef SPINFER_FORCE_KQ1
#define SPINFER_FORCE_KQ1 0
#endif

namespace spinfer {
namespace {

constexpr int kR = 2;               // GT rows per rowblock (128 output rows)
constexpr int kScanWarps = kR;      // one scan warp per GT row of the rowblock
// Consumer layout: kR GT rows x 4 TCTile columns x KQ GT-parities (warp q of a (row,
// column) pair takes GTs j = q, q+KQ, ... of a stage). KQ = 2 (16 consumer warps) gives
// the scheduler enough warps to hide ALU/XU/LDS latencies; it needs the accumulators to
// fit the tighter register budget, so N >= 24 uses KQ = 1.
template <int NT> struct Cfg {
    static constexpr int KQ = (NT <= 2 && !SPINFER_FORCE_KQ1) ? 2 : 1;
    static constexpr int CW = kR * 4 * KQ;                        // consumer warps
    static constexpr int FixWarp = CW;                            // warp ids: the scheduler favours the
    static constexpr int ScanWarp = CW + 1;                       // highest id, so roles go on top
    static constexpr int ProducerWarp = CW + 1 + kScanWarps;
    static constexpr int Threads = 32 * (CW + kScanWarps + 2);
};
constexpr int kMaxStages = 8;
#ifndef SPINFER_SCANSPIN
#define SPINFER_SCANSPIN 0
#endif
#ifndef SPINFER_CONSSPIN
#define SPINFER_CONSSPIN 0
#endif
#ifndef SPINFER_PIPEMIX
#define SPINFER_PIPEMIX 1
#endif
#ifndef SPINFER_MAXG
#define SPINFER_MAXG 4
#endif
// register split between the warp roles (setmaxnreg, per warpgroup): the consumer warpgroups
// grow to SPINFER_MAXNREG registers, the role warpgroup (fix-up, scan, producer) shrinks to
// SPINFER_ROLEREG; 0 = one budget for all warps
#ifndef SPINFER_MAXNREG
#define SPINFER_MAXNREG 0
#endif
#ifndef SPINFER_ROLEREG
#define SPINFER_ROLEREG 56
#endif
// software-pipelined consumer loop also for the 16-warp (KQ = 2) variant
// asynchronous rowblock epilogue: at a segment end that is not the CTA's last, every consumer
// warp parks its fp32 partial in the workspace (L2) and moves on; the fix-up warp sums the
// partials in warp order (deterministic) and writes Y / joins the split-K fix-up
#ifndef SPINFER_AEPI
#define SPINFER_AEPI 0
#endif
// waits of the fix-up warp / the producer: timed back-off (not woken by the CTA's other barrier
// traffic) instead of the event-woken suspend of mbar_wait_sleep; 0 = suspend
#ifndef SPINFER_FIXBO
#define SPINFER_FIXBO 0
#endif
#ifndef SPINFER_PRODBO
#define SPINFER_PRODBO 0
#endif
#ifndef SPINFER_PAGEPF
#define SPINFER_PAGEPF 1
#endif
// bitmaps complete on their own mbarrier: the scan builds a stage's table while the stage's
// values are still landing; consumers then wait for the table and for the values
#ifndef SPINFER_BMBAR
#define SPINFER_BMBAR 0
#endif
// slot release: the consumer warps count themselves on a shared counter and only the last one
// arrives on the slot's empty mbarrier (1 barrier event per stage instead of 16: every mbarrier
// event wakes every suspended waiter of the CTA)
#ifndef SPINFER_RELCNT
#define SPINFER_RELCNT 0
#endif
// scan warps walk the per-CTA stage descriptors instead of their own StageIter
#ifndef SPINFER_SCANDESC
#define SPINFER_SCANDESC 0
#endif
#ifndef SPINFER_EPREF
#define SPINFER_EPREF 0
#endif
#ifndef SPINFER_PIPE2
#define SPINFER_PIPE2 0
#endif
constexpr int kMaxG = SPINFER_MAXG;  // max GroupTile columns per stage (the scan unrolls over it)
constexpr int kConstWord = 48;      // smem word index (byte 192) of the SMBD selector-table constants
constexpr int kTraceCTAs = 4, kTraceStages = 64, kTraceW = 20, kTraceEv = 4;   // stage 63 = kernel-level events
// Workspace = [fix-up counters: one int32 per GT row, fixed-size region][split-K partials].
// The counter region has the same size for every shape so that one zeroed
// workspace can serve calls of different shapes (partials never overlap counters).
constexpr int kMaxCounters = 16384;                 // M <= 1,048,576 rows
constexpr size_t kCounterBytes = (size_t)kMaxCounters * 4;

struct Params {
    CUtensorMap tmap_x;          // X [K][N] fp16, box {N, 64}, swizzle 32B (N=16) / 64B (N=32) / none
    const int32_t *off;
    const uint64_t *bm;
    const uint16_t *vals;
    const uint16_t *X;
    uint16_t *Y;
    float *ws_part;
    const uint16_t *bias;   // fused epilogue (spinfer_spmm_ex): fp16 [M] or null
    int act;                // SPINFER_ACT_NONE / SPINFER_ACT_RELU
    float *ws_epi;      // [P][2 buffers][kR][8 warps][64 x N] fp32 partials of the asynchronous epilogue
    int32_t *ws_cnt;
    int KG, MG;
    int N;                                      // real N (the tcgen05 path pads X to NB via TMA OOB fill)
    uint32_t U;                                 // units (rowblock x GT column); U * P < 2^32
    int P;
    int G, S;
    uint32_t stage_bytes, st_bm, st_v0, st_v1;  // stage slot size; offsets in a slot (X slab at 0)
    uint32_t tbl_bytes;
    uint32_t o_desc, o_tbl, o_stage;            // region offsets from the smem base
    long long *trace;   // experiments only (SPINFER_TRACE): [kTraceCTAs][kTraceStages][8] clock64 stamps
    float avg_gt;       // n_values / NGT: predicts where a CTA's first value range lies (start-up page prefetch)
    int M;              // real rows of Y (M need not be a multiple of 64: rows >= M are padding, A8)
    int dbg;            // experiments only (SPINFER_DEBUG_MODE): bit0 = consumers skip decode/MMA, bit1 = scan skips work
};

// Experiment instrumentation (stage timeline, debug modes) is compiled in only with
// -DSPINFER_INSTRUMENT=1 (stage trace + debug modes) or =2 (debug modes only: trace stores
// slow down the traced CTAs, which then set the kernel time); the product build has none of it.
#ifndef SPINFER_INSTRUMENT
#define SPINFER_INSTRUMENT 0
#endif
// trace[p][stage][warp][ev] (lane 0 of the warp records): consumers ev0 wait start, ev1 wait
// end, ev2 decode end, ev3 slot released; scan ev0/ev1 wait, ev3 table published; producer
// ev0 wait start, ev1 copies issued. Stage kTraceStages-1: ev0 entry, ev1 after the initial
// __syncthreads, ev2 main loop done, ev3 exit.
__device__ __forceinline__ void trace_ev(const Params &prm, int p, int i, int w, int ev) {
#if SPINFER_INSTRUMENT == 1
    if (prm.trace && p < kTraceCTAs && i < kTraceStages - 1 && w < kTraceW)
        prm.trace[(((size_t)p * kTraceStages + i) * kTraceW + w) * kTraceEv + ev] = clock64();
#endif
}
constexpr size_t kTraceBase2 = (size_t)kTraceCTAs * kTraceStages * kTraceW * kTraceEv;   // then [CTA][entry, exit] ns, [CTA] smid
constexpr int kTraceMaxCTAs = 1024;
#if SPINFER_INSTRUMENT == 1
__device__ __forceinline__ unsigned long long globaltimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
#endif
__device__ __forceinline__ void trace_k(const Params &prm, int p, int w, int ev) {
#if SPINFER_INSTRUMENT == 1
    if (prm.trace && p < kTraceCTAs && w < kTraceW)
        prm.trace[(((size_t)p * kTraceStages + kTraceStages - 1) * kTraceW + w) * kTraceEv + ev] = clock64();
    // every CTA: entry (warp 0) and exit (last warp out) on the global ns timer
    if (prm.trace && p < kTraceMaxCTAs) {
        unsigned long long *g = reinterpret_cast<unsigned long long *>(prm.trace + kTraceBase2);
        if (ev == 0 && w == 0) {
            uint32_t smid;
            asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
            g[2 * p] = globaltimer_ns();
            g[2 * kTraceMaxCTAs + p] = smid;
        }
        if (ev == 3) atomicMax(g + 2 * p + 1, globaltimer_ns());
    }
#endif
}
__device__ __forceinline__ int dbg_mode(const Params &prm) {
#if SPINFER_INSTRUMENT
    return prm.dbg;
#else
    return 0;
#endif
}

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

// X slab swizzle (16-byte chunk granularity): row k of the slab holds N/8 chunks;
// chunk c of row k is stored at chunk slot c ^ swz(k) so that the 8 row reads of
// one ldmatrix phase hit 8 distinct bank groups (N = 16: rows are 32 B apart,
// rows k and k+4 would collide; N = 32: rows k, k+2). N = 8 and 24 are conflict-free.
// The TMA writes this layout: its SWIZZLE_32B / SWIZZLE_64B modes XOR the chunk index
// with smem address bits 7 (/ 7-8), i.e. with (k >> 2) & 1 (N = 16) and (k >> 1) & 3
// (N = 32) for a slab that starts 1024-byte aligned.
template <int NT>
__device__ __forceinline__ uint32_t x_swz(uint32_t k) {
    if constexpr (NT == 2) return (k >> 2) & 1u;
    else if constexpr (NT == 4) return (k >> 1) & 3u;
    else return 0u;
}

// SMBD for one BitmapTile and one lane, split into phases so
// a warp keeps many shared-memory loads in flight. The scan warps' table entry for
// (BT, lane-half h) is {w, A}: w = bitmap word h (bits 32h..32h+31), A = smem byte
// address of the first value of that half, minus 4. With sh = 2*(lane%16):
//   z  = w << (30 - sh)          top two bits = y = (bit sh, bit sh+1) of w
//   c2 = PopCount(z)             = MaskedPopCount (Alg. 2) + bit sh + bit sh+1
//   t_lo = V[c2 - 2], t_hi = V[c2 - 1]   (zero-extended u16 loads)
//   a0 = bit sh ? (bit sh+1 ? t_lo : t_hi) : 0     (Phase I)
//   a1 = bit sh+1 ? t_hi : 0                        (Phase II reuses the count)
// The four y cases are one PRMT of {t_lo, t_hi}; zero halves select the u16 loads'
// zero upper bytes (bytes 2/3 of t_lo, 6/7 of t_hi, optionally in sign-replicate mode):
//   y=0 -> (0,0)  y=1 -> (t_hi,0)  y=2 -> (0,t_hi)  y=3 -> (t_lo,t_hi)
// The selector is the quadratic sel(y) = y*(kSelA + kSelB*y) + kSelC (mod 2^16), found by
// exhaustive search (tools/selector_search.py; pinned in tests/test_host_logic.py) —
// two IMADs on the FMA pipe instead of ALU-pipe work (the ALU pipe is half rate on B200).
constexpr uint32_t kSelA = 0x7f62u, kSelB = 0x4cbfu, kSelC = 0x2333u;

// N = the caller's column count (row stride of Y); the kernel computes NT * 8 >= N columns
// (X zero-padded to a multiple of 8) and drops the padding columns here.
// Fused epilogue of one output (spinfer_spmm_ex): + bias[row] and the activation, in fp32.
__device__ __forceinline__ float epi_act(float v, float b, int act) {
    v += b;
    return act == SPINFER_ACT_RELU ? fmaxf(v, 0.f) : v;
}

// prm.N = the caller's column count (row stride of Y); the kernel computes NT * 8 >= N columns
// (X zero-padded to a multiple of 8) and drops the padding columns here.
// EPI: the general path — fused bias / activation (spinfer_spmm_ex) and the padding rows of a
// ragged M (A8); the plain path (EPI = false) is only launched for M % 64 == 0 without epilogue.
template <int NT, bool EPI>
__device__ __forceinline__ void store_y(const Params &prm, int row_base, float (&acc)[4][NT][4], int lane) {
    uint16_t *const Y = prm.Y;
    const int N = prm.N;
#pragma unroll
    for (int tr = 0; tr < 4; ++tr) {
        const int r0 = row_base + tr * 16 + (lane >> 2);
        if (EPI && (prm.bias || prm.act)) {   // fused epilogue (general instantiation only)
            const float b0 = prm.bias ? __half2float(__ushort_as_half(prm.bias[r0])) : 0.f;
            const float b1 = prm.bias ? __half2float(__ushort_as_half(prm.bias[r0 + 8])) : 0.f;
#pragma unroll
            for (int nt = 0; nt < NT; ++nt) {
                acc[tr][nt][0] = epi_act(acc[tr][nt][0], b0, prm.act);
                acc[tr][nt][1] = epi_act(acc[tr][nt][1], b0, prm.act);
                acc[tr][nt][2] = epi_act(acc[tr][nt][2], b1, prm.act);
                acc[tr][nt][3] = epi_act(acc[tr][nt][3], b1, prm.act);
            }
        }
#pragma unroll
        for (int nt = 0; nt < NT; ++nt) {
            int col = nt * 8 + 2 * (lane & 3);
            __half2 lo = __floats2half2_rn(acc[tr][nt][0], acc[tr][nt][1]);   // one RNE per output (A11)
            __half2 hi = __floats2half2_rn(acc[tr][nt][2], acc[tr][nt][3]);
            if (EPI && r0 + 8 >= prm.M) {   // last GT row of a ragged M (A8): padding rows are not stored
                __half *y0 = reinterpret_cast<__half *>(Y + (size_t)r0 * N);
                __half *y1 = reinterpret_cast<__half *>(Y + (size_t)(r0 + 8) * N);
                if (r0 < prm.M && col < N) y0[col] = __low2half(lo);
                if (r0 < prm.M && col + 1 < N) y0[col + 1] = __high2half(lo);
                if (r0 + 8 < prm.M && col < N) y1[col] = __low2half(hi);
                if (r0 + 8 < prm.M && col + 1 < N) y1[col + 1] = __high2half(hi);
            } else if (N == NT * 8) {
                *reinterpret_cast<__half2 *>(Y + (size_t)r0 * N + col) = lo;
                *reinterpret_cast<__half2 *>(Y + (size_t)(r0 + 8) * N + col) = hi;
            } else {
                __half *y0 = reinterpret_cast<__half *>(Y + (size_t)r0 * N);
                __half *y1 = reinterpret_cast<__half *>(Y + (size_t)(r0 + 8) * N);
                if (col < N) { y0[col] = __low2half(lo); y1[col] = __low2half(hi); }
                if (col + 1 < N) { y0[col + 1] = __high2half(lo); y1[col + 1] = __high2half(hi); }
            }
        }
    }
}

// Last contributor of a split rowblock: sum every contributor's fp32 partial in CTA order
// (deterministic; its own partial included), write Y, re-zero the counter.
template <int NT, bool EPI>
__device__ __forceinline__ void fixup_sum(const Params &prm, int rb, int r, int pf, int pl, int lane) {
    constexpr int N = NT * 8;
    __threadfence();
    float acc[4][NT][4];
#pragma unroll
    for (int tr = 0; tr < 4; ++tr)
#pragma unroll
        for (int nt = 0; nt < NT; ++nt)
#pragma unroll
            for (int e = 0; e < 4; ++e) acc[tr][nt][e] = 0.f;
    for (int qq = pf; qq <= pl; ++qq) {
        const int sl = (rb == unit_start(qq, prm.U, prm.P) / prm.KG) ? 0 : 1;
        const float4 *pp = reinterpret_cast<const float4 *>(prm.ws_part) + (((size_t)qq * 2 + sl) * kR + r) * (64 * N / 4);
#pragma unroll
        for (int tr = 0; tr < 4; ++tr)
#pragma unroll
            for (int nt = 0; nt < NT; ++nt) {
                float4 v = ldg_cg_f4(pp + (tr * NT + nt) * 32 + lane);
                acc[tr][nt][0] += v.x; acc[tr][nt][1] += v.y; acc[tr][nt][2] += v.z; acc[tr][nt][3] += v.w;
            }
    }
    const int grow = kR * rb + r;
    store_y<NT, EPI>(prm, grow * 64, acc, lane);
    if (lane == 0) prm.ws_cnt[grow] = 0;   // leave the workspace zeroed
}

template <int NT, bool EPI>
__global__ void __launch_bounds__(Cfg<NT>::Threads, 1) k_spmm(const __grid_constant__ Params prm) {
    constexpr int N = NT * 8;
    constexpr int KQ = Cfg<NT>::KQ, kCW = Cfg<NT>::CW;
    constexpr int kScanWarp = Cfg<NT>::ScanWarp, kProducerWarp = Cfg<NT>::ProducerWarp, kFixWarp = Cfg<NT>::FixWarp;
    // named barriers: 0 = __syncthreads, 1..kR = epilogue (per GT row), kDescBar = descriptors ready
    constexpr uint32_t kDescBar = 1 + kR;
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    // ring slots are 1024-byte aligned relative to this base: the TMA swizzle pattern of the
    // X slab is a function of the smem address bits (x_swz assumes slab-relative row index)
    uint8_t *const smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    const uint32_t sbase = smem_u32(smem);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int p = blockIdx.x;
    const uint32_t U = prm.U;
    const int KG = prm.KG, G = prm.G, S = prm.S;
    const int u0 = unit_start(p, U, prm.P), u1 = unit_start(p + 1, U, prm.P);

    // barriers: full[S], empty[S], scanned[2], tbl_empty[2]
    const uint32_t bar_full = sbase, bar_empty = sbase + 8 * kMaxStages;
    // barriers: full[S] (data landed), empty[S] (consumers done), scanned[S] (table written;
    // the scan warps acquired full[s] first, so consumers wait on scanned[s] only)
    const uint32_t bar_scan = sbase + 16 * kMaxStages;
    const uint32_t bar_fix = sbase + 208;   // [split segment A/C][GT row]: partial parked (32 lanes)
    const uint32_t bar_epi = sbase + 256;   // [buffer][GT row]: the row's consumer warps parked their partials
    const uint32_t bar_epifree = sbase + 288;   // [buffer]: the fix-up warp has read the buffer
    const uint32_t bar_bm = sbase + 320;    // [S]: the slot's bitmaps landed (SPINFER_BMBAR)
#if SPINFER_RELCNT
    const uint32_t rel_cnt = sbase + 384;   // [S] u32: consumer warps done with the slot (SPINFER_RELCNT)
#endif

    if (lane == 0) trace_k(prm, p, warp, 0);
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(bar_full + 8 * s, 1);       // the producer's arrive.expect_tx (+ TMA transaction bytes)
            mbar_init(bar_bm + 8 * s, 1);
            mbar_init(bar_empty + 8 * s, SPINFER_RELCNT ? 1 : kCW);
            reinterpret_cast<uint32_t *>(smem + 384)[s] = 0u;
        }
        for (int s = 0; s < S; ++s) mbar_init(bar_scan + 8 * s, kScanWarps);   // one elected arrive per scan warp
        for (int k = 0; k < 2 * kR; ++k) mbar_init(bar_fix + 8 * k, 32);
        for (int k = 0; k < 2 * kR; ++k) mbar_init(bar_epi + 8 * k, 4 * KQ);
        for (int k = 0; k < 2; ++k) mbar_init(bar_epifree + 8 * k, 1);
        fence_barrier_init();
        // SMBD selector-table constants, read back into registers by every consumer thread so
        // ptxas keeps them live in registers instead of re-materialising them per PRMT.
        reinterpret_cast<uint32_t *>(smem)[kConstWord] = kSelA;
        reinterpret_cast<uint32_t *>(smem)[kConstWord + 1] = kSelB;
        reinterpret_cast<uint32_t *>(smem)[kConstWord + 2] = kSelC;
    }
    // The producer's first GTileOffset reads go out before the block barrier (no shared state).
    StageIter pit;
    int4 poff = make_int4(0, 0, 0, 0);   // {start, end} of the stage's values, GT rows 0 and 1
    auto load_off = [&](const StageIter &sg) {
        const int g0 = kR * sg.rb * KG + sg.gc;
        int4 v;
        v.x = __ldg(prm.off + g0);
        v.y = __ldg(prm.off + g0 + sg.g);
        v.z = sg.rows > 1 ? __ldg(prm.off + g0 + KG) : 0;
        v.w = sg.rows > 1 ? __ldg(prm.off + g0 + KG + sg.g) : 0;
        return v;
    };
    if (warp == kProducerWarp && lane == 0) {
        prefetch_tmap(&prm.tmap_x);
#if SPINFER_PAGEPF
        // Start-up: the first value copies wait for their GTileOffset entries; touching the
        // predicted first value line of each GT row now overlaps that page's translation with
        // the offset loads (a hint only: nothing depends on the prediction).
        {
            const int rb0 = u0 / KG, gc0 = u0 - rb0 * KG;
            for (int r = 0; r < kR && kR * rb0 + r < prm.MG; ++r) {
                const long long g = (long long)(kR * rb0 + r) * KG + gc0;
                prefetch_l2(prm.vals + (long long)((double)g * prm.avg_gt));
            }
        }
#endif
        pit.init(u0, u1, prm);
        if (pit.valid()) poff = load_off(pit);
    }
    __syncthreads();
    if (lane == 0) trace_k(prm, p, warp, 1);
#if SPINFER_MAXNREG
    if (warp >= kCW) setmaxnreg_dec<SPINFER_ROLEREG>();
    else setmaxnreg_inc<SPINFER_MAXNREG>();
#endif

    if (warp == kProducerWarp) {
        // ------------------------------------------------------------ producer
        if (lane != 0) return;
        const uint64_t pol_w = policy_evict_first();
        const uint32_t xbytes = 64u * N * 2u;          // one GroupTile column of X
        for (; pit.valid();) {
            const StageIter sg = pit;
            const int i = sg.i, slot = sg.slot;
            if ((dbg_mode(prm) & 4) && i > 0) break;   // experiment: consumers reuse stage 0 forever
            trace_ev(prm, p, i, warp, 0);
#if SPINFER_PRODBO
            if (i >= S) mbar_wait_backoff(bar_empty + 8 * slot, sg.par() ^ 1u, 32u, SPINFER_PRODBO);
#else
            if (i >= S) mbar_wait_sleep(bar_empty + 8 * slot, sg.par() ^ 1u);
#endif
            const uint32_t st = sbase + prm.o_stage + slot * prm.stage_bytes;
            const uint32_t fb = bar_full + 8 * slot;
            const uint32_t bmb = (uint32_t)sg.g * 512u;
            // X and bitmaps first (no offsets needed); the arrive comes with the value bytes last,
            // so the phase cannot complete before every transaction is registered
#if SPINFER_BMBAR
            mbar_arrive_expect_tx(bar_bm + 8 * slot, (uint32_t)sg.rows * bmb);
            for (int r = 0; r < sg.rows; ++r)
                bulk_g2s(st + prm.st_bm + (uint32_t)(r * G) * 512u,
                         prm.bm + ((size_t)(kR * sg.rb + r) * KG + sg.gc) * 64, bmb, bar_bm + 8 * slot, pol_w);
            mbar_expect_tx(fb, (uint32_t)G * xbytes);
#else
            mbar_expect_tx(fb, (uint32_t)sg.rows * bmb + (uint32_t)G * xbytes);
            for (int r = 0; r < sg.rows; ++r)
                bulk_g2s(st + prm.st_bm + (uint32_t)(r * G) * 512u,
                         prm.bm + ((size_t)(kR * sg.rb + r) * KG + sg.gc) * 64, bmb, fb, pol_w);
#endif
            // X slab rows [64 gc, 64 (gc + G)) in one tensor TMA (box {N, 64 G}; rows past K are
            // zero-filled): L2-resident (every CTA reads X), default policy
            tma_2d_g2s(st, &prm.tmap_x, 0, 64 * sg.gc, fb);
            const int4 o = poff;
            const uint32_t vb0 = 2u * (uint32_t)(o.y - o.x);
            const uint32_t vb1 = sg.rows > 1 ? 2u * (uint32_t)(o.w - o.z) : 0u;
            if (vb0) bulk_g2s(st + prm.st_v0, prm.vals + o.x, vb0, fb, pol_w);
            if (vb1) bulk_g2s(st + prm.st_v1, prm.vals + o.z, vb1, fb, pol_w);
            mbar_arrive_expect_tx(fb, vb0 + vb1);
            // next stage's offsets: in flight while this warp waits for a free slot
            pit.next(prm);
            if (pit.valid()) poff = load_off(pit);
            trace_ev(prm, p, i, warp, 1);
        }
        trace_k(prm, p, warp, 3);
        return;
    }

    if (warp == kFixWarp) {
#if SPINFER_AEPI
        // ------------------------------------------------------------ epilogue + split-K fix-up
        // Walks the CTA's stage sequence. At every segment end except the last: waits for the
        // row's 4*KQ consumer partials (workspace, L2), sums them in warp order, and writes Y
        // (complete rowblock) or parks the CTA partial and joins the cross-CTA count; the last
        // contributor sums all partials in CTA order. The CTA's last segment is reduced
        // by the consumers themselves (nothing left to overlap); if it is split, its leader
        // parks the partial on bar_fix as before.
        {
            StageIter d;
            bool full_start = false;
            int segi = 0;
            for (d.init(u0, u1, prm); d.valid();) {
                const bool zero = d.seg_first();
                if (zero) full_start = (d.gc == 0);
                const bool seg_end = d.seg_last(prm);
                const bool complete = seg_end && full_start && (d.gc + d.g == KG);
                const int rb = d.rb, rows = d.rows;
                d.next(prm);
                if (!seg_end) continue;
                const bool last = !d.valid();
                const int myslot = (rb == u0 / KG) ? 0 : 1;
                const int pf = unit_owner(rb * KG, U, prm.P);
                const int pl = unit_owner((rb + 1) * KG - 1, U, prm.P);
                auto count_and_sum = [&](int r) {
                    int old = 0;
                    if (lane == 0) old = atomicAdd(prm.ws_cnt + kR * rb + r, 1);
                    old = __shfl_sync(0xffffffffu, old, 0);
                    if (old == pl - pf) fixup_sum<NT, EPI>(prm, rb, r, pf, pl, lane);   // last contributor
                };
                if (last) {
                    if (!complete)
                        for (int r = 0; r < rows; ++r) {
                            mbar_wait_sleep(bar_fix + 8u * (uint32_t)(2 * myslot + r), 0u);
                            __threadfence();   // cumulative: the consumer's partial stores before the count
                            count_and_sum(r);
                        }
                    break;
                }
                const uint32_t buf = (uint32_t)segi & 1u, ph = ((uint32_t)segi >> 1) & 1u;
                for (int r = 0; r < rows; ++r) {
                    mbar_wait_sleep(bar_epi + 8u * (buf * kR + (uint32_t)r), ph);
                    float acc[4][NT][4];
#pragma unroll
                    for (int tr = 0; tr < 4; ++tr)
#pragma unroll
                        for (int nt = 0; nt < NT; ++nt)
#pragma unroll
                            for (int e = 0; e < 4; ++e) acc[tr][nt][e] = 0.f;
                    const float4 *src = reinterpret_cast<const float4 *>(prm.ws_epi) +
                                        (((size_t)p * 2 + buf) * kR + r) * 8 * (64 * N / 4);
                    for (int w = 0; w < 4 * KQ; ++w)
#pragma unroll
                        for (int tr = 0; tr < 4; ++tr) {
                            float4 v[NT];
#pragma unroll
                            for (int nt = 0; nt < NT; ++nt)
                                v[nt] = ldg_cg_f4(src + (size_t)w * (64 * N / 4) + (tr * NT + nt) * 32 + lane);
#pragma unroll
                            for (int nt = 0; nt < NT; ++nt) {
                                acc[tr][nt][0] += v[nt].x; acc[tr][nt][1] += v[nt].y;
                                acc[tr][nt][2] += v[nt].z; acc[tr][nt][3] += v[nt].w;
                            }
                        }
                    const int grow = kR * rb + r;
                    if (complete) {
                        store_y<NT, EPI>(prm, grow * 64, acc, lane);
                    } else {
                        float4 *part = reinterpret_cast<float4 *>(prm.ws_part) + (((size_t)p * 2 + myslot) * kR + r) * (64 * N / 4);
#pragma unroll
                        for (int tr = 0; tr < 4; ++tr)
#pragma unroll
                            for (int nt = 0; nt < NT; ++nt)
                                part[(tr * NT + nt) * 32 + lane] =
                                    make_float4(acc[tr][nt][0], acc[tr][nt][1], acc[tr][nt][2], acc[tr][nt][3]);
                        __threadfence();
                        __syncwarp();
                        count_and_sum(r);
                    }
                }
                __syncwarp();
                if (lane == 0) mbar_arrive(bar_epifree + 8u * buf);   // the buffer may be overwritten
                ++segi;
            }
        }
        return;
#endif
        // ------------------------------------------------------------ split-K fix-up
        // At most two split segments per CTA (A: tail of the first rowblock, C: head of the
        // last), processed first in StageIter order; for each and each GT row the reducing
        // consumer parks its partial and arrives on bar_fix[seg][row].
        const int a_rb = u0 / KG, c_rb = (u1 - 1) / KG;
        const bool has_a = (u0 % KG) != 0;
        const bool has_c = (u1 % KG) != 0 && !(has_a && c_rb == a_rb);
        for (int sgi = 0; sgi < 2; ++sgi) {
            if (!(sgi == 0 ? has_a : has_c)) continue;
            const int rb = sgi == 0 ? a_rb : c_rb;
            const int myslot = (rb == u0 / KG) ? 0 : 1;
            const int rows = min(kR, prm.MG - kR * rb);
            for (int r = 0; r < rows; ++r) {
#if SPINFER_FIXBO
                // the parked partial is not urgent: poll every few microseconds at most instead of
                // waking on each of the CTA's ~30 barrier events per stage
                mbar_wait_backoff(bar_fix + 8u * (uint32_t)(2 * myslot + r), 0u, 256u, 2048u);
#else
                mbar_wait_sleep(bar_fix + 8u * (uint32_t)(2 * myslot + r), 0u);
#endif
                __threadfence();   // cumulative: the consumer's partial stores before the count
                const int pf = unit_owner(rb * KG, U, prm.P);
                const int pl = unit_owner((rb + 1) * KG - 1, U, prm.P);
                int old = 0;
                if (lane == 0) old = atomicAdd(prm.ws_cnt + kR * rb + r, 1);
                old = __shfl_sync(0xffffffffu, old, 0);
                if (old == pl - pf) fixup_sum<NT, EPI>(prm, rb, r, pf, pl, lane);   // last contributor
            }
        }
        return;
    }

    if (warp >= kScanWarp && warp < kScanWarp + kScanWarps) {
        // ------------------------------------------------------------ scan
        // Table per staged GT (r, j), 1024 B: [lane-half h][BT in GT storage order] {w, A},
        // so a consumer lane fetches the entries of 2 consecutive BTs with one 16-B load.
        // Scan warp r handles GT row r; the g GTs of a stage are scanned together (static
        // bounds, unconditional full-warp shuffles, absent GTs scan zeros) so the
        // independent shuffle chains interleave.
        constexpr int Q = kMaxG;
        const int r = warp - kScanWarp;               // this scan warp's GT row
        const bool work = !(dbg_mode(prm) & 2);
        if (r == 0) {
            // stage descriptors for the consumers (in the shadow of the first data latency)
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
                    const uint32_t sl = (dbg_mode(prm) & 4) ? 0u : (uint32_t)d.slot;   // experiment: reuse slot 0
                    sts_v4(sbase + prm.o_desc + 16u * (uint32_t)n,
                           make_uint4(w0, (uint32_t)d.gc | ((uint32_t)d.g << 16), prm.o_tbl + sl * prm.tbl_bytes,
                                      prm.o_stage + sl * prm.stage_bytes));
                }
                reinterpret_cast<volatile uint32_t *>(smem)[kConstWord + 3] = (uint32_t)n;
            }
            __syncwarp();
            named_bar_arrive(kDescBar, 32u * (kCW + 1 + SPINFER_SCANDESC));
        }
#if SPINFER_SCANDESC
        // walk the stage descriptors (scan warp 0 wrote them above) instead of the StageIter
        if (r != 0) named_bar_sync(kDescBar, 32u * (kCW + 2));
        const int nst_s = (int)reinterpret_cast<volatile uint32_t *>(smem)[kConstWord + 3];
        for (int i = 0; i < nst_s; ++i) {
            const uint4 dv = lds_v4(sbase + prm.o_desc + 16u * (uint32_t)i);
            const StageDesc dd{dv.x, dv.y, dv.z, dv.w};
            const int slot = dd.slot();
            const uint32_t spar = dd.par();
            const struct { int rows, g; } sg = {dd.rows(), dd.g()};
#else
        StageIter it;
        for (it.init(u0, u1, prm); it.valid(); it.next(prm)) {
            const StageIter &sg = it;
            const int i = it.i, slot = it.slot;
            const uint32_t spar = it.par();
#endif
            if ((dbg_mode(prm) & 4) && i > 0) break;
            // suspend (not spin) while waiting: these warps have the highest scheduling
            // priority and would otherwise steal issue slots from the consumers
            if (lane == 0) trace_ev(prm, p, i, warp, 0);
#if SPINFER_SCANSPIN
            mbar_wait(bar_full + 8 * slot, spar);
#else
#if SPINFER_BMBAR
            mbar_wait_sleep(bar_bm + 8 * slot, spar);   // the scan reads only the bitmaps
#else
            mbar_wait_sleep(bar_full + 8 * slot, spar);
#endif
#endif
            if (lane == 0) trace_ev(prm, p, i, warp, 1);
            uint2 ba[Q], bb[Q];
#pragma unroll
            for (int q = 0; q < Q; ++q) {
                const int j = q;
                const uint32_t bmsm = sbase + prm.o_stage + slot * prm.stage_bytes + prm.st_bm + (uint32_t)(r * G + j) * 512u;
                if (work && r < sg.rows && j < sg.g) {
                    ba[q] = lds_v2(bmsm + 8u * lane);          // BT `lane` of the GT (storage order)
                    bb[q] = lds_v2(bmsm + 256u + 8u * lane);   // BT `lane + 32`
                } else {
                    ba[q] = make_uint2(0u, 0u);
                    bb[q] = make_uint2(0u, 0u);
                }
            }
            const uint32_t st = sbase + prm.o_stage + slot * prm.stage_bytes;
            const uint32_t tb = sbase + prm.o_tbl + slot * prm.tbl_bytes;   // one table per ring slot
            uint32_t packed[Q], incl[Q];
#pragma unroll
            for (int q = 0; q < Q; ++q) {
                packed[q] = (__popc(ba[q].x) + __popc(ba[q].y)) | ((__popc(bb[q].x) + __popc(bb[q].y)) << 16);
                incl[q] = packed[q];
            }
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                uint32_t y[Q];
#pragma unroll
                for (int q = 0; q < Q; ++q) y[q] = __shfl_up_sync(0xffffffffu, incl[q], o);
#pragma unroll
                for (int q = 0; q < Q; ++q) incl[q] += (lane >= o) ? y[q] : 0u;
            }
            uint32_t tot_a[Q];
            int rel = 0;   // GT j's first value within the row's chunk: earlier GTs' counts, each padded
                           // to a multiple of 8 values (the GTileOffset rule, encode.cu)
#pragma unroll
            for (int q = 0; q < Q; ++q) {
                const uint32_t t = __shfl_sync(0xffffffffu, incl[q], 31);
                tot_a[q] = t & 0xFFFFu;
                const int j = q;
                if (work && r < sg.rows && j < sg.g) {
                    const uint32_t vsm = st + (r ? prm.st_v1 : prm.st_v0);
                    const uint32_t excl = incl[q] - packed[q];
                    const uint32_t ea = excl & 0xFFFFu, eb = tot_a[q] + (excl >> 16);   // PopCount prefix
                    const uint32_t Aa = vsm + 2u * (uint32_t)(rel + (int)ea);
                    const uint32_t Ab = vsm + 2u * (uint32_t)(rel + (int)eb);
                    const uint32_t te = tb + (uint32_t)(r * G + j) * 1024u + 8u * lane;
                    // entries hold (first value address - 4): the consumers address V[c2 - 2]
                    sts_v2(te, ba[q].x, Aa - 4u);
                    sts_v2(te + 512u, ba[q].y, Aa - 4u + 2u * __popc(ba[q].x));
                    sts_v2(te + 256u, bb[q].x, Ab - 4u);
                    sts_v2(te + 768u, bb[q].y, Ab - 4u + 2u * __popc(bb[q].x));
                }
                rel += (int)(((t & 0xFFFFu) + (t >> 16) + 7u) & ~7u);
            }
            // one arrive per warp: every mbarrier event wakes all sleeping waiters of the CTA,
            // so 64 per-thread arrivals would cost each waiting consumer ~60 extra polls
            __syncwarp();
            if (lane == 0) mbar_arrive(bar_scan + 8 * slot);
            if (lane == 0) trace_ev(prm, p, i, warp, 3);
        }
        if (lane == 0) trace_k(prm, p, warp, 3);
        return;
    }

    // ---------------------------------------------------------------- consumers
    // Lane constants, computed once: this lane's byte offset inside a slot's table (GT row r,
    // TCTile column c, lane-half h) and inside a slot's X slab (ldmatrix row and swizzled chunk),
    // the SMBD shift multiplier, and the warp's (q, r). Everything stage-dependent comes from
    // the stage descriptor (one 16-byte shared load per stage).
    const int q = warp % KQ, c = (warp / KQ) & 3, r = warp / (4 * KQ);
    uint32_t mulc = 1u << (30u - 2u * (uint32_t)(lane & 15));   // w * mulc == w << (30 - sh), sh = 2 (lane % 16)
#if SPINFER_PIPEMIX & 1
    mulc = opaque_u32(mulc);   // hide the power of two: IMAD (FMA pipe) instead of SHF (ALU pipe)
#endif
    const uint32_t four = opaque_u32(4u);
    (void)four;
    constexpr uint32_t cpr = N / 8;
    const uint32_t tbl_lane = (uint32_t)(r * G) * 1024u + (uint32_t)(lane >> 4) * 512u + (uint32_t)c * 128u;
    // ldmatrix.trans rows: matrix m = lane/8 -> (k half m&1, n chunk m>>1); row rr = lane%8.
    const uint32_t rr = lane & 7, mk = (lane >> 3) & 1, mn = (lane >> 4) & 1;
    const uint32_t x_lane = ((mk * 8u + rr) + 16u * (uint32_t)c) * cpr * 16u + ((mn ^ x_swz<NT>(rr)) * 16u);
    // selector polynomial constants, read from smem so ptxas keeps them in registers
    const uint32_t selA = reinterpret_cast<volatile uint32_t *>(smem)[kConstWord];
    const uint32_t selB = reinterpret_cast<volatile uint32_t *>(smem)[kConstWord + 1];
    const uint32_t selC = reinterpret_cast<volatile uint32_t *>(smem)[kConstWord + 2];
    float acc[4][NT][4];
    constexpr uint32_t kPart = 64u * N * 4u;                      // one fp32 64 x N partial

    // Software pipeline over half-GT steps (8 BTs = TCTile rows 2h', 2h'+1 of GT j):
    // while step h is assembled and multiplied, the value loads of step h+1 and the
    // table entries of step h+2 are already in flight. Steps alternate between two
    // register sets (A: first half of a GT, B: second half) so no copies are needed.
    // The pipeline runs continuously across stages: during the last step of stage i the
    // warp already waits for stage i+1 and issues its first loads.
    uint4 E[4];
    uint32_t tA0[8], tA1[8], sA[8], tB0[8], tB1[8], sB[8];
    auto load_E = [&](uint32_t tb, int step) {   // table entries of step `step` (4 x 16 B per lane)
#pragma unroll
        for (int k = 0; k < 4; ++k) E[k] = lds_v4(tb + (uint32_t)(step >> 1) * 1024u + (uint32_t)(step & 1) * 64u + 16u * k);
    };
    auto issue = [&](uint32_t (&t0)[8], uint32_t (&t1)[8], uint32_t (&s1)[8]) {   // value loads from E
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const uint32_t w = (k & 1) ? E[k >> 1].z : E[k >> 1].x;
            const uint32_t A = (k & 1) ? E[k >> 1].w : E[k >> 1].y;   // (first value of the half) - 4 bytes
            // z = w << (30 - sh) as a multiply (FMA pipe): its top two bits are the lane's pair
            // y = (bit sh, bit sh+1) and popc(z) = c2 = MaskedPopCount + b0 + b1 (Alg. 2)
            const uint32_t z = w * mulc;
            const uint32_t a = A + 2u * __popc(z);        // &V[c2 - 2]
            const uint32_t y = z >> 30;
            s1[k] = y * (y * selB + selA) + selC;          // selector polynomial (see kSelA)
            t0[k] = lds_u16(a);                            // V[c2 - 2]
            t1[k] = lds_u16(a + 2u);                       // V[c2 - 1]
        }
    };
    auto assemble = [&](const uint32_t (&t0)[8], const uint32_t (&t1)[8], const uint32_t (&s1)[8], int trb,
                        const uint32_t (&bfr)[NT][2]) {
#pragma unroll
        for (int tt = 0; tt < 2; ++tt) {
            uint32_t afr[4];
#pragma unroll
            for (int b = 0; b < 4; ++b) {
                const int k = tt * 4 + b;
                afr[b] = prmt(t0[k], t1[k], s1[k]);
            }
#pragma unroll
            for (int nt = 0; nt < NT; ++nt) mma_16816(acc[trb + tt][nt], afr, bfr[nt][0], bfr[nt][1]);
        }
    };
    const bool compute = !(dbg_mode(prm) & 1);
    constexpr bool kPipe = (KQ == 1) || SPINFER_PIPE2;          // explicit cross-step software pipeline (8 consumer warps)
    const bool reuse0 = (dbg_mode(prm) & 4) != 0;   // experiment: pure consumer throughput on stage 0's data
    auto load_x = [&](uint32_t xs, int j, uint32_t (&bfr)[NT][2]) {   // B fragments of GT j, TCTile column c
        const uint32_t xk = xs + (uint32_t)(64 * j) * cpr * 16u;     // xs includes this lane's x_lane
        if constexpr (NT == 1) {
            ldsm_x2_trans(xk, bfr[0][0], bfr[0][1]);
        } else {
#pragma unroll
            for (int nt = 0; nt + 1 < NT; nt += 2)     // chunk (nt + mn) ^ swz == (mn ^ swz) ^ nt for even nt
                ldsm_x4_trans(xk ^ ((uint32_t)nt * 16u), bfr[nt][0], bfr[nt][1], bfr[nt + 1][0], bfr[nt + 1][1]);
            if constexpr (NT % 2 == 1)
                ldsm_x2_trans(xk - ((mn ^ x_swz<NT>(rr)) * 16u) + (uint32_t)(NT - 1) * 16u, bfr[NT - 1][0], bfr[NT - 1][1]);
        }
    };
    const uint32_t desc = sbase + prm.o_desc;
    auto rd = [&](int si) {   // volatile shared load: re-read, never kept live across the decode loop
        const uint4 v = lds_v4(desc + 16u * (uint32_t)si);
        return StageDesc{v.x, v.y, v.z, v.w};
    };
    auto begin_stage = [&](const StageDesc &s, int si) {
        if (lane == 0) trace_ev(prm, p, si, warp, 0);
        if (!reuse0 || si == 0) {
            // suspend rather than spin: a spinning consumer steals issue slots from the
            // other 15 consumer warps that still have decode work
#if SPINFER_CONSSPIN
            mbar_wait(bar_scan + 8 * s.slot(), s.par());
#else
            mbar_wait_sleep(bar_scan + 8 * s.slot(), s.par());   // implies full[slot] (see above)
#endif
#if SPINFER_BMBAR
            mbar_wait_sleep(bar_full + 8 * s.slot(), s.par());   // values and X (usually landed already)
#endif
            if (lane == 0) trace_ev(prm, p, si, warp, 1);
        }
        if (kPipe && r < s.rows() && compute && q < s.g()) {
            const uint32_t tb = sbase + s.tbl + tbl_lane;
            load_E(tb, 2 * q);
            issue(tA0, tA1, sA);
            load_E(tb, 2 * q + 1);
        }
    };
    named_bar_sync(kDescBar, 32u * (kCW + 1 + SPINFER_SCANDESC));
    const int nst = (dbg_mode(prm) & 16) ? 0 : (int)reinterpret_cast<volatile uint32_t *>(smem)[kConstWord + 3];
    if (kPipe && nst > 0) begin_stage(rd(0), 0);
    // the next stage's descriptor is fetched during the current stage's decode (a shared load
    // at a stage boundary waits behind the decode traffic in the MIO queue)
    StageDesc dn = rd(0);
    int segi = 0;   // segment ends seen (asynchronous epilogue buffer / phase)
    (void)segi;
    for (int i = 0; i < nst; ++i) {
        const int cw = warp;
        const StageDesc d = dn;
        {
            if (d.zero()) {
#pragma unroll
                for (int a = 0; a < 4; ++a)
#pragma unroll
                    for (int b = 0; b < NT; ++b)
#pragma unroll
                        for (int e = 0; e < 4; ++e) acc[a][b][e] = 0.f;
            }
            if constexpr (!kPipe) begin_stage(d, i);
        }
        if (i + 1 < nst) dn = rd(i + 1);
        const int g = d.g();
        if (d.rows() > r && compute && q < g && !kPipe) {
            // KQ = 2: 4 consumer warps per scheduler hide the latencies; one register set.
            const uint32_t xs = sbase + d.stg + x_lane;
            const uint32_t tb = sbase + d.tbl + tbl_lane;
#if SPINFER_EPREF
            // the next step's table entries are loaded as soon as the current step has consumed
            // E (issue), so their latency hides behind the current step's assembly and MMAs
            load_E(tb, 2 * q);
            for (int j = q; j < g; j += KQ) {
                uint32_t bfr[NT][2];
                load_x(xs, j, bfr);
                issue(tA0, tA1, sA);
                load_E(tb, 2 * j + 1);
                assemble(tA0, tA1, sA, 0, bfr);
                issue(tA0, tA1, sA);
                if (j + KQ < g) load_E(tb, 2 * (j + KQ));
                assemble(tA0, tA1, sA, 2, bfr);
            }
#else
            for (int j = q; j < g; j += KQ) {
                uint32_t bfr[NT][2];
                load_x(xs, j, bfr);
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    load_E(tb, 2 * j + h);
                    issue(tA0, tA1, sA);
                    assemble(tA0, tA1, sA, 2 * h, bfr);
                }
            }
#endif
        } else if (d.rows() > r && compute && q < g) {
            const uint32_t xs = sbase + d.stg + x_lane;
            const uint32_t tb = sbase + d.tbl + tbl_lane;
            for (int j = q; j < g; j += KQ) {
                uint32_t bfr[NT][2];
                load_x(xs, j, bfr);
                // step (j, first half): issue (j, second half) into B, prefetch the entries of
                // this warp's next GT, assemble (j, first half) from A
                issue(tB0, tB1, sB);
                if (j + KQ < g) load_E(tb, 2 * (j + KQ));
                assemble(tA0, tA1, sA, 0, bfr);
                // step (j, second half): issue the next step (A: next GT, or the next stage's first step)
                if (j + KQ < g) {
                    issue(tA0, tA1, sA);
                    load_E(tb, 2 * (j + KQ) + 1);
                } else if (i + 1 < nst) {
                    begin_stage(rd(i + 1), i + 1);
                }
                assemble(tB0, tB1, sB, 2, bfr);
            }
        } else if (kPipe && i + 1 < nst) {
            begin_stage(rd(i + 1), i + 1);
        }
        if (lane == 0) trace_ev(prm, p, i, cw, 2);   // decode done
        const StageDesc e = d;
        const int rb = e.rb(), rows = e.rows();
#if SPINFER_AEPI
        if (e.seg_end() && i + 1 < nst) {
            // asynchronous epilogue (not the CTA's last segment): park this warp's partial, move on
            const uint32_t buf = (uint32_t)segi & 1u, use = (uint32_t)segi >> 1;
            ++segi;
            if (r < rows && !(dbg_mode(prm) & 8)) {
                if (use > 0) mbar_wait_sleep(bar_epifree + 8u * buf, (use - 1u) & 1u);
                float4 *dst = reinterpret_cast<float4 *>(prm.ws_epi) +
                              ((((size_t)p * 2 + buf) * kR + r) * 8 + (size_t)(c * KQ + q)) * (64 * N / 4);
#pragma unroll
                for (int tr = 0; tr < 4; ++tr)
#pragma unroll
                    for (int nt = 0; nt < NT; ++nt)
                        dst[(tr * NT + nt) * 32 + lane] = make_float4(acc[tr][nt][0], acc[tr][nt][1], acc[tr][nt][2], acc[tr][nt][3]);
                __syncwarp();
                if (lane == 0) mbar_arrive(bar_epi + 8u * (buf * kR + (uint32_t)r));   // release: the stores above
            }
        } else
#endif
        if (e.seg_end() && r < rows && !(dbg_mode(prm) & 8)) {   // experiment bit 8: no epilogue
            // -------------------------------------------------------- epilogue
            // (1) reduce the 4*KQ partials of GT row r into warp (c = 0, q = 0), tree via smem.
            // Scratch = this stage's value region of GT row r: only row r's consumer warps read
            // it, so once they all pass the first barrier it is free (the slot is released below).
            const uint32_t bid = 1u + (uint32_t)r, bcnt = 128u * KQ;
            const uint32_t scr = sbase + e.stg + (r ? prm.st_v1 : prm.st_v0);
            named_bar_sync(bid, bcnt);
            auto put = [&](uint32_t slot_) {
#pragma unroll
                for (int tr = 0; tr < 4; ++tr)
#pragma unroll
                    for (int nt = 0; nt < NT; ++nt)
                        sts_f4(scr + slot_ * kPart + (uint32_t)((tr * NT + nt) * 32 + lane) * 16u,
                               make_float4(acc[tr][nt][0], acc[tr][nt][1], acc[tr][nt][2], acc[tr][nt][3]));
            };
            auto add = [&](uint32_t slot_) {
#pragma unroll
                for (int tr = 0; tr < 4; ++tr)
#pragma unroll
                    for (int nt = 0; nt < NT; ++nt) {
                        float4 v = lds_f4(scr + slot_ * kPart + (uint32_t)((tr * NT + nt) * 32 + lane) * 16u);
                        acc[tr][nt][0] += v.x; acc[tr][nt][1] += v.y; acc[tr][nt][2] += v.z; acc[tr][nt][3] += v.w;
                    }
            };
            if constexpr (KQ == 2) {          // GT parities: q = 1 -> q = 0
                if (q == 1) put((uint32_t)c);
                named_bar_sync(bid, bcnt);
                if (q == 0) add((uint32_t)c);
                named_bar_sync(bid, bcnt);
            }
            if (q == 0 && c >= 2) put((uint32_t)(c - 2));     // TCTile columns: 4 -> 2 -> 1
            named_bar_sync(bid, bcnt);
            if (q == 0 && c < 2) add((uint32_t)c);
            named_bar_sync(bid, bcnt);
            if (q == 0 && c == 1) put(0u);
            named_bar_sync(bid, bcnt);
            if (q == 0 && c == 0) add(0u);
            named_bar_sync(bid, bcnt);
            // (2) write Y, or combine split rowblocks across CTAs (split-K fix-up)
            if (c == 0 && q == 0) {
                const int grow = kR * rb + r;
                const int row_base = grow * 64;
                if (e.complete()) {
                    store_y<NT, EPI>(prm, row_base, acc, lane);
                } else {
                    // split rowblock (split-K fix-up, the paper's ReductionWorkspace P:231): park the
                    // fp32 partial; the fix-up warp counts it and the last contributor sums all
                    // partials in CTA order (deterministic), writes Y and re-zeroes the counter.
                    // Split segments are a CTA's first stages (StageIter order), so the fix-up
                    // latency hides behind the full rowblocks.
                    const int myslot = (rb == u0 / KG) ? 0 : 1;
                    float4 *part = reinterpret_cast<float4 *>(prm.ws_part) + (((size_t)p * 2 + myslot) * kR + r) * (64 * N / 4);
#pragma unroll
                    for (int tr = 0; tr < 4; ++tr)
#pragma unroll
                        for (int nt = 0; nt < NT; ++nt)
                            part[(tr * NT + nt) * 32 + lane] =
                                make_float4(acc[tr][nt][0], acc[tr][nt][1], acc[tr][nt][2], acc[tr][nt][3]);
                    // hand the rest (fence, count, last-contributor sum) to the fix-up warp
                    mbar_arrive(bar_fix + 8u * (uint32_t)(2 * myslot + r));
                }
            }
        }
        __syncwarp();
        if (lane == 0 && !reuse0) {
#if SPINFER_RELCNT
            // acq_rel: this warp's reads of the slot happen-before the count; the last warp's
            // acquire makes all of them happen-before its arrive (release) and the refill
            const uint32_t old = atom_add_acqrel_shared(rel_cnt + 4u * (uint32_t)e.slot(), 1u);
            if (old % (uint32_t)kCW == (uint32_t)kCW - 1u) mbar_arrive(bar_empty + 8 * e.slot());
#else
            mbar_arrive(bar_empty + 8 * e.slot());   // frees the ring slot and its table
#endif
            trace_ev(prm, p, i, cw, 3);
        }
    }

    if (lane == 0) trace_k(prm, p, warp, 2);
    if (lane == 0) trace_k(prm, p, warp, 3);
}

// ================================================================ tcgen05 path
// Same stream-K stage sequence as k_spmm; what changes is the data path and who multiplies:
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
    static constexpr int ScanWarp = 17;      // 17, 18: SMBD tables of even / odd stages
    static constexpr int Threads = 19 * 32;  // <= 5 warps per SM sub-partition: 96 registers each
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
// k-team MMA issue by the last of the team's 4 lane-quarter warps to finish its A tiles (a shared
// atomic count per A buffer) instead of a named barrier of the 4 warps: no warp waits for another
#ifndef SPINFER_TC_SCANFULL
#define SPINFER_TC_SCANFULL 1
#endif
#ifndef SPINFER_TC_WARPFIX
#define SPINFER_TC_WARPFIX 1
#endif
#ifndef SPINFER_TC_AFULL
#define SPINFER_TC_AFULL 0
#endif
#ifndef SPINFER_TC_LAST
#define SPINFER_TC_LAST 0
#endif
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

    if (lane == 0) trace_k(prm, p, warp, 0);
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(bar_full + 8 * s, 1);
            mbar_init(bar_empty + 8 * s, kCW);             // every decode warp
            mbar_init(bar_emptyx + 8 * s, 4);              // the 4 k-teams' MMA commits
            mbar_init(bar_scan + 8 * s, 1);                // the stage's scan warp
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
    const uint32_t tmem = *reinterpret_cast<volatile uint32_t *>(smem + kTcTmemSlot);
    if (lane == 0) trace_k(prm, p, warp, 1);
    if (u0 >= u1 || (dbg_mode(prm) & 16)) {   // no work (more CTAs than units); experiment bit 16: launch only
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
        // split-K fix-up, served by this warp while it waits for free slots: at most two split
        // rowblocks per CTA (A: the tail of the rowblock it starts inside, C: the head of the one
        // it ends inside). The finishing k-team parks this CTA's fp32 partial and arrives on
        // fix[A/C]; this warp counts it and, as the last contributor, sums all partials in CTA
        // order (deterministic), writes Y and re-zeroes the counter (ReductionWorkspace).
        const int N = prm.N;
    const int Nw = (N + 7) & ~7;   // partial row stride (X was padded to a multiple of 8)
        const int a_rb = u0 / KG, c_rb = (u1 - 1) / KG;
        const bool has_a = (u0 % KG) != 0;
        const bool has_c = (u1 % KG) != 0 && !(has_a && c_rb == a_rb);
        int fx = has_a ? 0 : (has_c ? 1 : 2);   // next split segment to serve (2: none left)
        if (SPINFER_TC_WARPFIX) fx = 2;          // the epilogue warps do the fix-up themselves
        auto fixup = [&](int sgi) {
            const int rb = sgi == 0 ? a_rb : c_rb;
            const int rows = min(kR, prm.MG - kR * rb);
            __threadfence();   // cumulative: the team's partial stores before the count
            const int pf = unit_owner(rb * KG, U, prm.P);
            const int pl = unit_owner((rb + 1) * KG - 1, U, prm.P);
            int old = 0;
            if (lane == 0) old = atomicAdd(prm.ws_cnt + rb, 1);
            old = __shfl_sync(0xffffffffu, old, 0);
            if (old != pl - pf) return;
            __threadfence();
            for (int row_in = lane; row_in < 64 * rows; row_in += 32) {
                float v[NB];
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
            if (lane == 0) prm.ws_cnt[rb] = 0;   // leave the workspace zeroed
        };
        auto next_fx = [&]() { fx = (fx == 0 && has_c) ? 1 : 2; };
        StageIter pit;
        pit.init(u0, u1, prm);
        poff = load_off(pit);
        for (; pit.valid();) {
            const StageIter sg = pit;
            const int i = sg.i, slot = sg.slot;
            if (lane == 0) trace_ev(prm, p, i, warp, 0);
            if (i >= S) {
                while (true) {
                    if (fx < 2 && mbar_test_wait(sbase + kTcFix + 8u * (uint32_t)fx, 0u)) {
                        fixup(fx);
                        next_fx();
                        continue;
                    }
                    if (mbar_try_wait_sleep(bar_empty + 8 * slot, sg.par() ^ 1u)) break;
                }
            }
            const uint32_t st = sbase + prm.o_stage + slot * prm.stage_bytes;
            const uint32_t vb = 2u * (uint32_t)(poff.y - poff.x);   // lanes 0, 1: value bytes of their GT row
            const uint32_t vtot = __shfl_sync(0xffffffffu, vb, 0) + __shfl_sync(0xffffffffu, vb, 1);
            if (lane == 0) mbar_arrive_expect_tx(bar_full + 8 * slot, (uint32_t)G * xbytes + vtot);
            __syncwarp();
            if (lane < sg.rows && vb)
                bulk_g2s(st + (lane ? prm.st_v1 : prm.st_v0), prm.vals + poff.x, vb, bar_full + 8 * slot, pol_w);
            // the X slab region is free once the MMA of stage i - S has completed
            if (i >= S) mbar_wait(bar_emptyx + 8 * slot, sg.par() ^ 1u);
            if (lane == 0) tma_2d_g2s(st, &prm.tmap_x, 0, 64 * sg.gc, bar_full + 8 * slot);   // box {NB, 64 G}
            if (lane == 0) trace_ev(prm, p, i, warp, 1);
            pit.next(prm);
            if (pit.valid()) poff = load_off(pit);
        }
        while (fx < 2) {
            mbar_wait_backoff(sbase + kTcFix + 8u * (uint32_t)fx, 0u, 128u, 1024u);
            fixup(fx);
            next_fx();
        }
        if (lane == 0) trace_k(prm, p, warp, 3);
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
        // MIO queue) is hidden; two warps double the throughput.
        constexpr int Q = 2 * kMaxG;
        const int sw = warp - CfgTC::ScanWarp;
        struct Bm { uint2 a[Q], b[Q]; int o[kR]; };
        auto fetch = [&](const StageIter &sg, Bm &f) {
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
        if (sw == 1) it.next(prm);
        auto skip2 = [&](StageIter &x) { x.next(prm); if (x.valid()) x.next(prm); };
        Bm F;   // one register set: the next stage's loads are issued right after a table is
                // published and complete while the warp waits for that stage's slot
        if (it.valid()) fetch(it, F);
        auto one = [&](Bm &cur) -> bool {
            if (!it.valid()) return false;
            const StageIter sg = it;
            const int slot = sg.slot;
            if (lane == 0) trace_ev(prm, p, sg.i, warp, 0);
            if (sg.i >= S) mbar_wait_sleep(bar_empty + 8 * slot, sg.par() ^ 1u);   // the slot's table is free
            if (lane == 0) trace_ev(prm, p, sg.i, warp, 1);
            const uint32_t st = sbase + prm.o_stage + slot * prm.stage_bytes;
            const uint32_t tb = sbase + prm.o_tbl + slot * prm.tbl_bytes;
            if (dbg_mode(prm) & 2) {   // experiment: no table build
                __syncwarp();
                if (lane == 0) mbar_arrive(bar_scan + 8 * slot);
                skip2(it);
                if (it.valid()) fetch(it, cur);
                return true;
            }
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
            __syncwarp();
#if SPINFER_TC_SCANFULL
            // publish the table only once the slot's values and X have landed too, so the decode
            // warps wait on one barrier per stage
            mbar_wait_sleep(bar_full + 8 * slot, sg.par());
#endif
            if (lane == 0) mbar_arrive(bar_scan + 8 * slot);
            if (lane == 0) trace_ev(prm, p, sg.i, warp, 3);
            skip2(it);
            if (it.valid()) fetch(it, cur);   // this warp's next stage
            return true;
        };
        while (one(F)) {
        }
        if (lane == 0) trace_k(prm, p, warp, 3);
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
        // split rowblock: park this CTA's fp32 partial; the producer warp does the fix-up
        const int myslot = (rb == u0 / KG) ? 0 : 1;
        if (valid) {
            float4 *pp = reinterpret_cast<float4 *>(prm.ws_part + (((size_t)p * 2 + myslot) * 128 + row_in) * Nw);
#pragma unroll
            for (int c4 = 0; c4 < NB / 4; ++c4)
                if (c4 * 4 < Nw) pp[c4] = make_float4(v[4 * c4], v[4 * c4 + 1], v[4 * c4 + 2], v[4 * c4 + 3]);
        }
#if SPINFER_TC_WARPFIX
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
#else
        __threadfence();
        __syncwarp();
        const bool is_a = (u0 % KG) != 0 && rb == u0 / KG;
        if (lane == 0) mbar_arrive(sbase + kTcFix + (is_a ? 0u : 8u));
#endif
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
        if (lane == 0) trace_ev(prm, p, i, warp, 0);
        const bool reuse0 = (dbg_mode(prm) & 4) != 0;   // experiment: stage 0's data for every stage
        if (!reuse0 || i == 0) {
            mbar_wait_sleep(bar_scan + 8 * slot, d.par());   // table written (the scan runs ahead)
#if !SPINFER_TC_SCANFULL
            mbar_wait_sleep(bar_full + 8 * slot, d.par());   // values and X landed
#endif
        }
        if (lane == 0) trace_ev(prm, p, i, warp, 1);
        const uint32_t ab = (uint32_t)(kt * ABufs) + ar.b;
        if (i >= ABufs) mbar_wait(bar_ae + 8u * ab, ar.ph ^ 1u);
        tm_fence_after();
        if (r < d.rows() && kt < d.g() && !(dbg_mode(prm) & 1)) {
            const uint32_t tb = sbase + prm.o_tbl + (uint32_t)(reuse0 ? 0 : slot) * prm.tbl_bytes +
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
        if (lane == 0) mbar_arrive(bar_empty + 8 * slot);   // this warp is done with the slot's values/table
        const bool mm = kt < d.g();
#if SPINFER_TC_LAST
        // the last of the team's 4 lane-quarter warps to finish its A tiles multiplies
        bool issuer = false;
        {
            int old = 0;
            if (lane == 0) {
                __threadfence_block();   // release: this warp's TMEM stores (fenced above) before the count
                old = atomicAdd(reinterpret_cast<int *>(smem + kTcTeamCnt) + ab, 1);
                __threadfence_block();   // acquire: the other warps' stores before the MMA
            }
            issuer = (__shfl_sync(0xffffffffu, old, 0) & 3) == 3;
        }
#elif SPINFER_TC_AFULL
        // the team's 4 lane-quarter warps arrive on the A buffer's mbarrier (release: their TMEM
        // stores, fenced above); only the team leader waits for it and multiplies — the other
        // three go on to the next stage
        if (lane == 0) mbar_arrive(sbase + kTcAFull + 8u * ab);
        const bool issuer = (q == 0);
        if (issuer) mbar_wait(sbase + kTcAFull + 8u * ab, ar.ph);
#else
        // the team's 4 lane-quarter warps have written their A tiles: the team leader multiplies
        named_bar_sync(kTeamBar + (uint32_t)kt, 128);
        const bool issuer = (q == 0);
#endif
        if (issuer) {
            tm_fence_after();
            if (sf.zero && seg >= 2) {   // the D buffer's previous segment has been read out
                mbar_wait(bar_de + 8u * dpar, dph ^ 1u);
                tm_fence_after();
            }
            const uint32_t d_t = tmem + DCol + ((uint32_t)kt * 2u + dpar) * NB;
            const uint32_t a_t = tmem + ab * 32u;
            const uint32_t x_lo = (sbase + prm.o_stage + (uint32_t)(reuse0 ? 0 : slot) * prm.stage_bytes) >> 4;
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
        if (lane == 0) trace_ev(prm, p, i, warp, 2);
        if (pend) {
            epilogue(pend_db, pend_dph, pend_rb, pend_rows, pend_complete, pend_nt);
            pend = false;
        }
        if (sf.seg_end && (seg & 3) == kt) {
            pend = true;
            pend_db = dpar; pend_dph = dph; pend_rb = d.rb(); pend_rows = d.rows(); pend_complete = sf.complete;
            pend_nt = min(maxg, 4);
        }
        if (lane == 0) trace_ev(prm, p, i, warp, 3);
    }
    if (pend) epilogue(pend_db, pend_dph, pend_rb, pend_rows, pend_complete, pend_nt);
    tm_fence_before();
    named_bar_sync(kEndBar, 32u * kCW);   // every MMA has completed (the last epilogues waited on them)
    tm_fence_after();
    if (warp == 0) tm_dealloc(tmem, CfgTC::TmemCols);
    if (lane == 0) trace_k(prm, p, warp, 3);
}

// X [K][N] -> Xp [K][Np] with zero columns N..Np-1 (N not a multiple of 8)
__global__ void k_pad_x(const uint16_t *__restrict__ X, uint16_t *__restrict__ Xp, int K, int N, int Np) {
    const long long tot = (long long)K * Np;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < tot; i += (long long)gridDim.x * blockDim.x) {
        const int k = (int)(i / Np), n = (int)(i - (long long)k * Np);
        Xp[i] = n < N ? X[(size_t)k * N + n] : (uint16_t)0;
    }
}
inline size_t align_up_sz(size_t v, size_t a) { return (v + a - 1) / a * a; }

struct Plan {
    int P, G, S;
    long long U;
    size_t smem;
    Params prm;
};

int num_sms() {
    int dev = 0, n = kNumSMsDefault;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    cudaGetLastError();
    return n > 0 ? n : kNumSMsDefault;
}

int choose_P(long long U) {
    long long cap = num_sms();
    // SPINFER_MAX_CTAS caps the persistent grid (tests use it to force many stages per CTA)
    if (const char *e = getenv("SPINFER_MAX_CTAS")) { long long v = atoll(e); if (v > 0 && v < cap) cap = v; }
    long long P = std::min(cap, U);
    // keep the per-CTA stage descriptors (<= 16 B per unit) within a few KiB of shared memory
    while ((U + P - 1) / P > 1024) P += num_sms();
    return (int)std::max(1LL, P);
}

inline uint32_t align_up(uint32_t x, uint32_t a) { return (x + a - 1) / a * a; }

// cuTensorMapEncodeTiled through the runtime's driver entry point (no libcuda link).
using EncodeTiledFn = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                   const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int encode_x_map(CUtensorMap *m, const uint16_t *X, int K, int N, int NX, int box_rows, bool swizzle = true) {
    static EncodeTiledFn fn = nullptr;
    if (!fn) {
        void *f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess || !f) {
            cudaGetLastError();
            return SPINFER_ECUDA;
        }
        fn = reinterpret_cast<EncodeTiledFn>(f);
    }
    const cuuint64_t dims[2] = {(cuuint64_t)N, (cuuint64_t)K};
    const cuuint64_t strides[1] = {(cuuint64_t)N * 2};
    // box {NX, 64}: NX > N (tcgen05 path, N = 8 / 24) reads past the tensor's columns, which the
    // TMA fills with zeros (X padded to the MMA's N = 16 / 32 without a copy)
    const cuuint32_t box[2] = {(cuuint32_t)NX, (cuuint32_t)box_rows};
    const cuuint32_t estr[2] = {1u, 1u};
    const CUtensorMapSwizzle sw = !swizzle ? CU_TENSOR_MAP_SWIZZLE_NONE
                                  : NX == 16 ? CU_TENSOR_MAP_SWIZZLE_32B : NX == 32 ? CU_TENSOR_MAP_SWIZZLE_64B
                                                                                 : CU_TENSOR_MAP_SWIZZLE_NONE;
    CUresult r = fn(m, CU_TENSOR_MAP_DATA_TYPE_UINT16, 2, const_cast<uint16_t *>(X), dims, strides, box, estr,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? SPINFER_OK : SPINFER_EINVAL;
}

bool make_plan(int M, int K, int N, int max_gt_values, Plan *pl, bool tc) {
    const int MG = (M + kGT - 1) / kGT, KG = (K + kGT - 1) / kGT;   // zero-padded to whole GTs (A8)
    const int nRB = (MG + kR - 1) / kR;
    const long long U = (long long)nRB * KG;
    pl->P = choose_P(U);
    if ((unsigned long long)U * (unsigned long long)pl->P >= (1ull << 32)) return false;   // 32-bit unit math
    pl->U = U;
    const long long upc = (U + pl->P - 1) / pl->P;
    int dev = 0, smem_max = 232448;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&smem_max, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    cudaGetLastError();
    int maxv = max_gt_values > 0 ? max_gt_values : 4096;
    maxv = std::min(4096, (maxv + 7) & ~7);
    const uint32_t o_desc = 1024;
    const int NX = tc ? (N <= 16 ? 16 : 32) : N;   // X slab columns
    int gmax = kMaxG, smax = kMaxStages;
    if (const char *e = getenv("SPINFER_G")) gmax = std::max(1, std::min(kMaxG, atoi(e)));
    if (const char *e = getenv("SPINFER_S")) smax = std::max(2, std::min(kMaxStages, atoi(e)));
    for (int G = gmax; G >= 1; --G) {
        uint32_t tbl = (uint32_t)kR * G * 64 * 16;
        const uint32_t scr_row = tc ? 0u : (uint32_t)(N <= 16 ? 4 : 2) * 64 * N * 4;   // k_spmm: epilogue scratch per GT row
        uint32_t st_bm = (uint32_t)G * 64 * NX * 2;           // X slab first, then bitmaps
        uint32_t st_v0 = st_bm + (tc ? 0u : (uint32_t)kR * G * 512);   // tcgen05 path: bitmaps go to registers
        uint32_t vcap = align_up(std::max((uint32_t)G * maxv * 2, scr_row), 16);   // also the epilogue scratch
        uint32_t st_v1 = st_v0 + vcap;
        uint32_t stage = align_up(st_v1 + vcap, 1024);   // slots stay 1024-aligned (X swizzle)
        // stage descriptors: at most one per unit, and no more than ceil(units/G) + rowblock splits
        const uint32_t desc_bytes = align_up((uint32_t)(16 * std::min<long long>(upc, upc / G + upc / KG + 3)), 128);
        uint32_t fixed = o_desc + desc_bytes + 128 + 2048;   // +slack: t1 over-read, base and ring alignment
        if (tc) fixed = 1024 + align_up(desc_bytes, 1024) + 128 + 1024;   // tcgen05 path: descriptors (tables 1024-aligned)
        stage += tbl;                                     // k_spmm: each ring slot carries its table
        if ((long long)fixed + 2LL * stage > smem_max) continue;
        int S = (int)std::min<long long>(smax, ((long long)smem_max - fixed) / stage);
        if (S < 3 && G > 1) continue;
        pl->G = G;
        pl->S = S;
        Params &q = pl->prm;
        q.KG = KG; q.MG = MG; q.U = (uint32_t)U; q.P = pl->P; q.G = G; q.S = S;
        stage -= tbl;
        q.stage_bytes = stage; q.st_bm = st_bm; q.st_v0 = st_v0; q.st_v1 = st_v1;
        q.tbl_bytes = tbl;
        q.o_desc = o_desc;
        q.o_tbl = q.o_desc + desc_bytes;
        if (tc) q.o_tbl = q.o_desc + align_up(desc_bytes, 1024);
        q.o_stage = align_up(q.o_tbl + (uint32_t)S * tbl, 1024);
        pl->smem = (size_t)q.o_stage + (size_t)S * stage + 128 + 1024;   // +1024: runtime base alignment
        return true;
    }
    return false;
}

template <int NT, bool EPI>
int launch_nt(const Plan &pl, cudaStream_t st) {
    static int configured_smem[64] = {0};   // per device: max dynamic smem already set for this instantiation
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    if ((int)pl.smem > configured_smem[dev]) {
        if (cudaFuncSetAttribute(k_spmm<NT, EPI>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)pl.smem) != cudaSuccess)
            return SPINFER_ECUDA;
        configured_smem[dev] = (int)pl.smem;
    }
    k_spmm<NT, EPI><<<pl.P, Cfg<NT>::Threads, pl.smem, st>>>(pl.prm);
    return cudaGetLastError() == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
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
    k_spmm_tc<NB><<<pl.P, CfgTC::Threads, pl.smem, st>>>(pl.prm);
    return cudaGetLastError() == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
}

}  // namespace

int sm_count() {
    static int cached[64] = {0};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) { cudaGetLastError(); return num_sms(); }
    if (!cached[dev]) cached[dev] = num_sms();
    return cached[dev];
}
int choose_grid(long long units) {
    long long cap = sm_count();
    if (const char *e = getenv("SPINFER_MAX_CTAS")) { long long v = atoll(e); if (v > 0 && v < cap) cap = v; }
    return (int)std::max(1LL, std::min(cap, units));
}
int make_x_tmap(CUtensorMap *m, const uint16_t *X, int K, int N, int NX, int box_rows, bool swizzle) {
    return encode_x_map(m, X, K, N, NX, box_rows, swizzle);
}
int launch_pad_x(const uint16_t *X, uint16_t *Xp, int K, int N, int Np, cudaStream_t st) {
    const long long tot = (long long)K * Np;
    k_pad_x<<<(int)std::min<long long>((tot + 255) / 256, 4096), 256, 0, st>>>(X, Xp, K, N, Np);
    return cudaGetLastError() == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
}

size_t spmm_workspace_bytes(int M, int K, int N) {
    if (M <= 0 || K <= 0 || N <= 0 || N > 32 || (M + kGT - 1) / kGT >= kErrWord) return 0;
    const int MG = (M + kGT - 1) / kGT, KG = (K + kGT - 1) / kGT;
    const long long U = (long long)((MG + kR - 1) / kR) * KG;
    const int P = choose_P(U);
    const int Np = (N + 7) & ~7;   // computed columns (X zero-padded to a multiple of 8)
    size_t part = (size_t)P * 2 * kR * 64 * Np * 4;
    size_t epi = SPINFER_AEPI ? (size_t)P * 2 * kR * 8 * 64 * Np * 4 : 0;   // asynchronous epilogue partials
    size_t xpad = (N % 8) ? align_up_sz((size_t)K * Np * 2, 256) : 0;      // zero-padded copy of X
    const size_t old = kCounterBytes + part + epi + xpad;
    return std::max(old, N <= 16 ? spmm_dw_workspace_bytes(M, K, N) : (size_t)0);
}

int launch_spmm(const spinfer_tca *T, const uint16_t *X, uint16_t *Y, int M, int K, int N, const uint16_t *bias, int act,
                void *ws, size_t ws_bytes, cudaStream_t st) {
    Plan pl;
    // Kernel choice by N, from the B200 measurements: the mma.sync kernel for
    // N <= 16, the tcgen05 kernel (accumulators in TMEM) for N >= 24, where mma.sync needs twice
    // the HMMAs and accumulator registers (config 2 shape, mean us: N=24 114.9 vs 112.1, N=32
    // 126.8 vs 111.0). SPINFER_KERNEL=mma|tc overrides (tests and experiments).
    // N not a multiple of 8: the kernels compute Np = roundup(N, 8) columns from a zero-padded
    // copy of X in the workspace (k_pad_x) and store only the N real columns of Y
    const int Np = (N + 7) & ~7;
    const char *ke = getenv("SPINFER_KERNEL");
    // N <= 16: the decoupled-warp kernel (spmm_dw.cu); SPINFER_KERNEL=mma keeps the round-1 kernel
    if (Np <= 16 && !(ke && (ke[0] == 't' || ke[0] == 'm')))   // SPINFER_KERNEL=dw or unset
        return launch_spmm_dw(T, X, Y, M, K, N, bias, act, ws, ws_bytes, st);
    bool tc = Np >= 24;
    if (ke && ke[0] == 't') tc = true;
    if (ke && ke[0] == 'm') tc = false;
    // the tcgen05 kernel's fix-up keeps one counter per rowblock and TMEM lane quarter
    if (tc && 4LL * (((M + kGT - 1) / kGT + kR - 1) / kR) >= kErrWord) tc = false;
    if (!make_plan(M, K, Np, T->max_gt_values, &pl, tc)) return SPINFER_EINVAL;
    const size_t need = spmm_workspace_bytes(M, K, N);
    if (need == 0) return SPINFER_EINVAL;
    if (ws_bytes < need || ws == nullptr) return SPINFER_ENOSPC;
    Params &q = pl.prm;
    const uint16_t *Xk = X;
    if (N % 8) {
        uint16_t *Xp = reinterpret_cast<uint16_t *>(reinterpret_cast<uint8_t *>(ws) + kCounterBytes +
                                                    (size_t)pl.P * 2 * kR * 64 * Np * 4 +
                                                    (SPINFER_AEPI ? (size_t)pl.P * 2 * kR * 8 * 64 * Np * 4 : 0));
        const long long tot = (long long)K * Np;
        k_pad_x<<<(int)std::min<long long>((tot + 255) / 256, 4096), 256, 0, st>>>(X, Xp, K, N, Np);
        Xk = Xp;
    }
    if (int rc = encode_x_map(&q.tmap_x, Xk, K, Np, tc ? (Np <= 16 ? 16 : 32) : Np, 64 * pl.G)) return rc;
    q.N = N;
    q.off = T->gtile_offset;
    q.bm = T->bitmap;
    q.vals = T->values;
    q.X = Xk;
    q.Y = Y;
    q.bias = bias;
    q.act = act;
    // the general store path (fused bias / activation, padding rows of a ragged M) is a separate
    // instantiation, so the plain aligned path carries none of it
    const bool epi = bias != nullptr || act != SPINFER_ACT_NONE || (M % kGT) != 0;
    q.ws_cnt = reinterpret_cast<int32_t *>(ws);
    q.ws_part = reinterpret_cast<float *>(reinterpret_cast<uint8_t *>(ws) + kCounterBytes);
    q.ws_epi = q.ws_part + (size_t)pl.P * 2 * kR * 64 * Np;
    q.avg_gt = (float)((double)T->n_values / ((double)q.MG * (double)q.KG));
    q.M = M;
    q.dbg = 0;
    if (const char *e = getenv("SPINFER_DEBUG_MODE")) q.dbg = atoi(e);
    q.trace = nullptr;
    static long long *trace_buf = nullptr;
    const char *trace_path = getenv("SPINFER_TRACE");
    const size_t trace_n = kTraceBase2 + 3 * kTraceMaxCTAs;
    if (trace_path) {
        if (!trace_buf && cudaMalloc(&trace_buf, trace_n * 8) != cudaSuccess) return SPINFER_ECUDA;
        cudaMemsetAsync(trace_buf, 0, trace_n * 8, st);
        q.trace = trace_buf;
    }
    int rc = SPINFER_EINVAL;
    if (tc) {
        rc = Np <= 16 ? launch_tc<16>(pl, st) : launch_tc<32>(pl, st);
    } else switch (Np) {
        case 8: rc = epi ? launch_nt<1, true>(pl, st) : launch_nt<1, false>(pl, st); break;
        case 16: rc = epi ? launch_nt<2, true>(pl, st) : launch_nt<2, false>(pl, st); break;
        case 24: rc = epi ? launch_nt<3, true>(pl, st) : launch_nt<3, false>(pl, st); break;
        case 32: rc = epi ? launch_nt<4, true>(pl, st) : launch_nt<4, false>(pl, st); break;
        default: break;
    }
    if (trace_path && rc == SPINFER_OK) {   // debug only: synchronous dump of the stage timeline
        static long long host[kTraceBase2 + 3 * kTraceMaxCTAs];
        cudaMemcpyAsync(host, trace_buf, sizeof(host), cudaMemcpyDeviceToHost, st);
        cudaStreamSynchronize(st);
        if (FILE *f = fopen(trace_path, "wb")) { fwrite(host, 1, sizeof(host), f); fclose(f); }
    }
    return rc;
}

}  // namespace spinfer
