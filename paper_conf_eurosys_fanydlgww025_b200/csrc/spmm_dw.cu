// spmm_dw.cu — decoupled-warp TCA-BME SpMM Y = W x X for N <= 16 (sm_100a; §4.3,
// P:214-301). The library's kernel for N <= 16 (the decode regime of the paper's Fig. 1 shape).
//
// Design: one persistent CTA per SM walks its stream-K range of units (one GT
// column of a 128-row rowblock) in stages of G GroupTile columns x 2 GT rows, through an S-slot
// shared-memory ring; every warp role walks the stage sequence on its own (no lockstep):
//   * 2 producer warps (stages of one parity each): one warp instruction per stage issues the
//     bulk copies of both rows' bitmaps and packed values and the X slab's tensor copy from
//     different lanes (a thread's successive bulk copies serialise at ~310 ns each); a per-slot
//     header carries the stage shape, its segment index and the per-GT value offsets (GTileOffset,
//     P:196). A slot is refilled after a hardware named barrier with exactly the stage's GT owners.
//   * 16 consumer warps: warp (r, m) owns GT m % G of GT row r in the stages i = m / G (mod 8 / G).
//     Per GroupTile it computes the PopCount base of every BitmapTile with a 32-lane
//     shuffle scan into its own 1 KB table, then decodes the 16 TCTiles (MaskedPopCount, Alg. 2
//     P:282-287) into mma.m16n8k16 A fragments (X via ldmatrix.trans, fp32 accumulators in
//     registers, Listing 1).
//   * segment ends (the end of the CTA's part of a rowblock, the paper's ReductionWorkspace P:231,
//     P:263): a consumer parks its fp32 partial in the workspace and signals the reducer warp,
//     which sums the row's partials in warp order and writes Y (complete rowblock) or the CTA's
//     partial; the last CTA of a split rowblock sums the CTA partials in CTA order (8 warps per GT
//     row, in the consumers' end phase). The CTA's final segment is reduced by the 16 consumers
//     together through shared memory. Every sum runs in a fixed order: results do not depend on
//     timing.
// Corrupt or stale TCA-BME input (offsets not monotone / not 16-byte aligned / past n_values, a
// GT with more values than a stage slot holds, bitmaps with more set bits than the GT's values)
// never reads or writes outside the caller's buffers: the stage or GT is skipped and the
// workspace's error word is set (include/spinfer.h). The fused all-gather variant stores every
// Y row into each peer's Y as well (spinfer_spmm_tp_gather).
#include <cuda.h>
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include "internal.cuh"
#include "ptx.cuh"

namespace spinfer {
namespace {

// SPINFER_ABLATION (ablation builds only, tools/ablation.py; the product build leaves it 0):
//   1: paper-style SMBD (Alg. 2): every lane pops the BitmapTile's bitmap itself with a
//      serial PopCount base per BT, no warp-scan table; W staged in shared memory as usual;
//   2: no shared-memory staging of W at all: the same per-lane decode reads bitmaps and values
//      from global memory (only X is staged).
#ifndef SPINFER_ABLATION
#define SPINFER_ABLATION 0
#endif
constexpr int kRd = 2;                    // GT rows per rowblock (128 output rows)
constexpr int kCWd = 16;                  // consumer warps: r = w >> 3, m = w & 7
constexpr int kProdWarp0 = kCWd;          // producer warps kCWd, kCWd + 2 (SMSPs 0 and 2)
constexpr int kNProd = 2;                 // stage i is issued by producer i % 2
constexpr int kRedWarp = kCWd + 1;        // reducer warp (SMSP 1)
// slot release: hardware named barriers (ids kBarIdSlot0 + slot), not mbarriers — a warp
// suspended on an mbarrier try_wait is re-woken by every mbarrier event of the CTA
constexpr uint32_t kBarIdSlot0 = 3;   // 0: __syncthreads, 1-2: final-segment reduction
// 20 warps = 5 per SM sub-partition (4 consumers + 1 role warp): 96 registers each (the
// per-sub-partition register file); setmaxnreg rebalancing measured no gain
constexpr int kWarpsD = kCWd + 4;         // + warp 19 (idle)
constexpr int kThreadsD = 32 * kWarpsD;
constexpr int kMaxSd = 8;
constexpr int kMaxGd = 4;
constexpr int kNSeg = 4;                  // segment slots between consumers and the reducer
constexpr uint32_t kHdrBytes = 64;        // per-slot stage header: value offsets, poison flag
constexpr uint32_t kTblBytes = 1024;      // one GroupTile's SMBD table (64 BTs x 2 halves x 8 B)
// shared-memory map (bytes from the 1024-aligned base)
constexpr uint32_t kBarFull = 0, kBarEmpty = 64, kBarSegFull = 128, kBarSegFree = 192, kSegMask = 224;
constexpr uint32_t kFinFlag = 256;        // [2] final segment: partial count if this CTA sums the GT row
constexpr uint32_t kDefer = 272;          // count + [<= 4] (grow | nparts << 16): cross-CTA sums left to the consumers
constexpr uint32_t kBarIdDefer = 11;      // named barrier: reducer done -> consumers read the deferred list
constexpr uint32_t kHdrStop = 1u << 16, kHdrBad = 1u << 17;   // header word 1: g | rows << 8 | flags
constexpr uint32_t kOffHdr = 1024;
constexpr uint32_t kOffTbl = kOffHdr + kMaxSd * kHdrBytes;   // per-warp SMBD tables
constexpr uint32_t kOffRing = (kOffTbl + kCWd * kTblBytes + 1023) / 1024 * 1024;

struct DParams {
    CUtensorMap tmap_x;           // X [K][Np] fp16, box {Np, 64 G}, 32B swizzle for Np = 16 (conflict-free ldmatrix)
    const int32_t *off;
    const uint64_t *bm;
    const uint16_t *vals;
    uint16_t *Y;
    const uint16_t *bias;         // fused epilogue: fp16 [M] or null
    int act;
    float *ws_seg;                // [P][kNSeg][2][8] warp partials (m16n8k16 D layout), 64 x Np fp32 each
    float *ws_cta;                // [MG][cslots] CTA partials of split rowblocks (row-major 64 x Np)
    int32_t *ws_cnt;              // [MG] CTA counters of split rowblocks (zero between calls)
    int32_t *ws_err;              // error word (non-zero: corrupt TCA-BME input was skipped)
    int KG, MG, M, N, K;
    int n_values;                 // values[] length: value ranges past it are rejected
    uint32_t U;                   // units = rowblocks x KG; U * P < 2^32
    int P, G, S;
    int cslots;                   // CTA partial slots per GT row (max CTAs one rowblock overlaps)
    uint32_t slot_bytes, st_bm, st_v0, st_v1, vcap;   // slot: X slab | bitmaps | values row 0 | row 1
    float avg_gt;                 // n_values / NGT (start-up page prefetch hint)
    int npeer;                    // fused all-gather (spinfer_spmm_tp_gather): Y rows also stored into
    uint16_t *ypeer[kMaxPeers];   //   every peer's Y (ypeer[0..npeer), peer-mapped); 0: Y only
    long long *prof;              // experiments only (SPINFER_INSTRUMENT)
    int pdl;                      // launched with programmatic dependent launch (SPINFER_OPT_PDL)
};

#ifndef SPINFER_INSTRUMENT
#define SPINFER_INSTRUMENT 0
#endif
// Per-warp cycle accounting (instrumented build only): consumers k0 waiting for data, k1 scan,
// k2 decode, k3 segment hand-off, k4 GTs decoded, k5 first data seen, k6 exit, k7 other;
// producer k0 waiting for a free slot, k1 issuing; reducer k0 waiting, k1 reducing.
constexpr int kProfW = 20;
constexpr size_t kTraceOff = 1024 * kProfW * 8;   // stage trace of CTA 0 after the counters
[[maybe_unused]] constexpr size_t kEvOff = kTraceOff + 256 * 4;      // per-warp event trace of CTA 0: [16 warps][64 stages][6]
[[maybe_unused]] constexpr size_t kGtOff = kEvOff + 16 * 64 * 6;    // per CTA [1024][4]: globaltimer at entry, max exit
[[maybe_unused]] constexpr size_t kSmidOff = kGtOff + 1024 * 4;     // per CTA: the SM it ran on
struct Prof {
#if SPINFER_INSTRUMENT
    long long c[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    long long t = 0, t0 = 0;
    __device__ __forceinline__ void start() { t0 = t = clock64(); }
    __device__ __forceinline__ void lap(int k) { const long long n = clock64(); c[k] += n - t; t = n; }
    __device__ __forceinline__ void mark(int k) { c[k] = clock64() - t0; }
    __device__ __forceinline__ void count(int k) { ++c[k]; }
    __device__ __forceinline__ void dump(long long *prof, int p, int w, int lane) {
        if (prof && lane == 0 && p < 1024)
            for (int k = 0; k < 8; ++k) prof[((size_t)p * kProfW + w) * 8 + k] = c[k];
    }
    // CTA 0 stage trace: [i][k] k0 producer issue, k1 first owner wake (min), k2 last release, k3 producer wait start
    __device__ __forceinline__ void st(long long *prof, int p, int i, int k, bool mx) {
        if (!prof || p != 0 || i >= 256) return;
        unsigned long long *q = reinterpret_cast<unsigned long long *>(prof) + kTraceOff + (size_t)i * 4 + k;
        const unsigned long long v = (unsigned long long)(clock64() - t0 + 1);
        atomicMax(q, mx ? v : ~v);   // min fields hold the complement
    }
    __device__ __forceinline__ void ev(long long *prof, int p, int w, int i, int k) {
        if (prof && p == 0 && w < 16 && i < 64) prof[kEvOff + ((size_t)w * 64 + i) * 6 + k] = clock64() - t0;
    }
    // globaltimer (ns) at CTA entry (k = 0) and the latest exit of role k (1 consumers, 2 producers, 3 reducer)
    __device__ __forceinline__ void gt(long long *prof, int p, int k) {
        if (!prof || p >= 1024) return;
        unsigned long long g;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g));
        atomicMax(reinterpret_cast<unsigned long long *>(prof) + kGtOff + (size_t)p * 4 + k, g);
    }
#else
    __device__ __forceinline__ void gt(long long *, int, int) {}
    __device__ __forceinline__ void ev(long long *, int, int, int, int) {}
    __device__ __forceinline__ void start() {}
    __device__ __forceinline__ void lap(int) {}
    __device__ __forceinline__ void mark(int) {}
    __device__ __forceinline__ void count(int) {}
    __device__ __forceinline__ void dump(long long *, int, int, int) {}
    __device__ __forceinline__ void st(long long *, int, int, int, bool) {}
#endif
};

__device__ __forceinline__ int ustart(int p, uint32_t U, int P) { return (int)((uint32_t)p * U / (uint32_t)P); }
__device__ __forceinline__ int uowner(int u, uint32_t U, int P) { return (int)(((uint32_t)(u + 1) * (uint32_t)P - 1u) / U); }

// The CTA's stage walk (every warp runs its own copy). A CTA's unit range [u0, u1) runs in the
// order A = tail of the rowblock it starts inside (split with CTA p-1), C = head of the rowblock
// it ends inside (split with CTA p+1), then the full rowblocks: split rowblocks finish early, so
// their cross-CTA sums do not trail the kernel. A stage = up to G consecutive units of one
// rowblock; a segment = the stages of one part inside one rowblock.
struct Stages {
    int u, ue, us;
    int ns0, ne0, ns1, ne1;
    int rb, gc, g, rows;
    __device__ __forceinline__ void init(int u0, int u1, int KG, int G, int MG) {
        const int a_end = (u0 % KG) ? min(u1, (u0 / KG + 1) * KG) : u0;
        const int c_beg = (u1 % KG) ? max(a_end, (u1 / KG) * KG) : u1;
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
        part(q0s, q0e, KG, G, MG);
    }
    __device__ __forceinline__ void part(int s0, int e0, int KG, int G, int MG) {
        u = s0; us = s0; ue = e0;
        rb = (int)((uint32_t)u / (uint32_t)KG);
        gc = u - rb * KG;
        shape(KG, G, MG);
    }
    __device__ __forceinline__ void shape(int KG, int G, int MG) {
        g = min(min(G, KG - gc), ue - u);
        rows = min(kRd, MG - kRd * rb);
    }
    __device__ __forceinline__ bool valid() const { return u < ue; }
    __device__ __forceinline__ bool seg_first() const { return u == us || gc == 0; }
    __device__ __forceinline__ bool seg_last(int KG) const { return gc + g == KG || u + g == ue; }
    __device__ __forceinline__ void next(int KG, int G, int MG) {
        u += g;
        gc += g;
        if (gc == KG) { gc = 0; ++rb; }
        if (u == ue && ns0 < ne0) {
            const int s0 = ns0, e0 = ne0;
            ns0 = ns1; ne0 = ne1; ns1 = ne1;
            part(s0, e0, KG, G, MG);
        } else {
            shape(KG, G, MG);
        }
    }
};

// SMBD selector: PRMT of the two zero-extended u16 loads {V[c2-2], V[c2-1]} with selector
// y (kSelA + kSelB y) + kSelC for the lane's bit pair y (found by exhaustive search,
// tools/selector_search.py; pinned in tests/test_host_logic.py).
constexpr uint32_t kSelA = 0x7f62u, kSelB = 0x4cbfu, kSelC = 0x2333u;

__device__ __forceinline__ float epi_act(float v, float b, int act) {
    v += b;
    return act == SPINFER_ACT_RELU ? fmaxf(v, 0.f) : v;
}

// Y rows [row_base, row_base + 64) from accumulators in the m16n8k16 D layout. EPI: fused
// bias/activation, padding rows of a ragged M (A8), N not a multiple of 8. The fused all-gather
// stores the same rows into every peer's Y as well.
template <int NT, bool EPI, int TR = 4>
__device__ __forceinline__ void store_frag(const DParams &prm, int row_base, float (&acc)[TR][NT][4], int lane) {
    const int N = prm.N;
#pragma unroll
    for (int tr = 0; tr < TR; ++tr) {
        const int r0 = row_base + tr * 16 + (lane >> 2);
        if (EPI && (prm.bias || prm.act)) {
            // rows past M (padding of a ragged M) read no bias
            const float b0 = (prm.bias && r0 < prm.M) ? __half2float(__ushort_as_half(prm.bias[r0])) : 0.f;
            const float b1 = (prm.bias && r0 + 8 < prm.M) ? __half2float(__ushort_as_half(prm.bias[r0 + 8])) : 0.f;
#pragma unroll
            for (int nt = 0; nt < NT; ++nt) {
                acc[tr][nt][0] = epi_act(acc[tr][nt][0], b0, prm.act);
                acc[tr][nt][1] = epi_act(acc[tr][nt][1], b0, prm.act);
                acc[tr][nt][2] = epi_act(acc[tr][nt][2], b1, prm.act);
                acc[tr][nt][3] = epi_act(acc[tr][nt][3], b1, prm.act);
            }
        }
        for (int dst = 0; dst < max(1, prm.npeer); ++dst) {
        uint16_t *const Y = prm.npeer ? prm.ypeer[dst] : prm.Y;
#pragma unroll
        for (int nt = 0; nt < NT; ++nt) {
            const int col = nt * 8 + 2 * (lane & 3);
            const __half2 lo = __floats2half2_rn(acc[tr][nt][0], acc[tr][nt][1]);   // one RNE per output (A11)
            const __half2 hi = __floats2half2_rn(acc[tr][nt][2], acc[tr][nt][3]);
            if (!EPI) {
                *reinterpret_cast<__half2 *>(Y + (size_t)r0 * N + col) = lo;
                *reinterpret_cast<__half2 *>(Y + (size_t)(r0 + 8) * N + col) = hi;
            } else {
                __half *y0 = reinterpret_cast<__half *>(Y + (size_t)r0 * N);
                __half *y1 = reinterpret_cast<__half *>(Y + (size_t)(r0 + 8) * N);
                const bool v0 = r0 < prm.M, v1 = r0 + 8 < prm.M;
                if (N == NT * 8 && v0) *reinterpret_cast<__half2 *>(y0 + col) = lo;
                if (N == NT * 8 && v1) *reinterpret_cast<__half2 *>(y1 + col) = hi;
                if (N != NT * 8) {
                    if (v0 && col < N) y0[col] = __low2half(lo);
                    if (v0 && col + 1 < N) y0[col + 1] = __high2half(lo);
                    if (v1 && col < N) y1[col] = __low2half(hi);
                    if (v1 && col + 1 < N) y1[col + 1] = __high2half(hi);
                }
            }
        }
        }
    }
}

// NC consecutive outputs Y[row][col0 .. col0 + NC) (NC = 2 or 4, col0 a multiple of NC).
template <int NT, bool EPI, int NC>
__device__ __forceinline__ void store_cols(const DParams &prm, int row, int col0, const float (&v)[NC]) {
    const int N = prm.N;
    if (EPI && row >= prm.M) return;   // padding row of a ragged M (A8)
    float w[NC];
    const float b = (EPI && prm.bias) ? __half2float(__ushort_as_half(prm.bias[row])) : 0.f;
#pragma unroll
    for (int c = 0; c < NC; ++c) w[c] = EPI ? epi_act(v[c], b, prm.act) : v[c];
    for (int dst = 0; dst < max(1, prm.npeer); ++dst) {
    __half *y = reinterpret_cast<__half *>((prm.npeer ? prm.ypeer[dst] : prm.Y) + (size_t)row * N);
    if (!EPI || N == NT * 8) {
        if constexpr (NC == 4) {
            const __half2 a = __floats2half2_rn(w[0], w[1]), c2 = __floats2half2_rn(w[2], w[3]);
            uint2 u;
            u.x = *reinterpret_cast<const uint32_t *>(&a);
            u.y = *reinterpret_cast<const uint32_t *>(&c2);
            *reinterpret_cast<uint2 *>(y + col0) = u;
        } else {
            *reinterpret_cast<__half2 *>(y + col0) = __floats2half2_rn(w[0], w[1]);
        }
    } else {
#pragma unroll
        for (int c = 0; c < NC; ++c)
            if (col0 + c < N) y[col0 + c] = __float2half_rn(w[c]);
    }
    }
}

__device__ __forceinline__ void stg_f4(float4 *p, float4 v) {
    asm volatile("st.global.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w) : "memory");
}
__device__ __forceinline__ void stg_f2(float *p, float x, float y) {
    asm volatile("st.global.v2.f32 [%0], {%1, %2};" ::"l"(p), "f"(x), "f"(y) : "memory");
}
// Drop an L2 line without writing it back: every partial is read exactly once.
__device__ __forceinline__ void discard_l2(const void *p) {
    asm volatile("discard.global.L2 [%0], 128;" ::"l"(p) : "memory");
}
// The CTA partial of GT row `grow` (row-major 64 x Np fp32) is parked: count this CTA. True for
// the last of the CTAs overlapping the rowblock, which then sums all CTA partials (cta_sum) and
// re-zeroes the counter. One whole warp, after every partial store is ordered before it.
__device__ __forceinline__ bool cta_arrive(const DParams &prm, int rb, int grow, int lane, int &nparts) {
    const int pf = uowner(rb * prm.KG, prm.U, prm.P), pl = uowner((rb + 1) * prm.KG - 1, prm.U, prm.P);
    nparts = pl - pf + 1;
    __threadfence();
    int old = 0;
    if (lane == 0) old = atomicAdd(prm.ws_cnt + grow, 1);
    old = __shfl_sync(0xffffffffu, old, 0);
    if (old != pl - pf) return false;
    if (lane == 0) prm.ws_cnt[grow] = 0;   // leave the workspace zeroed for the next call
    __threadfence();                       // acquire: every CTA partial is visible
    return true;
}
// Sum, in CTA order, of the nparts CTA partials of GT row `grow` over the float4 columns
// [f0, f0 + 32 J) of the row-major 64 x Np block, written to Y. The loads of 4 partials are in
// flight together (the sum is latency-bound: up to ~20 partials on a long-K shard).
template <int NT, bool EPI, int J>
__device__ __forceinline__ void cta_sum(const DParams &prm, int grow, int nparts, int f0, int lane) {
    constexpr int Np = NT * 8, kF4 = 64 * Np / 4;
    const float4 *base = reinterpret_cast<const float4 *>(prm.ws_cta) + (size_t)grow * prm.cslots * kF4 + f0 + lane;
    float4 s[J];
#pragma unroll
    for (int j = 0; j < J; ++j) s[j] = make_float4(0.f, 0.f, 0.f, 0.f);
    auto add = [](float4 &x, const float4 y) { x.x += y.x; x.y += y.y; x.z += y.z; x.w += y.w; };
    int q = 0;
    for (; q + 4 <= nparts; q += 4) {
        float4 v[4][J];
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int j = 0; j < J; ++j) v[u][j] = __ldcg(base + (size_t)(q + u) * kF4 + 32 * j);
#pragma unroll
        for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int j = 0; j < J; ++j) add(s[j], v[u][j]);
    }
    for (; q < nparts; ++q)
#pragma unroll
        for (int j = 0; j < J; ++j) add(s[j], __ldcg(base + (size_t)q * kF4 + 32 * j));
#pragma unroll
    for (int j = 0; j < J; ++j) {
        const int e = 4 * (f0 + 32 * j + lane);   // element index in the row-major 64 x Np block
        const float v[4] = {s[j].x, s[j].y, s[j].z, s[j].w};
        store_cols<NT, EPI, 4>(prm, grow * 64 + e / Np, e % Np, v);
    }
    // every partial line is read exactly once: drop it from L2 without a write-back
    for (int q2 = 0; q2 < nparts; ++q2)
        if (lane < 4 * J) discard_l2(base - lane + (size_t)q2 * kF4 + 8 * lane);
}

template <int NT, bool EPI>
__global__ void __launch_bounds__(kThreadsD, 1) k_spmm_dw(const __grid_constant__ DParams prm) {
    constexpr int Np = NT * 8;
    constexpr int kF4 = 64 * Np / 4;   // float4 per 64 x Np partial
    // half mode (N 17-32, NT = 4): a consumer warp owns TCTile rows 2h, 2h + 1 of its GroupTile (32
    // output rows, 32 fp32 accumulators at N = 32); the two halves of a GT are two warps
    constexpr bool HALF = NT > 2;
    constexpr int TRW = HALF ? 2 : 4;   // TCTile rows per consumer warp
    constexpr int kSlotW = HALF ? 4 : 8;   // GT slots per GT row and phase set (warps per half-row)
    constexpr int JC = (kF4 + 255) / 256;   // float4 columns of a 64 x Np block per lane (8 warps)
    constexpr uint32_t kOwnW = HALF ? 2u : 1u;   // consumer warps per GT
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    uint8_t *const smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    const uint32_t sbase = smem_u32(smem);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int p = blockIdx.x;
    const int KG = prm.KG, G = prm.G, S = prm.S, MG = prm.MG;
    const uint32_t bar_full = sbase + kBarFull, bar_empty = sbase + kBarEmpty;
    const uint32_t bar_sfull = sbase + kBarSegFull, bar_sfree = sbase + kBarSegFree;
    const uint32_t seg_mask = sbase + kSegMask;
    const uint32_t ring = sbase + kOffRing;
    const int u0 = ustart(p, prm.U, prm.P), u1 = ustart(p + 1, prm.U, prm.P);

    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            mbar_init(bar_full + 8 * s, 32);             // the producer warp's lanes (lane 0: expect_tx) + TMA bytes
            mbar_init(bar_empty + 8 * s, kRd * kMaxGd);  // the stage's GT owners + the producer's pre-arrival
        }
        for (int k = 0; k < kNSeg; ++k) {
            mbar_init(bar_sfull + 16 * k, 8);             // row 0: its 8 consumer warps
            mbar_init(bar_sfull + 16 * k + 8, 8);         // row 1
            mbar_init(bar_sfree + 8 * k, 1);              // the reducer has read the slot
            sts_u32(seg_mask + 8 * k, 0u);
            sts_u32(seg_mask + 8 * k + 4, 0u);
        }
        sts_u32(sbase + kDefer, 0u);
        fence_barrier_init();
    }
    __syncthreads();
    // programmatic dependent launch (SPINFER_OPT_PDL): the next kernel on the stream may be scheduled
    // now; its CTAs take SMs as this grid's CTAs retire
    if (threadIdx.x == 0) grid_dep_launch();
    Prof pf;
    pf.start();
    if (threadIdx.x == 0) pf.gt(prm.prof, p, 0);
#if SPINFER_INSTRUMENT
    if (threadIdx.x == 0 && prm.prof && p < 1024) {
        uint32_t smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        prm.prof[kSmidOff + p] = smid;
    }
#endif
    // role warps: producers / reducer / idle. Each branch below ends in a return.
    if (warp >= kCWd) {
    if (warp == kCWd + 3) return;   // the idle warp (completes the warpgroup)

    if (warp == kProdWarp0 || warp == kProdWarp0 + 2) {
        // ------------------------------------------------------------------ producers (2 warps)
        // Producer q issues the stages i with i % 2 == q. Lanes 0-4 / 8-12 hold the GTileOffset
        // entries j = 0..4 of GT row 0 / 1 of a stage, loaded two own stages ahead with one load
        // instruction. All of a stage's copies go out in ONE bulk-copy instruction from different
        // lanes (lane 0 / 8: packed values of row 0 / 1, lane 1: the X slab, lanes 2, 3: the
        // bitmaps of rows 0, 1): a thread's successive bulk copies serialise at ~310 ns each
        // (tools/tma_sweep2.sh: 4 KB chunks from one thread 1.97 TB/s, 8 lanes x 4 KB per
        // instruction 5.7 TB/s).
        const int q = (warp - kProdWarp0) >> 1;
        const int orow = lane >> 3, oj = lane & 7;
        if (lane == 0) prefetch_tmap(&prm.tmap_x);
        Stages it;
        it.init(u0, u1, KG, G, MG);
        int nseg = 0, i = 0;
        uint32_t pslot = 0;            // ring slot of stage i
        uint32_t owners_pk = 0;        // 4 bits per slot: GT owners of the stage last issued into it
        auto step = [&](Stages &s, int &ns, int &ii) {   // one stage forward (segment count, index)
            if (s.seg_last(KG)) ++ns;
            s.next(KG, G, MG);
            ++ii;
        };
        if (q == 1 && it.valid()) { step(it, nseg, i); pslot = 1; }
        Stages ia = it;   // two own stages ahead of `it`: the offset prefetch
        int nsa = nseg, ia_i = i;
        // start-up: touch the predicted first value line of each GT row (page translation
        // overlaps the GTileOffset loads the first copies wait for; a hint only)
        if (it.valid() && lane < it.rows)
            prefetch_l2(prm.vals + (long long)((double)((long long)(kRd * it.rb + lane) * KG + it.gc) * prm.avg_gt));
        auto ld_off = [&](const Stages &sg) -> int {
            return (sg.valid() && orow < sg.rows && oj <= sg.g)
                       ? __ldg(prm.off + (long long)(kRd * sg.rb + orow) * KG + sg.gc + oj) : 0;
        };
        auto skip2 = [&](Stages &s, int &ns, int &ii) {
            for (int k = 0; k < kNProd && s.valid(); ++k) step(s, ns, ii);
        };
        int oc = ld_off(ia);
        skip2(ia, nsa, ia_i);
        int on = ld_off(ia);
        skip2(ia, nsa, ia_i);

        const uint64_t pol = policy_evict_first();
        while (it.valid()) {
            const uint32_t slot = pslot;
            pf.lap(1);
            if (lane == 0) pf.st(prm.prof, p, i, 3, true);
            // the slot's previous stage (i - S) released by its GT owners: hardware named barrier
            // (the waiting warp is not woken by the CTA's mbarrier traffic, no polling)
            if (i >= S) named_bar_sync(kBarIdSlot0 + slot, 32u * (1u + kOwnW * ((owners_pk >> (4 * slot)) & 15u)));
            pf.lap(0);
            if (lane == 0) pf.st(prm.prof, p, i, 0, true);
            const uint32_t st = ring + slot * prm.slot_bytes, fb = bar_full + 8 * slot;
            const uint32_t hb = sbase + kOffHdr + slot * kHdrBytes;
            const int g = it.g, rows = it.rows;
            owners_pk = (owners_pk & ~(15u << (4 * slot))) | ((uint32_t)(rows * g) << (4 * slot));
            // validate the stage's value ranges (never trust the caller's max_gt_values)
            const int obeg = __shfl_sync(0xffffffffu, oc, lane & 8);
            const int oend = __shfl_sync(0xffffffffu, oc, (lane & 8) + g);
            const int onxt = __shfl_down_sync(0xffffffffu, oc, 1);
            bool badl = false;
            if (orow < rows && oj < g) badl = onxt < oc;
            if (orow < rows && oj == 0)
                badl |= (oc & 7) != 0 || oc < 0 || oend > prm.n_values || 2LL * (oend - oc) > (long long)prm.vcap;
            const uint32_t badm = __ballot_sync(0xffffffffu, badl);   // lanes 0-7: row 0, 8-15: row 1
            const bool bad0 = (badm & 0xFFu) != 0, bad1 = (badm & 0xFF00u) != 0;
            const bool bad = orow ? bad1 : bad0;
            pf.lap(2);
            // header: stage shape, segment index, per-GT value offsets (bytes from the row's value region)
            if (orow < kRd && oj <= kMaxGd) sts_u32(hb + 16u + 20u * orow + 4u * oj, 2u * (uint32_t)(oc - obeg));
            if (lane == 31)
                sts_v4(hb, make_uint4((uint32_t)it.rb, (uint32_t)g | ((uint32_t)rows << 8) | ((bad0 || bad1) ? kHdrBad : 0u),
                                      (uint32_t)nseg, (uint32_t)it.gc));
#if SPINFER_ABLATION == 2
            if (oj == 0 && orow < kRd) sts_u32(hb + 56u + 4u * orow, (uint32_t)oc);   // the row's first value (global)
            const uint32_t vbl = 0u;
#else
            const uint32_t vbl = (oj == 0 && orow < rows && !bad) ? 2u * (uint32_t)(oend - oc) : 0u;   // lanes 0, 8
#endif
            const uint32_t vb1 = __shfl_sync(0xffffffffu, vbl, 8);
            // the X slab: one tensor copy of G GT columns (rows past K zero-filled by the TMA)
            const uint32_t xbytes = (uint32_t)G * 64u * Np * 2u;
            const uint32_t bmb = SPINFER_ABLATION == 2 ? 0u : (uint32_t)g * 512u;
            if (lane == 0) {
                if (badm) atomicOr(prm.ws_err, 1);
                // every transaction byte registered up front: the phase completes only when all
                // copies of the stage have landed
                mbar_arrive_expect_tx(fb, (uint32_t)rows * bmb + xbytes + vbl + vb1);
            } else {
                mbar_arrive(fb);   // each lane releases its own header stores
            }
            __syncwarp();          // expect_tx before any copy is issued
            pf.lap(3);
            uint32_t dst = 0, bytes = 0;
            const void *src = nullptr;
            if (oj == 0) {                                  // lanes 0, 8: packed values of row orow
                dst = st + (orow ? prm.st_v1 : prm.st_v0); src = prm.vals + oc; bytes = vbl;
            } else if (lane == 2 || lane == 3) {            // bitmaps of row lane - 2
                const int r = lane - 2;
                dst = st + prm.st_bm + (uint32_t)(r * G) * 512u;
                src = prm.bm + ((size_t)(kRd * it.rb + r) * KG + it.gc) * 64;
                bytes = r < rows ? bmb : 0u;
            }
            if (bytes) bulk_g2s(dst, src, bytes, fb, pol);
            // X may be the previous kernel's output (programmatic dependent launch, SPINFER_OPT_PDL):
            // this producer's first stage waits for that grid with its weight copies already in
            // flight. Every other global access of X, the workspace or Y follows from this stage's
            // data. Without PDL the wait returns at once. (Deferring the X copies of all first S / 2
            // stages instead measured 3 us slower on the OPT-30B stack.)
            if (i < kNProd) grid_dep_wait();
            if (lane == 1) tma_2d_g2s(st, &prm.tmap_x, 0, 64 * it.gc, fb);
            pf.lap(4);

            skip2(it, nseg, i);
            pslot += 2;
            if (pslot >= (uint32_t)S) pslot -= (uint32_t)S;
            oc = on;
            on = ld_off(ia);   // two own stages ahead: in flight while this warp issues the next stages
            skip2(ia, nsa, ia_i);
            pf.lap(5);
        }
        // stop sentinels: one per consumer phase, in the slots of the stage indices [nst, nst + phases)
        // (phases = 8 / G, 4 / G in half mode; S >= phases: distinct slots); this producer writes
        // those of its parity. The header carries the CTA's segment count.
        {
            const int nst = i;                      // the loop ends with i = the stage count
            for (int j = nst + ((nst & 1) != q ? 1 : 0); j < nst + (HALF ? 4 : 8) / G; j += 2) {
                const uint32_t slot = (uint32_t)(j % S);
                if (j >= S) named_bar_sync(kBarIdSlot0 + slot, 32u * (1u + kOwnW * ((owners_pk >> (4 * slot)) & 15u)));
                owners_pk &= ~(15u << (4 * slot));
                if (lane == 0) sts_v4(sbase + kOffHdr + slot * kHdrBytes, make_uint4(0u, kHdrStop, (uint32_t)nseg, 0u));
                mbar_arrive(bar_full + 8 * slot);
            }
        }
        if (lane == 0) pf.gt(prm.prof, p, 2);
        pf.mark(6);
        pf.dump(prm.prof, p, warp, lane);
        return;
    }

    if (warp == kRedWarp) {
        // ------------------------------------------------------------------ reducer (one warp)
        // Non-final segments of the CTA, in order: sum the GT row's warp partials (warp order),
        // then write Y (the CTA holds the whole rowblock) or park the CTA partial for the
        // cross-CTA sum.
        Stages it;
        it.init(u0, u1, KG, G, MG);
        int nseg = 0, sstart = 0;
        while (it.valid()) {
            if (it.seg_first()) sstart = it.u;
            const bool seg_end = it.seg_last(KG);
            const int rb = it.rb, rows = it.rows, send = it.u + it.g;
            it.next(KG, G, MG);
            if (!seg_end) continue;
            if (!it.valid()) break;   // the final segment: the consumers reduce it in shared memory
            const int k = nseg % kNSeg;
            const uint32_t par = (uint32_t)(nseg / kNSeg) & 1u;
            const bool complete = sstart == rb * KG && send == (rb + 1) * KG;
            for (int r = 0; r < rows; ++r) {
                pf.lap(1);
                mbar_wait_expo(bar_sfull + 16 * k + 8 * r, par, 256u, 4096u);
                pf.lap(0);
                const uint32_t cmask = lds_u32(seg_mask + 8 * k + 4 * r);   // warps that own a GT of the segment
                __syncwarp();   // every lane has read the mask before it is reset
                if (lane == 0) sts_u32(seg_mask + 8 * k + 4 * r, 0u);
                const float4 *src = reinterpret_cast<const float4 *>(prm.ws_seg) + ((((size_t)p * kNSeg + k) * kRd + r) * 8) * kF4;
                const int grow = kRd * rb + r;
                if constexpr (HALF) {
                    // rows 32 hh .. 32 hh + 31 are the sum over jm = 0..3 (warp order) of warps 2 jm + hh
#pragma unroll 1
                    for (int hh = 0; hh < 2; ++hh) {
                        float acc[2][NT][4];
#pragma unroll
                        for (int tr = 0; tr < 2; ++tr)
#pragma unroll
                            for (int nt = 0; nt < NT; ++nt) {
                                float4 v[4];
#pragma unroll
                                for (int u = 0; u < 4; ++u) {
                                    const int mw = 2 * u + hh;
                                    v[u] = ((cmask >> mw) & 1u) ? __ldcg(src + (size_t)mw * kF4 + (tr * NT + nt) * 32 + lane)
                                                                : make_float4(0.f, 0.f, 0.f, 0.f);
                                }
                                float4 t = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
                                for (int u = 0; u < 4; ++u) { t.x += v[u].x; t.y += v[u].y; t.z += v[u].z; t.w += v[u].w; }
                                acc[tr][nt][0] = t.x; acc[tr][nt][1] = t.y; acc[tr][nt][2] = t.z; acc[tr][nt][3] = t.w;
                            }
                        if (complete) {
                            store_frag<NT, EPI, 2>(prm, grow * 64 + 32 * hh, acc, lane);
                        } else {
                            const int pfirst = uowner(rb * KG, prm.U, prm.P);
                            float *const cdst = prm.ws_cta + ((size_t)grow * prm.cslots + (p - pfirst)) * (64 * Np);
#pragma unroll
                            for (int tr = 0; tr < 2; ++tr)
#pragma unroll
                                for (int nt = 0; nt < NT; ++nt) {
                                    const int row = 32 * hh + tr * 16 + (lane >> 2), col = nt * 8 + 2 * (lane & 3);
                                    stg_f2(cdst + row * Np + col, acc[tr][nt][0], acc[tr][nt][1]);
                                    stg_f2(cdst + (row + 8) * Np + col, acc[tr][nt][2], acc[tr][nt][3]);
                                }
                        }
                    }
                    for (int mw = 0; mw < 8; ++mw)   // each warp's partial: 2 x NT x 32 float4 = 32 lines
                        if ((cmask >> mw) & 1u) discard_l2(src + (size_t)mw * kF4 + 8 * lane);
                    if (!complete) {
                        __syncwarp();
                        int nparts;
                        if (cta_arrive(prm, rb, grow, lane, nparts) && lane == 0) {
                            const uint32_t nd = lds_u32(sbase + kDefer);
                            sts_u32(sbase + kDefer + 4 + 4 * nd, (uint32_t)grow | ((uint32_t)nparts << 16));
                            sts_u32(sbase + kDefer, nd + 1);
                        }
                    }
                } else {
                    float acc[4][NT][4];
#pragma unroll
                    for (int a = 0; a < 4; ++a)
#pragma unroll
                        for (int b = 0; b < NT; ++b)
#pragma unroll
                            for (int e = 0; e < 4; ++e) acc[a][b][e] = 0.f;
                    // warp order; a warp without a GT of the segment contributes +0 (sums start at +0:
                    // adding +0 changes no bit). Four warps' loads in flight together.
#pragma unroll
                    for (int tr = 0; tr < 4; ++tr)
#pragma unroll
                        for (int mh = 0; mh < 8; mh += 4) {
                            float4 v[4][NT];
#pragma unroll
                            for (int u = 0; u < 4; ++u)
#pragma unroll
                                for (int nt = 0; nt < NT; ++nt)
                                    v[u][nt] = ((cmask >> (mh + u)) & 1u) ? __ldcg(src + (size_t)(mh + u) * kF4 + (tr * NT + nt) * 32 + lane)
                                                                          : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
                            for (int u = 0; u < 4; ++u)
#pragma unroll
                                for (int nt = 0; nt < NT; ++nt) {
                                    const float4 w = v[u][nt];
                                    acc[tr][nt][0] += w.x; acc[tr][nt][1] += w.y; acc[tr][nt][2] += w.z; acc[tr][nt][3] += w.w;
                                }
                        }
                    for (int m = 0; m < 8; ++m)
                        if (((cmask >> m) & 1u) && lane < kF4 / 8) discard_l2(src + (size_t)m * kF4 + 8 * lane);
                    if (complete) {
                        store_frag<NT, EPI>(prm, grow * 64, acc, lane);
                    } else {
                        const int pfirst = uowner(rb * KG, prm.U, prm.P);
                        float *dst = prm.ws_cta + ((size_t)grow * prm.cslots + (p - pfirst)) * (64 * Np);
#pragma unroll
                        for (int tr = 0; tr < 4; ++tr)
#pragma unroll
                            for (int nt = 0; nt < NT; ++nt) {
                                const int row = tr * 16 + (lane >> 2), col = nt * 8 + 2 * (lane & 3);
                                stg_f2(dst + row * Np + col, acc[tr][nt][0], acc[tr][nt][1]);
                                stg_f2(dst + (row + 8) * Np + col, acc[tr][nt][2], acc[tr][nt][3]);
                            }
                        __syncwarp();
                        // the last CTA of the rowblock: the sum is deferred to the consumer warps' end
                        // phase (8 warps per GT row, all loads in flight; a single warp here would be
                        // latency-bound over up to ~20 partials)
                        int nparts;
                        if (cta_arrive(prm, rb, grow, lane, nparts) && lane == 0) {
                            const uint32_t nd = lds_u32(sbase + kDefer);
                            sts_u32(sbase + kDefer + 4 + 4 * nd, (uint32_t)grow | ((uint32_t)nparts << 16));
                            sts_u32(sbase + kDefer, nd + 1);
                        }
                    }
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(bar_sfree + 8 * k);   // the slot's partials may be overwritten
            ++nseg;
        }
        __syncwarp();
        named_bar_arrive(kBarIdDefer, 32u * (kCWd + 1));   // the deferred-sum list is complete
        pf.lap(1);
        if (lane == 0) pf.gt(prm.prof, p, 3);
        pf.mark(6);
        pf.dump(prm.prof, p, warp, lane);
        return;
    }

    }   // role warps

    // ---------------------------------------------------------------------- consumers
    // Warp (r, m) owns GT j = m % G of GT row r in every stage i with i % (8 / G) == m / G
    // (G in {1, 2, 4}: all 8 warps of a row busy); it reads the stage's shape and segment index
    // from the slot header. Half mode: warp (r, m) owns TCTile rows 2 hw, 2 hw + 1 (hw = m & 1) of
    // GT j = jm % G, jm = m >> 1, in the stages i % (4 / G) == jm / G.
    const int r = warp >> 3, m = warp & 7;
    const int hw = HALF ? (m & 1) : 0, jm = HALF ? (m >> 1) : m;
    const int jw = jm % G;
    const int tstride = (HALF ? 4 : 8) / G;   // stages between two of this warp's
    const uint32_t mulc = opaque_u32(1u << (30u - 2u * (uint32_t)(lane & 15)));   // z = w << (30 - sh) on the FMA pipe
    constexpr uint32_t selA = kSelA, selB = kSelB, selC = kSelC;   // IMAD immediates
    constexpr uint32_t cpr = Np / 8;   // 16-byte chunks per X row
    const uint32_t rr = lane & 7, mk = (lane >> 3) & 1, mn = (lane >> 4) & 1;
    // X slab row-major; with the tensor copy the 32B swizzle XORs the 16-byte chunk with row bit 2
    // (Np = 16), the 64B swizzle with row bits 1-2 (Np = 32: a second ldmatrix for columns 16-31)
    const uint32_t x_lane = (mk * 8u + rr) * cpr * 16u +
                            ((HALF ? (mn ^ ((rr >> 1) & 3u)) : (mn ^ (NT == 2 ? (rr >> 2) & 1u : 0u))) * 16u);
    [[maybe_unused]] const uint32_t x_lane2 = (mk * 8u + rr) * cpr * 16u + (((2u + mn) ^ ((rr >> 1) & 3u)) * 16u);
    float acc[TRW][NT][4];
#pragma unroll
    for (int a = 0; a < TRW; ++a)
#pragma unroll
        for (int b = 0; b < NT; ++b)
#pragma unroll
            for (int e = 0; e < 4; ++e) acc[a][b][e] = 0.f;

    uint4 E[4];
    auto load_E = [&](uint32_t tb) {   // entries of 8 consecutive BTs, this lane's half
#pragma unroll
        for (int k = 0; k < 4; ++k) E[k] = lds_v4(tb + 16u * k);
    };
    auto load_E_nv = [&](uint32_t tb) {
#pragma unroll
        for (int k = 0; k < 4; ++k) E[k] = lds_v4_nv(tb + 16u * k);
    };
    auto assemble_nv = [&](const uint32_t (&u0)[8], const uint32_t (&u1)[8], const uint32_t (&sl)[8], int trb,
                           const uint32_t (&bfr)[NT][2]) {
#pragma unroll
        for (int tt = 0; tt < 2; ++tt) {
            uint32_t afr[4];
#pragma unroll
            for (int b = 0; b < 4; ++b) afr[b] = prmt(u0[tt * 4 + b], u1[tt * 4 + b], sl[tt * 4 + b]);
#pragma unroll
            for (int nt = 0; nt < NT; ++nt) mma_16816_nv(acc[trb + tt][nt], afr, bfr[nt][0], bfr[nt][1]);
        }
    };
    auto issue_to = [&](uint32_t (&u0)[8], uint32_t (&u1)[8], uint32_t (&sl)[8]) {   // SMBD value loads into a set
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            const uint32_t w = (k & 1) ? E[k >> 1].z : E[k >> 1].x;
            const uint32_t A = (k & 1) ? E[k >> 1].w : E[k >> 1].y;
            const uint32_t z = w * mulc;
            const uint32_t a = A + 2u * __popc(z);
            const uint32_t y = z >> 30;
            sl[k] = y * (y * selB + selA) + selC;
            u0[k] = lds_u16(a);
            u1[k] = lds_u16(a + 2u);
        }
    };
    // segment hand-off to the reducer (non-final segments): park the partial if this warp owned a
    // GT of the segment, then arrive; `own` = false arrives for a segment without a GT of this warp
    auto seg_close = [&](int sg, bool own) {
        const int k = sg % kNSeg;
        if (sg >= kNSeg) mbar_wait_poll(bar_sfree + 8 * k, (uint32_t)((sg / kNSeg) - 1) & 1u, 256u);
        if (own) {
            float4 *dst = reinterpret_cast<float4 *>(prm.ws_seg) + ((((size_t)p * kNSeg + k) * kRd + r) * 8 + m) * kF4;
#pragma unroll
            for (int tr = 0; tr < TRW; ++tr)
#pragma unroll
                for (int nt = 0; nt < NT; ++nt)
                    stg_f4(dst + (tr * NT + nt) * 32 + lane, make_float4(acc[tr][nt][0], acc[tr][nt][1], acc[tr][nt][2], acc[tr][nt][3]));
            if (lane == 0) atomicOr(reinterpret_cast<uint32_t *>(smem + kSegMask + 8 * k + 4 * r), 1u << m);
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(bar_sfull + 16 * k + 8 * r);   // release: the stores above
    };

    const uint32_t tbl = sbase + kOffTbl + (uint32_t)warp * kTblBytes;
    const uint32_t tbl_lane = tbl + (uint32_t)(lane >> 4) * 512u;
    // PopCount bases of a GT's 64 BitmapTiles into the table at `tb`: lane l pops BTs l and
    // l + 32, one 32-lane shuffle scan; false if the GT is poisoned or its bitmaps hold more set
    // bits than its value range (corrupt input: never read past the stage's values)
    auto scan_gt = [&](uint32_t st_, uint32_t voff_, uint32_t vend_, uint2 ba_, uint2 bb_, uint32_t flags_,
                       uint32_t tb) -> bool {
        const uint32_t vsm = st_ + (r ? prm.st_v1 : prm.st_v0) + voff_;
        const uint32_t pax = __popc(ba_.x), pbx = __popc(bb_.x);
        const uint32_t packed = (pax + __popc(ba_.y)) | ((pbx + __popc(bb_.y)) << 16);
        uint32_t incl = packed;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
            incl += (lane >= o) ? y : 0u;
        }
        const uint32_t tot = __shfl_sync(0xffffffffu, incl, 31);
        const uint32_t tot_a = tot & 0xFFFFu;
        if ((flags_ & kHdrBad) || 2u * (tot_a + (tot >> 16)) > vend_ - voff_) return false;
        const uint32_t excl = incl - packed;
        const uint32_t Aa = vsm + 2u * (excl & 0xFFFFu) - 4u;
        const uint32_t Ab = vsm + 2u * (tot_a + (excl >> 16)) - 4u;
        const uint32_t te = tb + 8u * lane;
        sts_v2(te, ba_.x, Aa);
        sts_v2(te + 512u, ba_.y, Aa + 2u * pax);
        sts_v2(te + 256u, bb_.x, Ab);
        sts_v2(te + 768u, bb_.y, Ab + 2u * pbx);
        __syncwarp();
        return true;
    };

    int i = jm / G;                 // stage index
    uint32_t slot = (uint32_t)(i % S), ph = 0;   // ring position of stage i (S >= 2)
    int cur = -1;                   // open segment of this warp (-1: none)
    bool contrib = false, seen = false;
    int nseg_total = 0, f_rb = 0, f_rows = 0;
    while (true) {
        pf.lap(7);
        if (lane == 0) pf.ev(prm.prof, p, warp, i >> 1, 0);
        if (!mbar_test_wait(bar_full + 8 * slot, ph)) mbar_wait_sleep(bar_full + 8 * slot, ph);
        if (lane == 0) pf.ev(prm.prof, p, warp, i >> 1, 1);
        if (!seen) { seen = true; pf.mark(5); }
        pf.lap(0);
        if (lane == 0) pf.st(prm.prof, p, i, 1, false);
        const uint32_t hb = sbase + kOffHdr + slot * kHdrBytes;
        const uint32_t st = ring + slot * prm.slot_bytes;
        // everything this stage needs from shared memory, in one round trip: header, this GT's
        // value range, its 64 bitmaps (lane l: BTs l and l + 32)
        const uint4 h = lds_v4(hb);
        const uint32_t voff = lds_u32(hb + 16u + 20u * (uint32_t)r + 4u * (uint32_t)jw);
        const uint32_t vend = lds_u32(hb + 20u + 20u * (uint32_t)r + 4u * (uint32_t)jw);
        const uint32_t bms = st + prm.st_bm + (uint32_t)(r * G + jw) * 512u;
        const uint2 ba = lds_v2(bms + 8u * lane), bb = lds_v2(bms + 256u + 8u * lane);
        if (h.y & kHdrStop) { nseg_total = (int)h.z; break; }
        const int sg = (int)h.z, g = (int)(h.y & 0xFFu), rows = (int)((h.y >> 8) & 3u);
        if (sg != cur) {   // this stage opens a new segment
            if (cur >= 0 && r < f_rows) seg_close(cur, contrib);
            for (int s2 = cur + 1; s2 < sg; ++s2) seg_close(s2, false);   // segments with no stage of this parity
            cur = sg;
#pragma unroll
            for (int a = 0; a < TRW; ++a)
#pragma unroll
                for (int b = 0; b < NT; ++b)
#pragma unroll
                    for (int e = 0; e < 4; ++e) acc[a][b][e] = 0.f;
            contrib = false;
        }
        f_rb = (int)h.x; f_rows = rows;
        pf.lap(3);
        if (lane == 0) pf.ev(prm.prof, p, warp, i >> 1, 2);
        if (r < rows && jw < g) {
            contrib = true;
#if SPINFER_ABLATION
            const bool ok = !(h.y & kHdrBad);
            (void)ba; (void)bb; (void)vend;
#else
            const bool ok = scan_gt(st, voff, vend, ba, bb, h.y, tbl);
#endif
            pf.lap(1);
            if (lane == 0) pf.ev(prm.prof, p, warp, i >> 1, 3);
            if (ok) {
                // --- decode the 16 TCTiles: TCTile column tc, row pairs (0,1), (2,3)
                // the whole GT is one schedulable region: addresses laundered after the table writes,
                // accumulators fenced at the end, no volatile operation in between
                const uint32_t xs = launder_u32(st + x_lane + (uint32_t)(64 * jw) * cpr * 16u);
                const uint32_t tbl_lane_l = launder_u32(tbl_lane);
                uint32_t t0[8], t1[8], s1[8];
#if SPINFER_ABLATION
                uint32_t abl_base = 0;   // values of the GT's earlier BitmapTiles
                const uint32_t vsm_gt = st + (r ? prm.st_v1 : prm.st_v0) + voff;
#if SPINFER_ABLATION == 2
                const uint64_t *gbm = prm.bm + ((size_t)(kRd * (int)h.x + r) * KG + (int)h.w + jw) * 64;
                const uint16_t *gv = prm.vals + lds_u32(hb + 56u + 4u * (uint32_t)r) + voff / 2u;
#endif
                (void)vsm_gt; (void)tbl_lane_l;
#endif
#pragma unroll
                for (int tc = 0; tc < 4; ++tc) {
                    uint32_t bfr[NT][2];
                    const uint32_t xk = xs + (uint32_t)(16 * tc) * cpr * 16u;
                    if constexpr (NT == 1) {
                        ldsm_x2_trans_nv(xk, bfr[0][0], bfr[0][1]);
                    } else if constexpr (NT == 2) {
                        ldsm_x4_trans_nv(xk, bfr[0][0], bfr[0][1], bfr[1][0], bfr[1][1]);
                    } else {   // Np = 32: columns 0-15 and 16-31
                        ldsm_x4_trans_nv(xk, bfr[0][0], bfr[0][1], bfr[1][0], bfr[1][1]);
                        ldsm_x4_trans_nv(xk + (x_lane2 - x_lane), bfr[2][0], bfr[2][1], bfr[3][0], bfr[3][1]);
                    }
#if SPINFER_ABLATION
#pragma unroll
                    for (int hh = 0; hh < 2; ++hh) {
#pragma unroll
                        for (int k = 0; k < 8; ++k) {
                            const int b = tc * 16 + hh * 8 + k;   // BitmapTile index in the GT
#if SPINFER_ABLATION == 1
                            const uint2 bw = lds_v2(bms + 8u * (uint32_t)b);
#else
                            const uint2 bw = ldg_nc_v2(gbm + b);
#endif
                            const uint32_t w = (lane < 16) ? bw.x : bw.y;
                            const uint32_t pre = abl_base + ((lane >= 16) ? (uint32_t)__popc(bw.x) : 0u);
                            abl_base += (uint32_t)(__popc(bw.x) + __popc(bw.y));   // serial PopCount base
                            const uint32_t z = w * mulc;
                            const uint32_t c2 = pre + (uint32_t)__popc(z);   // values through the lane's pair
                            const uint32_t y = z >> 30;
                            s1[k] = y * (y * selB + selA) + selC;
#if SPINFER_ABLATION == 1
                            const uint32_t a = vsm_gt + 2u * c2 - 4u;
                            t0[k] = lds_u16(a);
                            t1[k] = lds_u16(a + 2u);
#else
                            t0[k] = __ldg(gv + (c2 >= 2u ? c2 - 2u : 0u));
                            t1[k] = __ldg(gv + (c2 >= 1u ? c2 - 1u : 0u));
#endif
                        }
                        assemble_nv(t0, t1, s1, 2 * hh, bfr);
                    }
#else
#pragma unroll
                    for (int hh = 0; hh < (HALF ? 1 : 2); ++hh) {   // TCTile row pairs (2 hh', 2 hh' + 1)
                        const int hq = HALF ? hw : hh;
                        load_E_nv(tbl_lane_l + (uint32_t)(tc * 16 + hq * 8) * 8u);
                        issue_to(t0, t1, s1);
                        assemble_nv(t0, t1, s1, HALF ? 0 : 2 * hh, bfr);
                    }
#endif
                }
#pragma unroll
                for (int a = 0; a < TRW; ++a)
#pragma unroll
                    for (int b = 0; b < NT; ++b)
                        asm volatile("" : "+f"(acc[a][b][0]), "+f"(acc[a][b][1]), "+f"(acc[a][b][2]), "+f"(acc[a][b][3]) :: "memory");
                __syncwarp();   // table reads done before the next GT's scan rewrites it
                pf.lap(2);
                if (lane == 0) pf.ev(prm.prof, p, warp, i >> 1, 4);
                pf.count(4);
            } else if (lane == 0) {
                atomicOr(prm.ws_err, 2);   // corrupt GT (or poisoned stage): skipped, Y is not valid
            }
            __syncwarp();
            named_bar_arrive(kBarIdSlot0 + slot, 32u * (1u + kOwnW * (uint32_t)(rows * g)));   // the slot's GT owner warps + its producer
            if (lane == 0) pf.st(prm.prof, p, i, 2, true);
            if (lane == 0) pf.ev(prm.prof, p, warp, i >> 1, 5);
        }
        i += tstride;
        slot += (uint32_t)tstride;
        if (slot >= (uint32_t)S) { slot -= (uint32_t)S; ph ^= 1u; }
    }
    // segments after this warp's last stage: close the non-final ones it did not see
    pf.lap(7);
    const int fseg = nseg_total - 1;   // the final segment (reduced below in shared memory)
    if (cur >= 0 && cur < fseg && r < f_rows) seg_close(cur, contrib);
    for (int s2 = cur + 1; s2 < fseg; ++s2) seg_close(s2, false);
    if (cur != fseg) {   // this warp holds nothing of the final segment
#pragma unroll
        for (int a = 0; a < TRW; ++a)
#pragma unroll
            for (int b = 0; b < NT; ++b)
#pragma unroll
                for (int e = 0; e < 4; ++e) acc[a][b][e] = 0.f;
    }
    pf.lap(3);

    // ---------------------------------------------------------------------- final segment
    // All consumer warps are past their last stage, so the ring is free: the 8 warps of each GT
    // row put their partials (row-major) into shared memory and warp m sums rows [8m, 8m + 8)
    // over the 8 partials in warp order. Its shape comes from the reducer-free walk below.
    named_bar_sync(1, 32 * kCWd);
    int frb = 0, frows = 0;
    bool fcomplete = false;
    if (fseg >= 0) {   // the final segment: the last rowblock piece of the CTA's last non-empty part (A, C, M order)
        const int a_end = (u0 % KG) ? min(u1, (u0 / KG + 1) * KG) : u0;
        const int c_beg = (u1 % KG) ? max(a_end, (u1 / KG) * KG) : u1;
        int ps, pe;
        if (a_end < c_beg) { ps = a_end; pe = c_beg; } else if (c_beg < u1) { ps = c_beg; pe = u1; } else { ps = u0; pe = a_end; }
        frb = (pe - 1) / KG;
        frows = min(kRd, MG - kRd * frb);
        fcomplete = max(ps, frb * KG) == frb * KG && pe == (frb + 1) * KG;
    }
    if (fseg >= 0 && r < frows) {
        // half mode: the two halves of GT slot jm share one 64 x Np buffer (rows 32 hw ..)
        const uint32_t mine = ring + (uint32_t)(r * kSlotW + jm) * (64u * Np * 4u) + (uint32_t)(32 * hw * Np * 4);
#pragma unroll
        for (int tr = 0; tr < TRW; ++tr)
#pragma unroll
            for (int nt = 0; nt < NT; ++nt) {
                const uint32_t row = tr * 16 + (lane >> 2), col = nt * 8 + 2 * (lane & 3);
                sts_v2(mine + (row * Np + col) * 4u, __float_as_uint(acc[tr][nt][0]), __float_as_uint(acc[tr][nt][1]));
                sts_v2(mine + ((row + 8) * Np + col) * 4u, __float_as_uint(acc[tr][nt][2]), __float_as_uint(acc[tr][nt][3]));
            }
    }
    named_bar_sync(1, 32 * kCWd);
    if (fseg >= 0 && r < frows) {
        constexpr int NC = Np / 4;   // outputs per lane: 8 rows x Np columns per warp
        constexpr int NC4 = NC > 4 ? 4 : NC;   // per store
        const int row = 8 * m + (lane >> 2), col0 = NC * (lane & 3);
        float v[NC];
#pragma unroll
        for (int c = 0; c < NC; ++c) v[c] = 0.f;
        for (int m2 = 0; m2 < kSlotW; ++m2) {   // warp order; warps without a GT of the segment hold +0
            const uint32_t a = ring + (uint32_t)(r * kSlotW + m2) * (64u * Np * 4u) + (uint32_t)(row * Np + col0) * 4u;
            if constexpr (NC >= 4) {
#pragma unroll
                for (int q = 0; q < NC / 4; ++q) {
                    const float4 w = lds_f4(a + 16u * q);
                    v[4 * q] += w.x; v[4 * q + 1] += w.y; v[4 * q + 2] += w.z; v[4 * q + 3] += w.w;
                }
            } else {
                const uint2 w = lds_v2(a);
                v[0] += __uint_as_float(w.x); v[1] += __uint_as_float(w.y);
            }
        }
        const int grow = kRd * frb + r;
        if (fcomplete) {
#pragma unroll
            for (int q = 0; q < NC / NC4; ++q) {
                float vq[NC4];
#pragma unroll
                for (int c = 0; c < NC4; ++c) vq[c] = v[NC4 * q + c];
                store_cols<NT, EPI, NC4>(prm, grow * 64 + row, col0 + NC4 * q, vq);
            }
        } else {
            const int pfirst = uowner(frb * KG, prm.U, prm.P);
            float *dst = prm.ws_cta + ((size_t)grow * prm.cslots + (p - pfirst)) * (64 * Np) + row * Np + col0;
            if constexpr (NC >= 4) {
#pragma unroll
                for (int q = 0; q < NC / 4; ++q)
                    stg_f4(reinterpret_cast<float4 *>(dst) + q, make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]));
            } else {
                stg_f2(dst, v[0], v[1]);
            }
        }
    }
    if (fseg >= 0 && !fcomplete) {
        named_bar_sync(2, 32 * kCWd);   // every warp's slice of the CTA partial is stored
        int nparts = 0;
        if (m == 0 && r < frows) {
            const bool last = cta_arrive(prm, frb, kRd * frb + r, lane, nparts);
            if (lane == 0) sts_u32(sbase + kFinFlag + 4 * r, last ? (uint32_t)nparts : 0u);
        }
        named_bar_sync(1, 32 * kCWd);
        // the last CTA of the rowblock: the row's warps sum 32 float4 columns each (all in flight)
        nparts = (int)lds_u32(sbase + kFinFlag + 4 * r);
        if (nparts && r < frows && m * 32 * JC < kF4) cta_sum<NT, EPI, JC>(prm, kRd * frb + r, nparts, m * 32 * JC, lane);
    }
    // cross-CTA sums of non-final segments whose last contributor was this CTA (the reducer's list):
    // GT row e is summed by the 8 warps of consumer row e % 2
    named_bar_sync(kBarIdDefer, 32u * (kCWd + 1));
    const int ndef = (int)lds_u32(sbase + kDefer);
    for (int e = r; e < ndef; e += kRd) {
        const uint32_t d = lds_u32(sbase + kDefer + 4 + 4 * e);
        if (m * 32 * JC < kF4) cta_sum<NT, EPI, JC>(prm, (int)(d & 0xFFFFu), (int)(d >> 16), m * 32 * JC, lane);
    }
    pf.lap(3);
    if (lane == 0) pf.gt(prm.prof, p, 1);
    pf.mark(6);
    pf.dump(prm.prof, p, warp, lane);
}

inline uint32_t al(uint32_t x, uint32_t a) { return (x + a - 1) / a * a; }

struct DPlan {
    int P, G, S;
    size_t smem;
    DParams prm;
};

// CTA partial slots per GT row: the most CTAs one rowblock can overlap.
int cta_slots(long long U, int P, int KG) {
    const long long upc_min = std::max(1LL, U / P);
    return (int)((KG + upc_min - 1) / upc_min + 1);
}

// Ring sizing: each slot holds the X slab (1024-aligned for the swizzle), both GT rows'
// bitmaps and value capacity G * max_gt_values.
bool make_dplan(int M, int K, int Np, int max_gt_values, DPlan *pl) {
    const int MG = (M + kGT - 1) / kGT, KG = (K + kGT - 1) / kGT;
    if (KG > 65535 || MG >= kErrWord) return false;
    const long long U = (long long)((MG + kRd - 1) / kRd) * KG;
    const int P = choose_grid_rb((MG + kRd - 1) / kRd, KG);
    if ((unsigned long long)U * (unsigned long long)P >= (1ull << 32)) return false;
    const int smem_max = smem_optin();
    int maxv = max_gt_values > 0 ? max_gt_values : 4096;
    maxv = std::min(4096, (maxv + 7) & ~7);
    int gmax = kMaxGd, smax = kMaxSd;
    if (option(SPINFER_OPT_STAGE_G) > 0) gmax = std::max(1, std::min(kMaxGd, option(SPINFER_OPT_STAGE_G)));
    if (option(SPINFER_OPT_STAGE_S) > 0) smax = std::max(2, std::min(kMaxSd, option(SPINFER_OPT_STAGE_S)));
    const int wslots = Np > 16 ? 4 : 8;   // GT slots per GT row (half mode, Np = 32: two warps per GT)
    const uint32_t final_scratch = 2u * wslots * 64u * Np * 4u;   // the final segment's partials reuse the ring
    // G in {4, 2, 1} (wslots / G consumer phases keep all 8 warps of a GT row busy); the largest
    // G with >= 4 slots, else the deepest valid ring. A ring needs >= wslots / G slots (one stop
    // sentinel per phase) and an even slot count (producer q always refills its own stages'
    // slots: the slot release barrier counts the GT owners of the stage it issued there).
    int bestG = 0, bestS = 0;
    for (int G = gmax >= 4 ? 4 : gmax >= 2 ? 2 : 1; G >= 1; G >>= 1) {
        const uint32_t st_bm = al((uint32_t)G * 64 * Np * 2, 128);
        const uint32_t vcap = al((uint32_t)G * maxv * 2, 128);
        const uint32_t slot = al(st_bm + kRd * G * 512 + 2 * vcap, 1024);
        const int S = (int)std::min<long long>(smax, ((long long)smem_max - kOffRing - 1024) / slot) & ~1;
        if ((uint32_t)S * slot < final_scratch || S < std::max(2, wslots / G)) continue;
        if (S >= 4) { bestG = G; bestS = S; break; }
        if (S > bestS) { bestG = G; bestS = S; }
    }
    if (bestG == 0) return false;
    const int G = bestG, S = bestS;
    DParams &q = pl->prm;
    q.KG = KG; q.MG = MG; q.M = M; q.U = (uint32_t)U; q.P = P; q.G = G; q.S = S;
    q.st_bm = al((uint32_t)G * 64 * Np * 2, 128);
    q.vcap = al((uint32_t)G * maxv * 2, 128);
    q.st_v0 = q.st_bm + kRd * G * 512;
    q.st_v1 = q.st_v0 + q.vcap;
    q.slot_bytes = al(q.st_v1 + q.vcap, 1024);
    q.cslots = cta_slots(U, P, KG);
    pl->P = P; pl->G = G; pl->S = S;
    pl->smem = (size_t)kOffRing + (size_t)S * q.slot_bytes + 1024;
    return true;
}

template <int NT, bool EPI>
int launch_dw(const DPlan &pl, cudaStream_t st) {
    static int configured[64] = {0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    if ((int)pl.smem > configured[dev]) {
        if (cudaFuncSetAttribute(k_spmm_dw<NT, EPI>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)pl.smem) != cudaSuccess)
            return SPINFER_ECUDA;
        configured[dev] = (int)pl.smem;
    }
    if (pl.prm.pdl) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3((unsigned)pl.P);
        cfg.blockDim = dim3((unsigned)kThreadsD);
        cfg.dynamicSmemBytes = pl.smem;
        cfg.stream = st;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[0].val.programmaticStreamSerializationAllowed = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        if (cudaLaunchKernelEx(&cfg, k_spmm_dw<NT, EPI>, pl.prm) != cudaSuccess) return SPINFER_ECUDA;
        return SPINFER_OK;
    }
    k_spmm_dw<NT, EPI><<<pl.P, kThreadsD, pl.smem, st>>>(pl.prm);
    return cudaGetLastError() == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
}

// Padded X width of the decoupled-warp kernel: 8, 16, or 32 (half mode, N 17-32)
inline int dw_np(int N) { return N > 16 ? 32 : (N + 7) & ~7; }

struct DwLayout {
    size_t seg, cta, xpad, total;
};
DwLayout dw_layout(int M, int K, int N) {
    const int MG = (M + kGT - 1) / kGT, KG = (K + kGT - 1) / kGT;
    const long long U = (long long)((MG + kRd - 1) / kRd) * KG;
    const int P = choose_grid_rb((MG + kRd - 1) / kRd, KG);
    const int Np = dw_np(N);
    DwLayout l;
    l.seg = (size_t)P * kNSeg * kRd * 8 * 64 * Np * 4;
    l.cta = (size_t)MG * cta_slots(U, P, KG) * 64 * Np * 4;
    l.xpad = (N != Np) ? ((size_t)K * Np * 2 + 255) / 256 * 256 : 0;
    l.total = kCounterRegion + l.seg + l.cta + l.xpad;
    return l;
}

}  // namespace

// Workspace of the decoupled-warp kernel: [CTA counters + error word][warp partials]
// [CTA partials][padded X].
size_t spmm_dw_workspace_bytes(int M, int K, int N) { return dw_layout(M, K, N).total; }

int launch_spmm_dw(const spinfer_tca *T, const uint16_t *X, uint16_t *Y, int M, int K, int N, const uint16_t *bias,
                   int act, void *ws, size_t ws_bytes, cudaStream_t st, uint16_t *const *ypeer, int npeer) {
    if (N < 1 || N > 32) return SPINFER_EINVAL;
    const int Np = dw_np(N);
    DPlan pl;
    if (!make_dplan(M, K, Np, T->max_gt_values, &pl)) return SPINFER_EINVAL;
    const DwLayout lay = dw_layout(M, K, N);
    if (ws == nullptr || ws_bytes < lay.total) return SPINFER_ENOSPC;
    DParams &q = pl.prm;
    uint8_t *w8 = reinterpret_cast<uint8_t *>(ws);
    const uint16_t *Xk = X;
    if (N != Np) {
        uint16_t *Xp = reinterpret_cast<uint16_t *>(w8 + kCounterRegion + lay.seg + lay.cta);
        if (int rc = launch_pad_x(X, Xp, K, N, Np, st)) return rc;
        Xk = Xp;
    }
    if (int rc = make_x_tmap(&q.tmap_x, Xk, K, Np, Np, 64 * pl.G, true)) return rc;
    q.K = K;
    q.off = T->gtile_offset;
    q.bm = T->bitmap;
    q.vals = T->values;
    q.Y = Y;
    q.bias = bias;
    q.act = act;
    q.N = N;
    q.ws_cnt = reinterpret_cast<int32_t *>(w8);
    q.ws_err = reinterpret_cast<int32_t *>(w8) + kErrWord;
    q.ws_seg = reinterpret_cast<float *>(w8 + kCounterRegion);
    q.ws_cta = reinterpret_cast<float *>(w8 + kCounterRegion + lay.seg);
    q.n_values = (int)T->n_values;
    q.avg_gt = (float)((double)T->n_values / ((double)q.MG * (double)q.KG));
    q.prof = nullptr;
    q.pdl = option(SPINFER_OPT_PDL) ? 1 : 0;
    if (npeer < 0 || npeer > kMaxPeers || (npeer && !ypeer)) return SPINFER_EINVAL;
    q.npeer = npeer;
    for (int d = 0; d < kMaxPeers; ++d) q.ypeer[d] = d < npeer ? ypeer[d] : nullptr;
    const bool epi = bias != nullptr || act != SPINFER_ACT_NONE || (M % kGT) != 0 || N != Np;
    auto go = [&]() {
        if (Np == 8) return epi ? launch_dw<1, true>(pl, st) : launch_dw<1, false>(pl, st);
        if (Np == 32) return epi ? launch_dw<4, true>(pl, st) : launch_dw<4, false>(pl, st);
        return epi ? launch_dw<2, true>(pl, st) : launch_dw<2, false>(pl, st);
    };
#if SPINFER_INSTRUMENT
    if (const char *path = getenv("SPINFER_PROF")) {   // experiments: dump per-warp cycle counters
        static long long *prof_buf = nullptr;
        const size_t n = kSmidOff + 1024;
        if (!prof_buf && cudaMalloc(&prof_buf, n * 8) != cudaSuccess) return SPINFER_ECUDA;
        cudaMemsetAsync(prof_buf, 0, n * 8, st);
        q.prof = prof_buf;
        const int rc = go();
        long long *host = (long long *)malloc(n * 8);
        cudaMemcpyAsync(host, prof_buf, n * 8, cudaMemcpyDeviceToHost, st);
        cudaStreamSynchronize(st);
        if (FILE *f = fopen(path, "wb")) { fwrite(host, 8, n, f); fclose(f); }
        free(host);
        return rc;
    }
#endif
    return go();
}

}  // namespace spinfer
