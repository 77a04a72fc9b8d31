// spmm.cu — host side of the SpMM: kernel choice, workspace sizing, the X tensor map, the
// zero-padded X copy, and the library options (include/spinfer.h spinfer_set_option).
//   N <= 16: the decoupled-warp mma.sync kernel (spmm_dw.cu);
//   N 17..32: the tcgen05 kernel (spmm_tc.cu), accumulators in TMEM;
//   N > 32: the wide (prefill) tcgen05 kernel (spmm_wide.cu), W decoded into shared memory.
#include <cuda.h>   // CUtensorMap (type + enums only; the encoder comes via cudaGetDriverEntryPoint)
#include <algorithm>
#include <atomic>
#include "internal.cuh"

namespace spinfer {
namespace {

std::atomic<int> g_options[SPINFER_OPT_COUNT];

int num_sms() {
    int dev = 0, n = kNumSMsDefault;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    cudaGetLastError();
    return n > 0 ? n : kNumSMsDefault;
}

// cuTensorMapEncodeTiled through the runtime's driver entry point (no libcuda link).
using EncodeTiledFn = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                   const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

// X [K][Np] -> Xp [K][Np] with zero columns N..Np-1 (N not a multiple of 8)
__global__ void k_pad_x(const uint16_t *__restrict__ X, uint16_t *__restrict__ Xp, int K, int N, int Np) {
    const long long tot = (long long)K * Np;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < tot; i += (long long)gridDim.x * blockDim.x) {
        const int k = (int)(i / Np), n = (int)(i - (long long)k * Np);
        Xp[i] = n < N ? X[(size_t)k * N + n] : (uint16_t)0;
    }
}

}  // namespace

int option(int key) { return (key >= 0 && key < SPINFER_OPT_COUNT) ? g_options[key].load(std::memory_order_relaxed) : 0; }
int set_option(int key, int value) {
    if (key < 0 || key >= SPINFER_OPT_COUNT || value < 0) return SPINFER_EINVAL;
    if (key == SPINFER_OPT_KERNEL && value > SPINFER_KERNEL_TC) return SPINFER_EINVAL;
    g_options[key].store(value, std::memory_order_relaxed);
    return SPINFER_OK;
}

int sm_count() {
    static int cached[64] = {0};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) { cudaGetLastError(); return num_sms(); }
    if (!cached[dev]) cached[dev] = num_sms();
    return cached[dev];
}

// Persistent grid: one CTA per SM (SPINFER_OPT_MAX_CTAS caps it: tests force split rowblocks).
int choose_grid(long long units) {
    long long cap = sm_count();
    const int mc = option(SPINFER_OPT_MAX_CTAS);
    if (mc > 0 && mc < cap) cap = mc;
    return (int)std::max(1LL, std::min(cap, units));
}

// Stream-K grid over RB rowblocks of KG units. With no more rowblocks than SMs, a grid of
// k * RB CTAs (k = SMs / RB) puts every CTA boundary on a k-th of a rowblock: each CTA works on
// one rowblock (one segment, at most k partials to combine) instead of straddling two. Taken
// when it keeps >= 80 % of the SMs busy (measured: OPT-13B O 5120^2 32.8 -> 24.6 us with 120
// CTAs, QKV 15360x5120 43.0 -> 38.9 us).
int choose_grid_rb(long long RB, long long KG) {
    const long long units = RB * KG;
    const int P = choose_grid(units);
    if (RB <= 0 || RB > P || option(SPINFER_OPT_MAX_CTAS) > 0) return P;
    const long long k = std::min<long long>(P / RB, KG);
    const long long Pa = k * RB;
    return (Pa * 5 >= (long long)P * 4) ? (int)Pa : P;
}

// X [K][N] fp16 row-major as a 2-D tensor map, box {box_n, box_k}; box columns past N and rows
// past K are zero-filled by the TMA (X padded to the MMA's N without a copy).
int make_x_tmap_box(CUtensorMap *m, const uint16_t *X, int K, int N, int box_n, int box_k, CUtensorMapSwizzle sw) {
    // the last few encodings per host thread (decode loops call with the same X buffers)
    struct Entry { const uint16_t *X; int K, N, box_n, box_k, sw; CUtensorMap map; };
    static thread_local Entry cache[8];
    static thread_local int next = 0;
    for (const Entry &e : cache)
        if (e.X == X && X && e.K == K && e.N == N && e.box_n == box_n && e.box_k == box_k && e.sw == (int)sw) {
            *m = e.map;
            return SPINFER_OK;
        }
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
    const cuuint32_t box[2] = {(cuuint32_t)box_n, (cuuint32_t)box_k};
    const cuuint32_t estr[2] = {1u, 1u};
    CUresult r = fn(m, CU_TENSOR_MAP_DATA_TYPE_UINT16, 2, const_cast<uint16_t *>(X), dims, strides, box, estr,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return SPINFER_EINVAL;
    cache[next] = Entry{X, K, N, box_n, box_k, (int)sw, *m};
    next = (next + 1) % 8;
    return SPINFER_OK;
}

// Opt-in shared memory per block of the current device (cached).
int smem_optin() {
    static std::atomic<int> cached[64];
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev >= 0 && dev < 64) {
        const int v = cached[dev].load(std::memory_order_relaxed);
        if (v) return v;
    }
    int v = 232448;
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev) != cudaSuccess) {
        cudaGetLastError();
        v = 232448;
    }
    if (dev >= 0 && dev < 64) cached[dev].store(v, std::memory_order_relaxed);
    return v;
}

// The narrow kernels' X slab: box {NX, box_rows}; 32B / 64B swizzle = the ldmatrix / MMA-descriptor
// bank-conflict-free layouts of a 16 / 32 column slab.
int make_x_tmap(CUtensorMap *m, const uint16_t *X, int K, int N, int NX, int box_rows, bool swizzle) {
    const CUtensorMapSwizzle sw = !swizzle ? CU_TENSOR_MAP_SWIZZLE_NONE
                                  : NX == 16 ? CU_TENSOR_MAP_SWIZZLE_32B : NX == 32 ? CU_TENSOR_MAP_SWIZZLE_64B
                                                                                 : CU_TENSOR_MAP_SWIZZLE_NONE;
    return make_x_tmap_box(m, X, K, N, NX, box_rows, sw);
}

int launch_pad_x(const uint16_t *X, uint16_t *Xp, int K, int N, int Np, cudaStream_t st) {
    const long long tot = (long long)K * Np;
    k_pad_x<<<(int)std::min<long long>((tot + 255) / 256, 4096), 256, 0, st>>>(X, Xp, K, N, Np);
    return cudaGetLastError() == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
}

// The workspace serves whichever kernel a call picks: the largest of their layouts.
size_t spmm_workspace_bytes(int M, int K, int N) {
    if (M <= 0 || K <= 0 || N <= 0 || N > kMaxN || (M + kGT - 1) / kGT >= kErrWord) return 0;
    if (N > 32) return spmm_wide_workspace_bytes(M, K, N);
    const size_t tc = spmm_tc_workspace_bytes(M, K, N);
    const size_t dw = N <= 32 ? spmm_dw_workspace_bytes(M, K, N) : 0;
    return std::max(tc, dw);
}

int launch_spmm(const spinfer_tca *T, const uint16_t *X, uint16_t *Y, int M, int K, int N, const uint16_t *bias, int act,
                void *ws, size_t ws_bytes, cudaStream_t st) {
    // Kernel choice by N, from the B200 measurements: the decoupled-warp mma.sync
    // kernel for N <= 16, the tcgen05 kernel for N > 16 (N not a multiple of 8 computes the next
    // multiple of 8 and stores the N real columns). SPINFER_OPT_KERNEL overrides (tests, ablation).
    const int Np = (N + 7) & ~7;
    if (Np > 32) return launch_spmm_wide(T, X, Y, M, K, N, bias, act, ws, ws_bytes, st);
    const int ko = option(SPINFER_OPT_KERNEL);
    const bool dw = ko == SPINFER_KERNEL_DW ? true : ko == SPINFER_KERNEL_TC ? false : Np <= 16;
    if (dw && Np > 32) return SPINFER_EINVAL;
    if (dw) return launch_spmm_dw(T, X, Y, M, K, N, bias, act, ws, ws_bytes, st);
    return launch_spmm_tc(T, X, Y, M, K, N, bias, act, ws, ws_bytes, st);
}

}  // namespace spinfer
