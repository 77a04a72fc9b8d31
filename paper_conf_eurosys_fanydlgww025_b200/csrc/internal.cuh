// internal.cuh — declarations shared by the library's translation units.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>
#include "spinfer.h"

namespace spinfer {

constexpr int kGT = 64;    // GroupTile edge (reading A1)
constexpr int kNumSMsDefault = 148;
constexpr int kMaxN = 65536;
constexpr int kMaxPeers = 8;             // fused all-gather: ranks of one NVLink domain             // widest X (TMA coordinates and the wide kernel's tiling)

int check_device();        // SPINFER_OK or SPINFER_ENODEV / SPINFER_ECUDA
inline bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }
int validate_tca(const spinfer_tca *T, int M, int K);

// encode.cu
int launch_encode_count(const uint16_t *W, int M, int K, int32_t *gtile_offset, int64_t *stats_dev,
                        cudaStream_t st);
int launch_encode_fill(const uint16_t *W, const spinfer_tca *T, cudaStream_t st);
int launch_decode(const spinfer_tca *T, uint16_t *W_out, cudaStream_t st);
int launch_rebase_offsets(const int32_t *off, int64_t g0, int64_t n, int32_t *out, cudaStream_t st);

// Workspace head shared by the SpMM kernels: int32 GT-row counters [0, kErrWord) and, at word
// kErrWord, the error word (non-zero after a call that met corrupt TCA-BME input).
constexpr size_t kCounterRegion = 65536;
constexpr int kErrWord = 16383;

// spmm.cu
int option(int key);                     // spinfer_set_option values (0 = default)
int set_option(int key, int value);
int sm_count();                          // SMs of the current device (cached per device)
int smem_optin();                        // opt-in shared memory per block of the current device (cached)
int choose_grid(long long units);        // persistent grid size: min(SMs, units)
int choose_grid_rb(long long RB, long long KG);   // stream-K grid aligned to rowblocks when that pays
int make_x_tmap(CUtensorMap *m, const uint16_t *X, int K, int N, int NX, int box_rows, bool swizzle);
int make_x_tmap_box(CUtensorMap *m, const uint16_t *X, int K, int N, int box_n, int box_k, CUtensorMapSwizzle sw);
int launch_pad_x(const uint16_t *X, uint16_t *Xp, int K, int N, int Np, cudaStream_t st);
size_t spmm_workspace_bytes(int M, int K, int N);
int launch_spmm(const spinfer_tca *T, const uint16_t *X, uint16_t *Y, int M, int K, int N, const uint16_t *bias, int act, void *ws,
                size_t ws_bytes, cudaStream_t st);

// spmm_wide.cu (tcgen05 kernel with W decoded into shared memory, N > 32)
size_t spmm_wide_workspace_bytes(int M, int K, int N);
int launch_spmm_wide(const spinfer_tca *T, const uint16_t *X, uint16_t *Y, int M, int K, int N, const uint16_t *bias,
                     int act, void *ws, size_t ws_bytes, cudaStream_t st);

// spmm_tc.cu (tcgen05 kernel, N 17..32)
size_t spmm_tc_workspace_bytes(int M, int K, int N);
int launch_spmm_tc(const spinfer_tca *T, const uint16_t *X, uint16_t *Y, int M, int K, int N, const uint16_t *bias,
                   int act, void *ws, size_t ws_bytes, cudaStream_t st);

// spmm_dw.cu (decoupled-warp kernel, N <= 16)
size_t spmm_dw_workspace_bytes(int M, int K, int N);
int launch_spmm_dw(const spinfer_tca *T, const uint16_t *X, uint16_t *Y, int M, int K, int N, const uint16_t *bias,
                   int act, void *ws, size_t ws_bytes, cudaStream_t st, uint16_t *const *ypeer = nullptr, int npeer = 0);
// gather.cu (fused all-gather epilogue: peer signalling)
int launch_gather_signal(uint32_t *const *flag_peers, int world, cudaStream_t st);
int launch_gather_wait(uint32_t *flag, uint32_t *state, int world, int32_t *err, uint32_t timeout_us, cudaStream_t st);

}  // namespace spinfer
