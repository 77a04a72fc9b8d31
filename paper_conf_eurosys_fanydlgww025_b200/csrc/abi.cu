// abi.cu — the extern "C" boundary declared in include/spinfer.h: argument
// validation, status codes, and dispatch to the sm_100a kernels.
#include <atomic>
#include <cstring>
#include "internal.cuh"

namespace spinfer {

int check_device() {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return SPINFER_ENODEV; }
    static std::atomic<int> verdict[64];   // per device: 0 unknown, 1 sm_100, 2 other (host cost per call)
    if (dev >= 0 && dev < 64) {
        const int v = verdict[dev].load(std::memory_order_relaxed);
        if (v) return v == 1 ? SPINFER_OK : SPINFER_ENODEV;
    }
    int major = 0, minor = 0;
    if (cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev) != cudaSuccess ||
        cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev) != cudaSuccess) {
        cudaGetLastError();
        return SPINFER_ENODEV;
    }
    const bool ok = major == 10 && minor == 0;   // built for sm_100a only
    if (dev >= 0 && dev < 64) verdict[dev].store(ok ? 1 : 2, std::memory_order_relaxed);
    return ok ? SPINFER_OK : SPINFER_ENODEV;
}

// any M, K > 0: shapes that are not multiples of 64 are zero-padded to whole GroupTiles (A8)
static bool shape_ok(int M, int K) { return M > 0 && K > 0; }

int validate_tca(const spinfer_tca *T, int M, int K) {
    if (!T || !T->gtile_offset || !T->bitmap || !T->values) return SPINFER_EINVAL;
    if (T->M != M || T->K != K || T->gt_h != kGT || T->gt_w != kGT || !shape_ok(M, K)) return SPINFER_EINVAL;
    if (T->n_values < 0) return SPINFER_EINVAL;
    if (T->n_values >= (1LL << 31)) return SPINFER_EOVERFLOW;
    if (T->max_gt_values > kGT * kGT) return SPINFER_EINVAL;
    if (!aligned16(T->gtile_offset) || !aligned16(T->bitmap) || !aligned16(T->values)) return SPINFER_EINVAL;
    return SPINFER_OK;
}

}  // namespace spinfer

using namespace spinfer;

extern "C" {

int spinfer_encode_count(const uint16_t *W, int M, int K, int32_t *gtile_offset, int64_t *n_values, int64_t *nnz,
                         int32_t *max_gt_values, void *stream) {
    if (!W || !gtile_offset || !n_values || !nnz || !shape_ok(M, K) || !aligned16(W)) return SPINFER_EINVAL;
    int rc = check_device();
    if (rc) return rc;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    void *tmp = nullptr;
    if (cudaMallocAsync(&tmp, 64, st) != cudaSuccess) { cudaGetLastError(); return SPINFER_ECUDA; }
    int64_t stats[8] = {0};
    rc = SPINFER_ECUDA;
    if (cudaMemsetAsync(tmp, 0, 64, st) == cudaSuccess) {
        rc = launch_encode_count(W, M, K, gtile_offset, reinterpret_cast<int64_t *>(tmp), st);
        if (rc == SPINFER_OK) {
            if (cudaMemcpyAsync(stats, tmp, 64, cudaMemcpyDeviceToHost, st) != cudaSuccess ||
                cudaStreamSynchronize(st) != cudaSuccess)
                rc = SPINFER_ECUDA;
        }
    }
    cudaFreeAsync(tmp, st);
    if (rc) { cudaGetLastError(); return rc; }
    if (stats[2] >= (1LL << 31)) return SPINFER_EOVERFLOW;
    *nnz = stats[0];
    *n_values = stats[2];
    if (max_gt_values) *max_gt_values = (int32_t)stats[1];
    return SPINFER_OK;
}

int spinfer_encode_fill(const uint16_t *W, const spinfer_tca *T, void *stream) {
    if (!W || !aligned16(W) || !T) return SPINFER_EINVAL;
    int rc = validate_tca(T, T->M, T->K);
    if (rc) return rc;
    if ((rc = check_device())) return rc;
    return launch_encode_fill(W, T, reinterpret_cast<cudaStream_t>(stream));
}

int spinfer_decode(const spinfer_tca *T, uint16_t *W_out, void *stream) {
    if (!T || !W_out || !aligned16(W_out)) return SPINFER_EINVAL;
    int rc = validate_tca(T, T->M, T->K);
    if (rc) return rc;
    if ((rc = check_device())) return rc;
    return launch_decode(T, W_out, reinterpret_cast<cudaStream_t>(stream));
}

size_t spinfer_spmm_workspace_bytes(int M, int K, int N) {
    if (!shape_ok(M, K) || N < 1 || N > kMaxN) return 0;
    return spmm_workspace_bytes(M, K, N);
}

int spinfer_spmm_ex(const spinfer_tca *T, const uint16_t *X, uint16_t *Y, int M, int K, int N,
                    const uint16_t *bias, int act, void *workspace, size_t ws_bytes, void *stream) {
    if (!X || !Y || N < 1 || N > kMaxN) return SPINFER_EINVAL;
    if (act != SPINFER_ACT_NONE && act != SPINFER_ACT_RELU) return SPINFER_EINVAL;
    if (bias && (reinterpret_cast<uintptr_t>(bias) & 1u)) return SPINFER_EINVAL;
    if (!aligned16(X) || !aligned16(Y) || (workspace && !aligned16(workspace))) return SPINFER_EINVAL;
    int rc = validate_tca(T, M, K);
    if (rc) return rc;
    if ((rc = check_device())) return rc;
    return launch_spmm(T, X, Y, M, K, N, bias, act, workspace, ws_bytes, reinterpret_cast<cudaStream_t>(stream));
}

int spinfer_spmm(const spinfer_tca *T, const uint16_t *X, uint16_t *Y, int M, int K, int N, void *workspace,
                 size_t ws_bytes, void *stream) {
    return spinfer_spmm_ex(T, X, Y, M, K, N, nullptr, SPINFER_ACT_NONE, workspace, ws_bytes, stream);
}

int spinfer_tp_rows(int M, int world, int rank, int *row_begin, int *row_count) {
    if (!row_begin || !row_count || M <= 0 || world <= 0 || rank < 0 || rank >= world)
        return SPINFER_EINVAL;
    const int MG = (M + kGT - 1) / kGT, q = MG / world, rem = MG % world;
    int b = (rank * q + (rank < rem ? rank : rem)) * kGT;
    int c = (q + (rank < rem ? 1 : 0)) * kGT;
    if (b > M) b = M;                  // A8: the ragged tail belongs to the rank owning the last GT row
    if (b + c > M) c = M - b;
    *row_begin = b;
    *row_count = c;
    return SPINFER_OK;
}

int spinfer_tca_shard(const spinfer_tca *T, int row_begin, int row_count, int32_t *offset_out, spinfer_tca *out,
                      void *stream) {
    if (!T || !out || !offset_out) return SPINFER_EINVAL;
    int rc = validate_tca(T, T->M, T->K);
    if (rc) return rc;
    if (row_begin < 0 || row_count <= 0 || row_begin % kGT || row_begin + row_count > T->M ||
        (row_count % kGT && row_begin + row_count != T->M) || !aligned16(offset_out))
        return SPINFER_EINVAL;
    if ((rc = check_device())) return rc;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    const int64_t KG = (T->K + kGT - 1) / kGT;
    const int64_t a = row_begin / kGT, b = (row_begin + row_count + kGT - 1) / kGT;
    int32_t ends[2] = {0, 0};
    if (cudaMemcpyAsync(&ends[0], T->gtile_offset + a * KG, 4, cudaMemcpyDeviceToHost, st) != cudaSuccess ||
        cudaMemcpyAsync(&ends[1], T->gtile_offset + b * KG, 4, cudaMemcpyDeviceToHost, st) != cudaSuccess ||
        launch_rebase_offsets(T->gtile_offset, a * KG, (b - a) * KG, offset_out, st) != SPINFER_OK ||
        cudaStreamSynchronize(st) != cudaSuccess) {
        cudaGetLastError();
        return SPINFER_ECUDA;
    }
    if (ends[0] < 0 || ends[1] < ends[0] || ends[1] > T->n_values || ends[0] % 8) return SPINFER_EINVAL;
    spinfer_tca o = *T;
    o.M = row_count;
    o.nnz = -1;
    o.n_values = ends[1] - ends[0];
    o.gtile_offset = offset_out;
    o.bitmap = T->bitmap + a * KG * 64;
    o.values = T->values + ends[0];
    *out = o;
    return SPINFER_OK;
}

int spinfer_spmm_tp(const spinfer_tca *T_shard, const uint16_t *X, uint16_t *Y_full, int M_full, int K, int N,
                    int world, int rank, void *workspace, size_t ws_bytes, void *stream) {
    int b = 0, c = 0;
    int rc = spinfer_tp_rows(M_full, world, rank, &b, &c);
    if (rc) return rc;
    if (!T_shard || !Y_full) return SPINFER_EINVAL;
    if (T_shard->M != c) return SPINFER_EINVAL;
    if (c == 0) return SPINFER_OK;   // rank owns no rows (more ranks than GT rows)
    return spinfer_spmm(T_shard, X, Y_full + (size_t)b * N, c, K, N, workspace, ws_bytes, stream);
}

int spinfer_spmm_tp_gather(const spinfer_tca *T_shard, const uint16_t *X, uint16_t *const *Y_full_peers, int M_full,
                           int K, int N, int world, int rank, uint32_t *const *flag_peers, void *workspace,
                           size_t ws_bytes, void *stream) {
    int b = 0, c = 0;
    int rc = spinfer_tp_rows(M_full, world, rank, &b, &c);
    if (rc) return rc;
    if (!T_shard || !X || !Y_full_peers || !flag_peers || world > kMaxPeers || N < 1 || ((N + 7) & ~7) > 16)
        return SPINFER_EINVAL;
    for (int r = 0; r < world; ++r)
        if (!Y_full_peers[r] || !flag_peers[r] || !aligned16(Y_full_peers[r])) return SPINFER_EINVAL;
    if ((rc = check_device())) return rc;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    if (c > 0) {
        if (T_shard->M != c || !aligned16(X) || (workspace && !aligned16(workspace))) return SPINFER_EINVAL;
        if ((rc = validate_tca(T_shard, c, K))) return rc;
        uint16_t *ypeer[kMaxPeers];
        for (int r = 0; r < world; ++r) ypeer[r] = Y_full_peers[r] + (size_t)b * N;
        if ((rc = launch_spmm_dw(T_shard, X, ypeer[rank], c, K, N, nullptr, SPINFER_ACT_NONE, workspace, ws_bytes, st,
                                 ypeer, world)))
            return rc;
    }
    return launch_gather_signal(flag_peers, world, st);
}

int spinfer_gather_wait(uint32_t *flag, uint32_t *state, int world, void *workspace, uint32_t timeout_us, void *stream) {
    if (!flag || !state || world < 1 || world > kMaxPeers) return SPINFER_EINVAL;
    int rc = check_device();
    if (rc) return rc;
    int32_t *err = workspace ? reinterpret_cast<int32_t *>(workspace) + kErrWord : nullptr;
    return launch_gather_wait(flag, state, world, err, timeout_us, reinterpret_cast<cudaStream_t>(stream));
}

int spinfer_spmm_check(void *workspace, int32_t *flags, void *stream) {
    if (!workspace || !flags || !aligned16(workspace)) return SPINFER_EINVAL;
    int rc = check_device();
    if (rc) return rc;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    int32_t *err = reinterpret_cast<int32_t *>(workspace) + kErrWord;
    if (cudaMemcpyAsync(flags, err, 4, cudaMemcpyDeviceToHost, st) != cudaSuccess ||
        cudaMemsetAsync(err, 0, 4, st) != cudaSuccess || cudaStreamSynchronize(st) != cudaSuccess) {
        cudaGetLastError();
        return SPINFER_ECUDA;
    }
    return SPINFER_OK;
}

int spinfer_set_option(int key, int value) { return set_option(key, value); }
int spinfer_get_option(int key) { return option(key); }

const char *spinfer_status_str(int status) {
    switch (status) {
        case SPINFER_OK: return "SPINFER_OK";
        case SPINFER_EINVAL: return "SPINFER_EINVAL: invalid argument";
        case SPINFER_ENOSPC: return "SPINFER_ENOSPC: workspace too small";
        case SPINFER_EOVERFLOW: return "SPINFER_EOVERFLOW: n_values >= 2^31";
        case SPINFER_ECUDA: return "SPINFER_ECUDA: CUDA error";
        case SPINFER_ENODEV: return "SPINFER_ENODEV: device is not sm_100";
        default: return "SPINFER: unknown status";
    }
}

const char *spinfer_version(void) { return "spinfer-b200 0.2 (sm_100a; TCA-BME GT=64; SMBD: mma.sync N<=16, tcgen05 N 17-32, tcgen05 wide N>32)"; }

}  // extern "C"
