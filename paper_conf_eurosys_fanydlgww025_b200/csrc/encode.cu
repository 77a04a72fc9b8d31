// encode.cu — GPU TCA-BME encoder and decoder (§4.2; the
// paper's encoder is an offline "preprocessing" step it does not describe).
//
// Thread mapping (all three kernels): a 256-thread block covers 4 GroupTiles;
// thread t handles BitmapTile bi = t % 64 of GT g = 4*blockIdx.x + t/64, where
// bi is the BT's position in the GT's storage order (TCTile tt = bi/4 column-
// major in the GT; BT b = bi%4 column-major in the TCTile, TL/BL/TR/BR,
// P:192). Bit 8*i + j of the BT's bitmap is element (row i, col j).
// Each thread reads its BT as 8 x 16-byte rows (one uint4 per row).
#include <algorithm>
#include "internal.cuh"

namespace spinfer {
namespace {

constexpr int kGTPerBlock = 4;
constexpr int kThreads = 64 * kGTPerBlock;

struct BtPos {
    int64_t g;      // GroupTile index (row-major)
    int bi;         // BT index in GT storage order (0..63)
    int row0, col0; // top-left element of the BT
};

__device__ __forceinline__ BtPos bt_pos(int KG) {
    BtPos p;
    int t = threadIdx.x;
    p.g = (int64_t)blockIdx.x * kGTPerBlock + (t >> 6);
    p.bi = t & 63;
    int tt = p.bi >> 2, b = p.bi & 3;
    int tr = tt & 3, tc = tt >> 2;   // TCTiles column-major inside the GT
    int br = b & 1, bc = b >> 1;     // BTs column-major inside the TCTile
    int gr = (int)(p.g / KG), gc = (int)(p.g % KG);
    p.row0 = gr * kGT + tr * 16 + br * 8;
    p.col0 = gc * kGT + tc * 16 + bc * 8;
    return p;
}

__device__ __forceinline__ uint32_t nz_byte(uint4 v) {
    // bit j set iff half j of the 8 halves in v is non-zero ((bits & 0x7FFF) != 0, reading A7)
    uint32_t w[4] = {v.x, v.y, v.z, v.w};
    uint32_t m = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        m |= ((w[q] & 0x7FFFu) != 0u) << (2 * q);
        m |= ((w[q] & 0x7FFF0000u) != 0u) << (2 * q + 1);
    }
    return m;
}

// 8 consecutive halves W[r][c0 .. c0+7] of the zero-padded matrix (reading A8): one 16-byte
// load when the row segment is inside W and 16-byte aligned (K % 8 == 0), else element-wise.
__device__ __forceinline__ uint4 row8(const uint16_t *__restrict__ W, int M, int K, int r, int c0) {
    if (r >= M) return make_uint4(0u, 0u, 0u, 0u);
    if ((K & 7) == 0 && c0 + 8 <= K) return __ldg(reinterpret_cast<const uint4 *>(W + (size_t)r * K + c0));
    uint32_t w[4] = {0u, 0u, 0u, 0u};
#pragma unroll
    for (int j = 0; j < 8; ++j)
        if (c0 + j < K) w[j >> 1] |= (uint32_t)__ldg(W + (size_t)r * K + c0 + j) << (16 * (j & 1));
    return make_uint4(w[0], w[1], w[2], w[3]);
}

__device__ __forceinline__ uint64_t bt_bitmap(const uint16_t *__restrict__ W, int M, int K, int row0, int col0) {
    uint64_t bm = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) bm |= (uint64_t)nz_byte(row8(W, M, K, row0 + i, col0)) << (8 * i);
    return bm;
}

// Exclusive prefix of `c` over the 64 threads of one GT (2 warps) + GT total.
__device__ __forceinline__ int gt_exclusive_scan(int c, int *total) {
    __shared__ int wsum[kThreads / 32];
    int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    int x = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) wsum[warp] = x;
    __syncthreads();
    int first = wsum[warp & ~1];
    int excl = x - c + ((warp & 1) ? first : 0);
    *total = first + wsum[warp | 1];
    return excl;
}

__global__ void __launch_bounds__(kThreads) k_encode_count(const uint16_t *__restrict__ W, int M, int K, int KG,
                                                           int64_t NGT, int32_t *__restrict__ padcount,
                                                           unsigned long long *__restrict__ stats) {
    BtPos p = bt_pos(KG);
    int c = 0;
    if (p.g < NGT) c = __popcll(bt_bitmap(W, M, K, p.row0, p.col0));
    int total;
    (void)gt_exclusive_scan(c, &total);
    __shared__ unsigned long long blk_nnz;
    __shared__ int blk_max;
    if (threadIdx.x == 0) { blk_nnz = 0; blk_max = 0; }
    __syncthreads();
    if (p.bi == 0 && p.g < NGT) {
        int padded = (total + 7) & ~7;   // 16-byte aligned GT segments (reading A6)
        padcount[p.g] = padded;
        atomicAdd(&blk_nnz, (unsigned long long)total);
        atomicMax(&blk_max, padded);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        atomicAdd(&stats[0], blk_nnz);
        atomicMax(&stats[1], (unsigned long long)blk_max);
    }
}

// In-place exclusive scan of a[0..n) (padded GT counts) into GTileOffset[0..n],
// a[n] = total. One block; stats[2] = total as int64 (overflow check on host).
__global__ void __launch_bounds__(1024) k_scan_offsets(int32_t *__restrict__ a, int64_t n,
                                                       unsigned long long *__restrict__ stats) {
    __shared__ long long part[32];
    int t = threadIdx.x, lane = t & 31, warp = t >> 5;
    int64_t chunk = (n + 1023) / 1024;
    int64_t lo = min((int64_t)t * chunk, n), hi = min(lo + chunk, n);
    long long s = 0;
    for (int64_t i = lo; i < hi; ++i) s += a[i];
    long long x = s;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        long long y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) part[warp] = x;
    __syncthreads();
    if (warp == 0) {
        long long v = part[lane], w = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            long long y = __shfl_up_sync(0xffffffffu, w, o);
            if (lane >= o) w += y;
        }
        part[lane] = w - v;   // exclusive warp offsets
        if (lane == 31) {
            a[n] = (int32_t)w;
            stats[2] = (unsigned long long)w;
        }
    }
    __syncthreads();
    long long run = part[warp] + x - s;
    for (int64_t i = lo; i < hi; ++i) {
        long long v = a[i];
        a[i] = (int32_t)run;
        run += v;
    }
}

__global__ void __launch_bounds__(kThreads) k_encode_fill(const uint16_t *__restrict__ W, int M, int K, int KG, int64_t NGT,
                                                          const int32_t *__restrict__ off,
                                                          uint64_t *__restrict__ bitmap,
                                                          uint16_t *__restrict__ values) {
    BtPos p = bt_pos(KG);
    bool live = p.g < NGT;
    uint64_t bm = live ? bt_bitmap(W, M, K, p.row0, p.col0) : 0ull;
    int c = __popcll(bm);
    int total;
    int excl = gt_exclusive_scan(c, &total);
    if (!live) return;
    bitmap[p.g * 64 + p.bi] = bm;                 // same nested order as Values (reading A5)
    int64_t pos = (int64_t)off[p.g] + excl;       // BT base = GT offset + PopCount of earlier BTs
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        if (((bm >> (8 * i)) & 0xFFu) == 0) continue;
        uint4 v = row8(W, M, K, p.row0 + i, p.col0);
        uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            uint16_t h = (uint16_t)(w[j >> 1] >> (16 * (j & 1)));
            if ((bm >> (8 * i + j)) & 1ull) values[pos++] = h;   // ascending bit order (reading A3)
        }
    }
    if (p.bi == 63) {                              // +0.0 padding to the next 8-half boundary (A6)
        int64_t end = off[p.g + 1];
        for (int64_t q = (int64_t)off[p.g] + total; q < end; ++q) values[q] = 0;
    }
}

__global__ void __launch_bounds__(kThreads) k_decode(const int32_t *__restrict__ off,
                                                     const uint64_t *__restrict__ bitmap,
                                                     const uint16_t *__restrict__ values, int M, int K, int KG,
                                                     int64_t NGT, uint16_t *__restrict__ W) {
    BtPos p = bt_pos(KG);
    bool live = p.g < NGT;
    uint64_t bm = live ? bitmap[p.g * 64 + p.bi] : 0ull;
    int total;
    int excl = gt_exclusive_scan(__popcll(bm), &total);
    if (!live) return;
    int64_t pos = (int64_t)off[p.g] + excl;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        uint32_t w[4] = {0, 0, 0, 0};
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            if ((bm >> (8 * i + j)) & 1ull) w[j >> 1] |= (uint32_t)values[pos++] << (16 * (j & 1));
        }
        const int r = p.row0 + i;
        if (r >= M) continue;                                  // zero padding is not written (A8)
        if ((K & 7) == 0 && p.col0 + 8 <= K) {
            *reinterpret_cast<uint4 *>(W + (size_t)r * K + p.col0) = make_uint4(w[0], w[1], w[2], w[3]);
        } else {
#pragma unroll
            for (int j = 0; j < 8; ++j)
                if (p.col0 + j < K) W[(size_t)r * K + p.col0 + j] = (uint16_t)(w[j >> 1] >> (16 * (j & 1)));
        }
    }
}

// Row shard (P-E5): out[i] = off[g0 + i] - off[g0], i in [0, n]
__global__ void k_rebase_offsets(const int32_t *__restrict__ off, int64_t g0, int64_t n, int32_t *__restrict__ out) {
    const int32_t base = off[g0];
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = off[g0 + i] - base;
}

}  // namespace

int launch_rebase_offsets(const int32_t *off, int64_t g0, int64_t n, int32_t *out, cudaStream_t st) {
    const int64_t blocks = std::min<int64_t>((n + 1 + 255) / 256, 1024);
    k_rebase_offsets<<<(int)blocks, 256, 0, st>>>(off, g0, n, out);
    return cudaGetLastError() == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
}

int launch_encode_count(const uint16_t *W, int M, int K, int32_t *gtile_offset, int64_t *stats_dev,
                        cudaStream_t st) {
    int KG = (K + kGT - 1) / kGT;
    int64_t NGT = (int64_t)((M + kGT - 1) / kGT) * KG;   // zero-padded to whole GroupTiles (A8)
    int64_t blocks = (NGT + kGTPerBlock - 1) / kGTPerBlock;
    k_encode_count<<<(unsigned)blocks, kThreads, 0, st>>>(W, M, K, KG, NGT, gtile_offset,
                                                          reinterpret_cast<unsigned long long *>(stats_dev));
    k_scan_offsets<<<1, 1024, 0, st>>>(gtile_offset, NGT, reinterpret_cast<unsigned long long *>(stats_dev));
    return cudaGetLastError() == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
}

int launch_encode_fill(const uint16_t *W, const spinfer_tca *T, cudaStream_t st) {
    int KG = (T->K + kGT - 1) / kGT;
    int64_t NGT = (int64_t)((T->M + kGT - 1) / kGT) * KG;
    int64_t blocks = (NGT + kGTPerBlock - 1) / kGTPerBlock;
    k_encode_fill<<<(unsigned)blocks, kThreads, 0, st>>>(W, T->M, T->K, KG, NGT, T->gtile_offset, T->bitmap, T->values);
    return cudaGetLastError() == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
}

int launch_decode(const spinfer_tca *T, uint16_t *W_out, cudaStream_t st) {
    int KG = (T->K + kGT - 1) / kGT;
    int64_t NGT = (int64_t)((T->M + kGT - 1) / kGT) * KG;
    int64_t blocks = (NGT + kGTPerBlock - 1) / kGTPerBlock;
    k_decode<<<(unsigned)blocks, kThreads, 0, st>>>(T->gtile_offset, T->bitmap, T->values, T->M, T->K, KG, NGT, W_out);
    return cudaGetLastError() == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
}

}  // namespace spinfer
