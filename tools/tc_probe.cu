// tc_probe.cu — experiment tool (not product code): checks the tcgen05 building blocks the
// SpMM kernel relies on, on the real GPU:
//   test 1: tcgen05.st.16x128b.x2 register -> (TMEM lane, column) mapping (read back with 32x32b)
//   test 2: tcgen05.mma.kind::f16, A from TMEM (written with 16x128b.x2 in the mma.sync
//           A-fragment layout), B = X [K][NB] row-major loaded by 2-D TMA with the 32B/64B
//           swizzle (MN-major canonical layout), D fp32 in TMEM, 4 k16 steps; N padded by TMA
//           OOB zero fill when the tensor is narrower than the box.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o tools/tc_probe tools/tc_probe.cu -lcuda
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <vector>
#include <cmath>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d: %s\n", #x, __LINE__, cudaGetErrorString(e)); exit(1);} } while (0)

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void tm_alloc(uint32_t dst_smem, uint32_t ncols) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(dst_smem), "r"(ncols) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tm_dealloc(uint32_t taddr, uint32_t ncols) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}
__device__ __forceinline__ void tm_st_16x128b_x2(uint32_t taddr, uint32_t r0, uint32_t r1, uint32_t r2, uint32_t r3) {
    asm volatile("tcgen05.st.sync.aligned.16x128b.x2.b32 [%0], {%1, %2, %3, %4};" ::"r"(taddr), "r"(r0), "r"(r1), "r"(r2), "r"(r3) : "memory");
}
__device__ __forceinline__ void tm_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void tm_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void tm_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tm_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tm_ld_32x32b_x8(uint32_t taddr, uint32_t (&r)[8]) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]) : "r"(taddr));
}
__device__ __forceinline__ void mma_f16_ts(uint32_t d_t, uint32_t a_t, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}"
                 ::"r"(d_t), "r"(a_t), "l"(bdesc), "r"(idesc), "r"(acc) : "memory");
}
__device__ __forceinline__ void mma_commit(uint32_t bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_init(uint32_t b, uint32_t c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(b), "r"(c)); }
__device__ __forceinline__ void mbar_wait(uint32_t b, uint32_t ph) {
    asm volatile("{.reg .pred p; W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W;}" ::"r"(b), "r"(ph) : "memory");
}
__device__ __forceinline__ void mbar_expect(uint32_t b, uint32_t tx) {
    asm volatile("{.reg .b64 s; mbarrier.arrive.expect_tx.shared::cta.b64 s, [%0], %1;}" ::"r"(b), "r"(tx) : "memory");
}
__device__ __forceinline__ void tma_2d(uint32_t dst, const void *tmap, int c0, int c1, uint32_t bar) {
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                 ::"r"(dst), "l"(reinterpret_cast<uint64_t>(tmap)), "r"(c0), "r"(c1), "r"(bar) : "memory");
}

__global__ void k_layout(uint32_t *out) {   // out[128][8]
    __shared__ uint32_t tslot;
    const int w = threadIdx.x / 32, l = threadIdx.x % 32;
    if (w == 0) tm_alloc(smem_u32(&tslot), 512);
    tm_fence_before(); __syncthreads(); tm_fence_after();
    const uint32_t tb = tslot;
    for (int h = 0; h < 2; ++h) {
        const int tr = 2 * w + h;
        uint32_t r[4];
        for (int j = 0; j < 4; ++j) r[j] = (uint32_t)(tr << 16) | (uint32_t)(l << 8) | (uint32_t)j;
        tm_st_16x128b_x2(tb + ((uint32_t)(16 * tr) << 16), r[0], r[1], r[2], r[3]);
    }
    tm_wait_st();
    uint32_t v[8];
    tm_ld_32x32b_x8(tb + ((uint32_t)(32 * w) << 16), v);
    tm_wait_ld();
    for (int j = 0; j < 8; ++j) out[(32 * w + l) * 8 + j] = v[j];
    tm_fence_before(); __syncthreads(); tm_fence_after();
    if (w == 0) tm_dealloc(tb, 512);
}

struct Args { CUtensorMap tmap; };

template <int NB>
__global__ void k_mma(const __grid_constant__ Args args, const __half *A /*[128][64]*/, float *out /*[128][NB]*/, int swz_type) {
    extern __shared__ __align__(1024) uint8_t sm_raw[];
    uint8_t *sm = sm_raw + ((1024u - (smem_u32(sm_raw) & 1023u)) & 1023u);
    __shared__ uint32_t tslot;
    __shared__ __align__(8) uint64_t bars[2];
    const int w = threadIdx.x / 32, l = threadIdx.x % 32;
    const uint32_t xs = smem_u32(sm);
    if (threadIdx.x == 0) {
        mbar_init(smem_u32(&bars[0]), 1); mbar_init(smem_u32(&bars[1]), 1);
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    if (w == 0) tm_alloc(smem_u32(&tslot), 512);
    tm_fence_before(); __syncthreads(); tm_fence_after();
    const uint32_t tb = tslot;
    if (threadIdx.x == 0) {
        mbar_expect(smem_u32(&bars[0]), 64 * NB * 2);
        tma_2d(xs, &args.tmap, 0, 0, smem_u32(&bars[0]));
    }
    // A fragments: k16 step s at TMEM columns 32 + 8 s
    const int g = l / 4, c = l % 4;
    auto pk = [&](int row, int col) {
        __half2 h = __halves2half2(A[row * 64 + col], A[row * 64 + col + 1]);
        return *reinterpret_cast<uint32_t *>(&h);
    };
    for (int s = 0; s < 4; ++s)
        for (int h = 0; h < 2; ++h) {
            const int tr = 2 * w + h, r0 = 16 * tr + g, k0 = 16 * s + 2 * c;
            tm_st_16x128b_x2(tb + ((uint32_t)(16 * tr) << 16) + 32u + 8u * s, pk(r0, k0), pk(r0 + 8, k0), pk(r0, k0 + 8), pk(r0 + 8, k0 + 8));
        }
    tm_wait_st();
    tm_fence_before(); __syncthreads(); tm_fence_after();
    if (threadIdx.x == 0) {
        mbar_wait(smem_u32(&bars[0]), 0);
        const uint32_t idesc = (1u << 4) | (0u << 7) | (0u << 10) | (1u << 16) | ((uint32_t)(NB >> 3) << 17) | ((128u >> 4) << 24);
        for (int s = 0; s < 4; ++s) {
            const uint32_t start = xs + (uint32_t)s * 16u * NB * 2u;
            const uint64_t sbo = (uint64_t)(8 * NB * 2) >> 4;
            const uint64_t lbo = 1;
            uint64_t d = (uint64_t)((start >> 4) & 0x3FFF) | (lbo << 16) | (sbo << 32) | (1ull << 46) | ((uint64_t)swz_type << 61);
            mma_f16_ts(tb + 0u, tb + 32u + 8u * s, d, idesc, s > 0 ? 1u : 0u);
        }
        const long long t0 = clock64();
        mma_commit(smem_u32(&bars[1]));
        mbar_wait(smem_u32(&bars[1]), 0);
        const long long t1 = clock64();
        // second round: 16 MMAs back to back (a stage's worth), then commit
        for (int s = 0; s < 16; ++s) {
            const uint32_t start = xs + (uint32_t)(s & 3) * 16u * NB * 2u;
            const uint64_t sbo = (uint64_t)(8 * NB * 2) >> 4;
            uint64_t d = (uint64_t)((start >> 4) & 0x3FFF) | (1ull << 16) | (sbo << 32) | (1ull << 46) | ((uint64_t)swz_type << 61);
            mma_f16_ts(tb + 64u, tb + 32u + 8u * (s & 3), d, (1u << 4) | (1u << 16) | ((uint32_t)(NB >> 3) << 17) | ((128u >> 4) << 24), s > 0 ? 1u : 0u);
        }
        const long long t2 = clock64();
        mma_commit(smem_u32(&bars[1]));
        mbar_wait(smem_u32(&bars[1]), 1);
        const long long t3 = clock64();
        printf("NB=%d: 4 MMAs issue+commit->arrive %lld cycles (issue part incl. above); 16 MMAs issue %lld, commit->arrive %lld cycles\n", NB, t1 - t0, t2 - t1, t3 - t2);
    }
    __syncwarp();
    mbar_wait(smem_u32(&bars[1]), 0);
    tm_fence_after();
    for (int cb = 0; cb < NB; cb += 8) {
        uint32_t v[8];
        tm_ld_32x32b_x8(tb + ((uint32_t)(32 * w) << 16) + (uint32_t)cb, v);
        tm_wait_ld();
        for (int j = 0; j < 8; ++j) out[(32 * w + l) * NB + cb + j] = __uint_as_float(v[j]);
    }
    tm_fence_before(); __syncthreads(); tm_fence_after();
    if (w == 0) tm_dealloc(tb, 512);
}

using EncodeTiledFn = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                   const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

template <int NB>
int run_mma(int Nreal) {
    const int K = 64;
    std::vector<__half> hA(128 * 64), hX(K * Nreal);
    std::vector<float> fA(128 * 64), fX(K * Nreal);
    srand(1 + Nreal);
    for (int i = 0; i < 128 * 64; ++i) { int v = rand() % 7 - 3; fA[i] = v; hA[i] = __float2half((float)v); }
    for (int i = 0; i < K * Nreal; ++i) { int v = rand() % 5 - 2; fX[i] = v; hX[i] = __float2half((float)v); }
    __half *dA, *dX; float *dO;
    CK(cudaMalloc(&dA, hA.size() * 2)); CK(cudaMalloc(&dX, hX.size() * 2)); CK(cudaMalloc(&dO, 128 * NB * 4));
    CK(cudaMemcpy(dA, hA.data(), hA.size() * 2, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dX, hX.data(), hX.size() * 2, cudaMemcpyHostToDevice));
    CK(cudaMemset(dO, 0xFF, 128 * NB * 4));
    void *f = nullptr; cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q));
    Args args;
    const cuuint64_t dims[2] = {(cuuint64_t)Nreal, (cuuint64_t)K};
    const cuuint64_t strides[1] = {(cuuint64_t)Nreal * 2};
    const cuuint32_t box[2] = {(cuuint32_t)NB, 64u};
    const cuuint32_t estr[2] = {1u, 1u};
    const CUtensorMapSwizzle sw = NB == 16 ? CU_TENSOR_MAP_SWIZZLE_32B : CU_TENSOR_MAP_SWIZZLE_64B;
    CUresult r = ((EncodeTiledFn)f)(&args.tmap, CU_TENSOR_MAP_DATA_TYPE_UINT16, 2, dX, dims, strides, box, estr,
                                    CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) { printf("tmap encode failed %d\n", (int)r); return 1; }
    const int swz_type = NB == 16 ? 6 : 4;
    CK(cudaFuncSetAttribute(k_mma<NB>, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024));
    k_mma<NB><<<1, 128, 64 * 1024>>>(args, dA, dO, swz_type);
    CK(cudaDeviceSynchronize());
    std::vector<float> hO(128 * NB);
    CK(cudaMemcpy(hO.data(), dO, hO.size() * 4, cudaMemcpyDeviceToHost));
    int bad = 0;
    for (int i = 0; i < 128; ++i)
        for (int n = 0; n < NB; ++n) {
            double ref = 0;
            if (n < Nreal) for (int k = 0; k < K; ++k) ref += (double)fA[i * 64 + k] * fX[k * Nreal + n];
            if (std::fabs(ref - hO[i * NB + n]) > 1e-3) { if (bad < 8) printf("  mismatch i=%d n=%d got %f ref %f\n", i, n, hO[i * NB + n], ref); ++bad; }
        }
    printf("mma NB=%d Nreal=%d: %s (%d bad)\n", NB, Nreal, bad ? "FAIL" : "OK", bad);
    cudaFree(dA); cudaFree(dX); cudaFree(dO);
    return bad != 0;
}

int main() {
    uint32_t *dout; CK(cudaMalloc(&dout, 128 * 8 * 4));
    k_layout<<<1, 128>>>(dout);
    CK(cudaDeviceSynchronize());
    std::vector<uint32_t> h(128 * 8);
    CK(cudaMemcpy(h.data(), dout, h.size() * 4, cudaMemcpyDeviceToHost));
    int bad = 0;
    for (int row = 0; row < 128; ++row)
        for (int col = 0; col < 8; ++col) {
            const int tr = row / 16, rr = row % 16, g = rr % 8, hi = rr / 8, c = col % 4, hc = col / 4;
            const uint32_t lane = g * 4 + c, j = hi + 2 * hc;   // expected: A-fragment order
            const uint32_t exp = (uint32_t)(tr << 16) | (lane << 8) | j;
            if (h[row * 8 + col] != exp) { if (bad < 8) printf("  layout row %d col %d got %06x exp %06x\n", row, col, h[row * 8 + col], exp); ++bad; }
        }
    printf("16x128b.x2 layout == mma A-fragment: %s (%d bad)\n", bad ? "FAIL" : "OK", bad);
    int rc = bad != 0;
    rc |= run_mma<16>(16);
    rc |= run_mma<16>(8);
    rc |= run_mma<32>(32);
    rc |= run_mma<32>(24);
    printf("probe %s\n", rc ? "FAILED" : "PASSED");
    return rc;
}
