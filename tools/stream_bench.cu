// stream_bench.cu — microbenchmark: achievable HBM read bandwidth on B200 for the
// load mechanisms the SpMM pipeline can use (experiment tool, not product code).
//   mode 0: one thread per CTA issues cp.async.bulk (1-D TMA) chunks into an S-slot ring
//   mode 1: 4 producer lanes (one per warp of a producer warpgroup) issue bulk chunks round-robin
//   mode 2: cp.async 16 B (LDGSTS) by all threads into the ring, commit/wait groups
//   mode 3: plain ld.global.v4 streaming by all threads (registers, reduced to avoid DCE)
// Usage: stream_bench MB CHUNK_KB SLOTS THREADS MODE
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint32_t b, uint32_t c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(b), "r"(c)); }
__device__ __forceinline__ void mbar_expect(uint32_t b, uint32_t tx) {
    asm volatile("{.reg .b64 s; mbarrier.arrive.expect_tx.shared::cta.b64 s, [%0], %1;}" ::"r"(b), "r"(tx) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t b) { asm volatile("{.reg .b64 s; mbarrier.arrive.shared::cta.b64 s, [%0];}" ::"r"(b) : "memory"); }
__device__ __forceinline__ void mbar_wait(uint32_t b, uint32_t ph) {
    asm volatile("{.reg .pred p; W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1; @!p bra W;}" ::"r"(b), "r"(ph) : "memory");
}
__device__ __forceinline__ void bulk(uint32_t dst, const void *src, uint32_t n, uint32_t bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst), "l"(src), "r"(n), "r"(bar) : "memory");
}

extern __shared__ __align__(128) uint8_t sm[];

__global__ void k_bulk(const uint8_t *src, size_t bytes, int chunk, int S, int nprod, unsigned long long *sink) {
    const int P = gridDim.x, p = blockIdx.x;
    size_t per = (bytes / P) / chunk * chunk;
    const uint8_t *base = src + per * p;
    long long nch = per / chunk;
    uint32_t bars = smem_u32(sm), ring = bars + 1024;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(bars + 16 * s, 1); mbar_init(bars + 16 * s + 8, 1); }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    if (warp < nprod && lane == 0) {
        for (long long i = warp; i < nch; i += nprod) {
            int s = (int)(i % S);
            if (i >= S) mbar_wait(bars + 16 * s + 8, ((i / S) - 1) & 1);
            mbar_expect(bars + 16 * s, chunk);
            bulk(ring + (uint32_t)s * chunk, base + i * chunk, chunk, bars + 16 * s);
        }
    } else if (warp == nprod) {   // consumer: release as soon as full
        unsigned long long acc = 0;
        for (long long i = 0; i < nch; ++i) {
            int s = (int)(i % S);
            mbar_wait(bars + 16 * s, (i / S) & 1);
            if (lane == 0) { acc += sm[1024 + (size_t)s * chunk]; mbar_arrive(bars + 16 * s + 8); }
            __syncwarp();
        }
        if (lane == 0 && acc == 12345) *sink = acc;
    }
}

// mode 4: NP producer warps issue LDGSTS (16 B per lane) for a chunk, completion via
// cp.async.mbarrier.arrive.noinc on the slot's full barrier (count 32*NP); one consumer warp releases.
__global__ void k_ldgsts_mbar(const uint8_t *src, size_t bytes, int chunk, int S, int NP, unsigned long long *sink) {
    const int P = gridDim.x, p = blockIdx.x;
    size_t per = (bytes / P) / chunk * chunk;
    const uint8_t *base = src + per * p;
    long long nch = per / chunk;
    uint32_t bars = smem_u32(sm), ring = bars + 1024;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(bars + 16 * s, 32 * NP); mbar_init(bars + 16 * s + 8, 1); }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    if (warp < NP) {
        int t = warp * 32 + lane, nt = 32 * NP;
        for (long long i = 0; i < nch; ++i) {
            int s = (int)(i % S);
            if (i >= S) mbar_wait(bars + 16 * s + 8, ((i / S) - 1) & 1);
            for (int o = t * 16; o < chunk; o += nt * 16)
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(ring + (uint32_t)s * chunk + o), "l"(base + i * chunk + o));
            asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(bars + 16 * s) : "memory");
        }
    } else if (warp == NP) {
        unsigned long long acc = 0;
        for (long long i = 0; i < nch; ++i) {
            int s = (int)(i % S);
            mbar_wait(bars + 16 * s, (i / S) & 1);
            if (lane == 0) { acc += sm[1024 + (size_t)s * chunk]; mbar_arrive(bars + 16 * s + 8); }
            __syncwarp();
        }
        if (lane == 0 && acc == 12345) *sink = acc;
    }
}

// mode 5: one warp, lanes 0..L-1 each issue 1/L of every chunk as its own bulk copy.
__global__ void k_bulk_lanes(const uint8_t *src, size_t bytes, int chunk, int S, int L, unsigned long long *sink) {
    const int P = gridDim.x, p = blockIdx.x;
    size_t per = (bytes / P) / chunk * chunk;
    const uint8_t *base = src + per * p;
    long long nch = per / chunk;
    uint32_t bars = smem_u32(sm), ring = bars + 1024;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) { mbar_init(bars + 16 * s, 1); mbar_init(bars + 16 * s + 8, 1); }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    int piece = chunk / L;
    if (warp == 0) {
        for (long long i = 0; i < nch; ++i) {
            int s = (int)(i % S);
            if (i >= S) mbar_wait(bars + 16 * s + 8, ((i / S) - 1) & 1);
            if (lane == 0) mbar_expect(bars + 16 * s, chunk);
            __syncwarp();
            if (lane < L) bulk(ring + (uint32_t)s * chunk + lane * piece, base + i * chunk + lane * piece, piece, bars + 16 * s);
        }
    } else if (warp == 1) {
        unsigned long long acc = 0;
        for (long long i = 0; i < nch; ++i) {
            int s = (int)(i % S);
            mbar_wait(bars + 16 * s, (i / S) & 1);
            if (lane == 0) { acc += sm[1024 + (size_t)s * chunk]; mbar_arrive(bars + 16 * s + 8); }
            __syncwarp();
        }
        if (lane == 0 && acc == 12345) *sink = acc;
    }
}

__global__ void k_ldgsts(const uint8_t *src, size_t bytes, int chunk, int S, unsigned long long *sink) {
    const int P = gridDim.x, p = blockIdx.x;
    size_t per = (bytes / P) / chunk * chunk;
    const uint8_t *base = src + per * p;
    long long nch = per / chunk;
    uint32_t ring = smem_u32(sm);
    unsigned long long acc = 0;
    int nt = blockDim.x;
    for (long long i = 0; i < nch + S - 1; ++i) {
        if (i < nch) {
            int s = (int)(i % S);
            for (int o = threadIdx.x * 16; o < chunk; o += nt * 16)
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(ring + (uint32_t)s * chunk + o), "l"(base + i * chunk + o));
        }
        asm volatile("cp.async.commit_group;");
        asm volatile("cp.async.wait_group %0;" ::"n"(6));
        __syncthreads();
        if (i >= S - 1) acc += sm[(size_t)((i - S + 1) % S) * chunk + threadIdx.x];
        __syncthreads();
    }
    if (acc == 12345) *sink = acc;
}

__global__ void k_ldg(const uint4 *src, size_t n16, unsigned long long *sink) {
    size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x, stride = (size_t)gridDim.x * blockDim.x;
    uint32_t acc = 0;
#pragma unroll 8
    for (; i < n16; i += stride) {
        uint4 v;
        asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(src + i));
        acc ^= v.x ^ v.y ^ v.z ^ v.w;
    }
    if (acc == 0x12345) *sink = acc;
}

int main(int argc, char **argv) {
    size_t MB = argc > 1 ? atol(argv[1]) : 512;
    int chunk = (argc > 2 ? atoi(argv[2]) : 16) * 1024;
    int S = argc > 3 ? atoi(argv[3]) : 8;
    int threads = argc > 4 ? atoi(argv[4]) : 128;
    int mode = argc > 5 ? atoi(argv[5]) : 0;
    size_t bytes = MB << 20;
    uint8_t *src; unsigned long long *sink;
    cudaMalloc(&src, bytes); cudaMalloc(&sink, 8);
    cudaMemset(src, 1, bytes);
    uint8_t *flush; cudaMalloc(&flush, 512 << 20);
    uint8_t *flush2; cudaMalloc(&flush2, 512 << 20); cudaMemset(flush2, 0, 512 << 20);
    int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    size_t smem = (mode == 2 ? 0 : 1024) + (size_t)S * chunk;
    cudaFuncSetAttribute(k_bulk, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(k_ldgsts, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(k_ldgsts_mbar, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(k_bulk_lanes, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int ctas = argc > 6 ? atoi(argv[6]) : 1;   // CTAs per SM (bulk modes)
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    float best = 1e9;
    for (int it = 0; it < 6; ++it) {
        cudaMemsetAsync(flush, it, 512 << 20);
        k_ldg<<<nsm * 8, 512, 0>>>((const uint4 *)flush2, (512u << 20) / 16, sink);   // clean L2: a read pass evicts the dirty lines
        cudaEventRecord(a);
        if (mode == 0) k_bulk<<<nsm * ctas, 64, smem>>>(src, bytes, chunk, S, 1, sink);
        else if (mode == 4) k_ldgsts_mbar<<<nsm * ctas, threads, smem>>>(src, bytes, chunk, S, threads / 32 - 1, sink);
        else if (mode == 5) k_bulk_lanes<<<nsm * ctas, 64, smem>>>(src, bytes, chunk, S, threads, sink);
        else if (mode == 1) k_bulk<<<nsm, 32 * 5, smem>>>(src, bytes, chunk, S, 4, sink);
        else if (mode == 2) k_ldgsts<<<nsm, threads, smem>>>(src, bytes, chunk, S, sink);
        else k_ldg<<<nsm * 8, threads, 0>>>((const uint4 *)src, bytes / 16, sink);
        cudaEventRecord(b); cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        if (it > 0 && ms < best) best = ms;
    }
    cudaError_t e = cudaGetLastError();
    printf("mode %d ctas/SM %d MB %zu chunk %dKB S %d thr %d: %.1f us  %.0f GB/s %s\n", mode, ctas, MB, chunk / 1024, S, threads, best * 1e3,
           bytes / (best * 1e-3) / 1e9, e == cudaSuccess ? "" : cudaGetErrorString(e));
    return 0;
}
