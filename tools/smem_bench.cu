// smem_bench.cu — SM-level throughput of shared-memory / shuffle access patterns on
// B200 (experiment tool, not product code). Each warp runs a long unrolled loop of
// independent operations; result = SM cycles per warp-instruction (all warps).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

template <int MODE>
__global__ void kb(uint32_t *out, int iters, unsigned long long *cyc) {
    __shared__ __align__(16) uint32_t sm[8192];
    for (int i = threadIdx.x; i < 8192; i += blockDim.x) sm[i] = i * 2654435761u;
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t base = (uint32_t)__cvta_generic_to_shared(sm) + (warp * 512) % 16384;
    uint32_t acc = lane;
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int u = 0; u < 16; ++u) {
            uint32_t off = (uint32_t)((u * 97 + it * 13) & 511) * 16u;
            if (MODE == 0) {          // LDS.U16, 32 lanes within 64 B (SMBD value loads)
                uint16_t v; asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(base + off + ((lane * 7) & 31) * 2));
                acc += v;
            } else if (MODE == 1) {   // LDS.128, 2 distinct addresses (half-warps)
                uint32_t a, b, c, d; asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(a), "=r"(b), "=r"(c), "=r"(d) : "r"(base + off + (lane >> 4) * 16));
                acc += a ^ b ^ c ^ d;
            } else if (MODE == 2) {   // LDS.128 broadcast
                uint32_t a, b, c, d; asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(a), "=r"(b), "=r"(c), "=r"(d) : "r"(base + off));
                acc += a ^ b ^ c ^ d;
            } else if (MODE == 3) {   // LDS.64, 2 distinct addresses
                uint32_t a, b; asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(a), "=r"(b) : "r"(base + off + (lane >> 4) * 8));
                acc += a ^ b;
            } else if (MODE == 4) {   // LDS.32 coalesced 128 B
                uint32_t a; asm volatile("ld.shared.u32 %0, [%1];" : "=r"(a) : "r"(base + off + lane * 4));
                acc += a;
            } else if (MODE == 5) {   // SHFL.IDX, data-dependent source lane
                acc += __shfl_sync(0xffffffffu, acc, (acc + u) & 31);
            } else if (MODE == 6) {   // LDS.U16 + SHFL interleaved (do they share a pipe?)
                uint16_t v; asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(base + off + ((lane * 7) & 31) * 2));
                acc += v + __shfl_sync(0xffffffffu, acc, (lane + u) & 31);
            } else if (MODE == 7) {   // LDS.64, 32 lanes within 64 B (8 unique words)
                uint32_t a, b; asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(a), "=r"(b) : "r"(base + off + ((lane * 3) & 7) * 8));
                acc += a ^ b;
            } else if (MODE == 8) {   // LDS.128 of 2 distinct addresses, 4 per quarter (8 lanes same addr)
                uint32_t a, b, c, d; asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(a), "=r"(b), "=r"(c), "=r"(d) : "r"(base + off + ((lane >> 3) & 1) * 16));
                acc += a ^ b ^ c ^ d;
            } else if (MODE == 9) {   // LDS.32, 32 lanes within 64 B (duplicates), unaligned-ish spread
                uint32_t a; asm volatile("ld.shared.u32 %0, [%1];" : "=r"(a) : "r"(base + off + ((lane * 7) & 15) * 4));
                acc += a;
            } else if (MODE == 10) {  // PRMT+POPC ALU mix only (reference)
                acc = __byte_perm(acc, acc * 3u, 0x5410) + __popc(acc ^ u);
            }
        }
    }
    long long t1 = clock64();
    if (acc == 0x1234567) out[0] = acc;
    if (threadIdx.x == 0) atomicAdd(cyc, (unsigned long long)(t1 - t0));
}

template <int MODE>
void run(const char *name, int warps) {
    uint32_t *out; unsigned long long *cyc;
    cudaMalloc(&out, 4); cudaMalloc(&cyc, 8);
    int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    int iters = 2000;
    kb<MODE><<<nsm, 32 * warps>>>(out, 10, cyc);
    cudaMemset(cyc, 0, 8);
    kb<MODE><<<nsm, 32 * warps>>>(out, iters, cyc);
    unsigned long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
    double per_cta = (double)c / nsm;
    double inst = (double)iters * 16 * warps * (MODE == 6 ? 2 : 1);
    printf("%-48s warps %2d: %.3f SM-cycles per warp-instruction\n", name, warps, per_cta / inst);
}

int main() {
    for (int w : {8, 16}) {
        run<0>("LDS.U16 lanes within 64B", w);
        run<1>("LDS.128 2 addresses (half-warps)", w);
        run<8>("LDS.128 2 addresses (alternating quarters)", w);
        run<2>("LDS.128 broadcast", w);
        run<3>("LDS.64 2 addresses", w);
        run<7>("LDS.64 8 words within 64B", w);
        run<4>("LDS.32 coalesced 128B", w);
        run<9>("LDS.32 within 64B", w);
        run<5>("SHFL.IDX", w);
        run<6>("LDS.U16 + SHFL (per op)", w);
        run<10>("PRMT+POPC+IADD ALU", w);
    }
    return 0;
}
