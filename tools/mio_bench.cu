// mio_bench.cu — do POPC (XU) and LDS share the MIO queue? (experiment tool)
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
template <int MODE>
__global__ void kb(uint32_t *out, int iters, unsigned long long *cyc) {
    __shared__ __align__(16) uint32_t sm[4096];
    for (int i = threadIdx.x; i < 4096; i += blockDim.x) sm[i] = i * 2654435761u;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    uint32_t base = (uint32_t)__cvta_generic_to_shared(sm) + ((threadIdx.x >> 5) * 256) % 8192;
    uint32_t x[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) x[k] = threadIdx.x * 2654435761u + k * 977u;
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            uint32_t off = ((x[k] & 31u) + (uint32_t)lane) * 2u;   // data-dependent, within 126 B
            if (MODE == 0 || MODE == 2) { uint16_t v; asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(base + off)); x[k] += v; }
            if (MODE == 1 || MODE == 2) { uint32_t p; asm volatile("popc.b32 %0, %1;" : "=r"(p) : "r"(x[k] ^ (uint32_t)it)); x[k] += p; }
            if (MODE == 3) { uint32_t p; asm volatile("prmt.b32 %0, %1, %2, %3;" : "=r"(p) : "r"(x[k]), "r"(off), "r"(x[k] >> 3)); x[k] += p;
                             uint16_t v; asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(base + off)); x[k] += v; }
        }
    }
    long long t1 = clock64();
    uint32_t s = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) s ^= x[k];
    if (s == 0x1234567) out[0] = s;
    if (threadIdx.x == 0) atomicAdd(cyc, (unsigned long long)(t1 - t0));
}
template <int MODE> void run(const char *name, int warps) {
    uint32_t *out; unsigned long long *cyc; cudaMalloc(&out, 4); cudaMalloc(&cyc, 8);
    int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    int iters = 2000;
    kb<MODE><<<nsm, 32 * warps>>>(out, 10, cyc); cudaMemset(cyc, 0, 8);
    kb<MODE><<<nsm, 32 * warps>>>(out, iters, cyc);
    unsigned long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
    printf("%-26s warps %2d: %.3f SM-cycles per group\n", name, warps, (double)c / nsm / ((double)iters * 8 * warps));
}
int main() {
    for (int w : {16, 32}) { run<0>("LDS.U16", w); run<1>("POPC", w); run<2>("LDS.U16 + POPC", w); run<3>("LDS.U16 + PRMT", w); }
}
