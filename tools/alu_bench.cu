// alu_bench.cu — SM-level throughput of POPC and alternatives (experiment tool).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
template <int MODE>
__global__ void kb(uint32_t *out, int iters, unsigned long long *cyc) {
    uint32_t x[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) x[k] = threadIdx.x * 2654435761u + k * 977u;
    const uint32_t m = (1u << (threadIdx.x & 31)) - 1u;
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            uint32_t v = x[k] ^ (uint32_t)it;
            if (MODE == 0) x[k] += __popc(v & m);                      // POPC (XU?)
            else if (MODE == 1) x[k] += (v & m) * 3u;                  // IMAD (reference)
            else if (MODE == 2) x[k] += __byte_perm(v, m, 0x5410);     // PRMT
            else if (MODE == 3) { uint32_t y = v & m; y = y - ((y >> 1) & 0x55555555u); y = (y & 0x33333333u) + ((y >> 2) & 0x33333333u);
                                  x[k] += (((y + (y >> 4)) & 0x0F0F0F0Fu) * 0x01010101u) >> 24; }   // SWAR popcount
            else if (MODE == 4) x[k] += __shfl_xor_sync(0xffffffffu, v, k + 1);
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
    int iters = 4000;
    kb<MODE><<<nsm, 32 * warps>>>(out, 10, cyc); cudaMemset(cyc, 0, 8);
    kb<MODE><<<nsm, 32 * warps>>>(out, iters, cyc);
    unsigned long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
    double per = (double)c / nsm / ((double)iters * 8 * warps);
    printf("%-28s warps %2d: %.3f SM-cycles per warp-op (op-group)\n", name, warps, per);
}
int main() {
    for (int w : {8, 16, 32}) {
        run<0>("POPC(v&m)+IADD", w); run<1>("LOP+IMAD", w); run<2>("PRMT+IADD", w);
        run<3>("SWAR popcount (~12 ops)", w); run<4>("SHFL.BFLY+IADD", w);
    }
}
