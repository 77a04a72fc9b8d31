// alu_bench2.cu — per-opcode SM throughput (8 independent chains per thread), experiment tool.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
template <int MODE>
__global__ void kb(uint32_t *out, int iters, unsigned long long *cyc) {
    uint32_t x[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) x[k] = threadIdx.x * 2654435761u + k * 977u;
    uint32_t m = (1u << (threadIdx.x & 31)) - 1u, c2 = m ^ 0x5a5a5a5au;
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int k = 0; k < 8; ++k) {
            uint32_t v = x[k];
            if (MODE == 0) asm volatile("popc.b32 %0, %1;" : "=r"(x[k]) : "r"(v));
            else if (MODE == 1) asm volatile("prmt.b32 %0, %1, %2, %3;" : "=r"(x[k]) : "r"(v), "r"(m), "r"(c2));
            else if (MODE == 2) asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(x[k]) : "r"(v), "r"(m), "r"(c2));
            else if (MODE == 3) asm volatile("shr.b32 %0, %1, %2;" : "=r"(x[k]) : "r"(v), "r"(m));
            else if (MODE == 4) asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(x[k]) : "r"(v), "r"(m), "r"(c2));
            else if (MODE == 5) asm volatile("add.u32 %0, %1, %2;" : "=r"(x[k]) : "r"(v), "r"(m));
            else if (MODE == 6) { asm volatile("popc.b32 %0, %1;" : "=r"(x[k]) : "r"(v)); asm volatile("prmt.b32 %0, %1, %2, %3;" : "=r"(m) : "r"(v), "r"(m), "r"(c2)); }
            else if (MODE == 7) asm volatile("bfe.u32 %0, %1, %2, 2;" : "=r"(x[k]) : "r"(v), "r"(m));
            else if (MODE == 8) asm volatile("shf.r.wrap.b32 %0, %1, %2, %3;" : "=r"(x[k]) : "r"(v), "r"(m), "r"(c2));
            else if (MODE == 9) { uint32_t r; asm volatile("{.reg .pred p; setp.ne.u32 p, %1, 0; selp.b32 %0, %2, %3, p;}" : "=r"(r) : "r"(v & 4u), "r"(m), "r"(c2)); x[k] = r; }
        }
    }
    long long t1 = clock64();
    uint32_t s = m;
#pragma unroll
    for (int k = 0; k < 8; ++k) s ^= x[k];
    if (s == 0x1234567) out[0] = s;
    if (threadIdx.x == 0) atomicAdd(cyc, (unsigned long long)(t1 - t0));
}
template <int MODE> void run(const char *name, int warps, double nops) {
    uint32_t *out; unsigned long long *cyc; cudaMalloc(&out, 4); cudaMalloc(&cyc, 8);
    int nsm; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    int iters = 4000;
    kb<MODE><<<nsm, 32 * warps>>>(out, 10, cyc); cudaMemset(cyc, 0, 8);
    kb<MODE><<<nsm, 32 * warps>>>(out, iters, cyc);
    unsigned long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
    double per = (double)c / nsm / ((double)iters * 8 * warps * nops);
    printf("%-22s warps %2d: %.3f SM-cycles per warp-instruction\n", name, warps, per);
}
int main() {
    for (int w : {16, 32}) {
        run<0>("POPC", w, 1); run<1>("PRMT", w, 1); run<2>("LOP3", w, 1); run<3>("SHR", w, 1);
        run<4>("IMAD", w, 1); run<5>("IADD", w, 1); run<6>("POPC+PRMT (per inst)", w, 2);
        run<7>("BFE", w, 1); run<8>("SHF.wrap", w, 1); run<9>("ISETP+SEL (per pair)", w, 1);
    }
}
