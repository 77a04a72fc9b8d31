// launch_probe.cu — experiment tool: what does launching a 1-CTA-per-SM kernel cost on B200,
// measured like bench.py (CUDA events around the launch, an L2 flush before it)?
//   A: empty kernel, no dynamic smem          B: empty kernel, 228 KB dynamic smem
//   C: B + TMEM alloc/dealloc of 512 columns   each after a flush, and back to back
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o tools/launch_probe tools/launch_probe.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>

__global__ void k_empty(int *sink) { if (threadIdx.x == 9999) *sink = 1; }
__global__ void k_smem(int *sink) {
    extern __shared__ uint8_t sm[];
    if (threadIdx.x == 9999) *sink = sm[5];
}
__global__ void k_tmem(int *sink) {
    extern __shared__ uint8_t sm[];
    __shared__ uint32_t slot;
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"((uint32_t)__cvta_generic_to_shared(&slot)) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(slot) : "memory");
    if (threadIdx.x == 9999) *sink = sm[5];
}
__global__ void k_flush(uint4 *p, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) p[i] = make_uint4(0, 0, 0, 0);
}

int main() {
    int *sink; cudaMalloc(&sink, 4);
    uint4 *fl; size_t fb = 256u << 20; cudaMalloc(&fl, fb);
    const int smem = 228 * 1024;
    cudaFuncSetAttribute(k_smem, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(k_tmem, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    auto run = [&](const char *name, int which, bool flush) {
        std::vector<float> t;
        for (int it = 0; it < 25; ++it) {
            if (flush) k_flush<<<1184, 256>>>(fl, fb / 16);
            cudaEventRecord(a);
            if (which == 0) k_empty<<<148, 640>>>(sink);
            else if (which == 1) k_smem<<<148, 640, smem>>>(sink);
            else k_tmem<<<148, 640, smem>>>(sink);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b);
            if (it >= 5) t.push_back(ms * 1e3f);
        }
        std::sort(t.begin(), t.end());
        printf("%-34s %s: median %.2f us  min %.2f us\n", name, flush ? "after flush " : "back-to-back", t[t.size() / 2], t[0]);
    };
    for (int f = 1; f >= 0; --f) {
        run("empty kernel, no smem", 0, f);
        run("empty kernel, 228 KB smem", 1, f);
        run("228 KB smem + TMEM alloc 512 cols", 2, f);
    }
    return 0;
}
