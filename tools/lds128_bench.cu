// Wavefront cost of LDS.128 / LDS.64 / LDS.U16 access patterns (run under ncu with
// l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum; one kernel per pattern).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/lds128_bench tools/lds128_bench.cu
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ uint4 lds4(uint32_t a) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
    return v;
}
__device__ __forceinline__ uint2 lds2(uint32_t a) {
    uint2 v;
    asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
    return v;
}

// pattern: 0 = all lanes same 16 B; 1 = halves at +0 / +512 (same banks); 2 = halves at +0 / +16;
// 3 = every lane distinct consecutive 16 B; 4 = LDS.64 halves at +0/+512; 5 = LDS.64 halves +0/+8
template <int PAT>
__global__ void k(uint32_t *out, int iters) {
    __shared__ __align__(16) uint32_t buf[4096];
    for (int i = threadIdx.x; i < 4096; i += blockDim.x) buf[i] = i;
    __syncthreads();
    const uint32_t base = (uint32_t)__cvta_generic_to_shared(buf);
    const int lane = threadIdx.x & 31;
    uint32_t off;
    if (PAT == 0) off = 0;
    else if (PAT == 1 || PAT == 4) off = (lane >> 4) * 512;
    else if (PAT == 2) off = (lane >> 4) * 16;
    else if (PAT == 5) off = (lane >> 4) * 8;
    else off = lane * 16;
    uint32_t acc = 0;
    for (int it = 0; it < iters; ++it) {
        const uint32_t a = base + off + (uint32_t)(it & 7) * 1024u;
        if (PAT <= 3) {
            uint4 v = lds4(a);
            acc += v.x ^ v.y ^ v.z ^ v.w;
        } else {
            uint2 v = lds2(a);
            acc += v.x ^ v.y;
        }
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

int main() {
    uint32_t *out;
    cudaMalloc(&out, 1 << 20);
    const int iters = 1000;
    k<0><<<1, 32>>>(out, iters);
    k<1><<<1, 32>>>(out, iters);
    k<2><<<1, 32>>>(out, iters);
    k<3><<<1, 32>>>(out, iters);
    k<4><<<1, 32>>>(out, iters);
    k<5><<<1, 32>>>(out, iters);
    cudaDeviceSynchronize();
    printf("done %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
