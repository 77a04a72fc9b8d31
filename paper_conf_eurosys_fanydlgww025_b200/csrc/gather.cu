// gather.cu — peer signalling of the fused all-gather epilogue (spinfer_spmm_tp_gather; SURVEY §8(f)
// rank 1: the communication cost the paper attributes its multi-GPU losses to).
//
// The SpMM kernel stores its rank's rows of Y straight into every rank's Y buffer (peer-mapped
// device memory over NVLink / NVSwitch). Completion is one counter per rank: after the kernel,
// each rank adds 1 to every rank's counter (release, system scope); a rank that needs the full
// Y waits until its counter has grown by `world` since its previous wait (acquire). The expected
// value lives in device memory (`state`), so the sequence works unchanged under CUDA-graph replay.
#include "internal.cuh"

namespace spinfer {
namespace {

__global__ void k_gather_signal(uint32_t *f0, uint32_t *f1, uint32_t *f2, uint32_t *f3, uint32_t *f4, uint32_t *f5,
                                uint32_t *f6, uint32_t *f7, int world) {
    const int r = threadIdx.x;
    if (r >= world) return;
    uint32_t *const f[kMaxPeers] = {f0, f1, f2, f3, f4, f5, f6, f7};
    // the preceding SpMM kernel completed (stream order): its peer stores are performed; the
    // release orders this signal after them for the peer that acquires it
    asm volatile("fence.acq_rel.sys;" ::: "memory");
    asm volatile("red.release.sys.global.add.u32 [%0], 1;" ::"l"(f[r]) : "memory");
}

__global__ void k_gather_wait(const uint32_t *flag, uint32_t *state, int world, int32_t *err, uint32_t timeout_us) {
    // a PDL-launched SpMM of the next layer (SPINFER_OPT_PDL) may start streaming its weights now; it
    // reads X (this gather's output) only after griddepcontrol.wait, i.e. after this kernel completed
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const uint32_t target = *state + (uint32_t)world;
    *state = target;
    uint64_t t0;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
    while (true) {
        uint32_t v;
        asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(flag) : "memory");
        if ((int32_t)(v - target) >= 0) break;
        uint64_t t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        if (timeout_us && t - t0 > (uint64_t)timeout_us * 1000ull) {   // a peer never signalled
            if (err) atomicOr(err, 4);
            break;
        }
        __nanosleep(256);
    }
}

}  // namespace

int launch_gather_signal(uint32_t *const *fp, int world, cudaStream_t st) {
    if (world < 1 || world > kMaxPeers) return SPINFER_EINVAL;
    uint32_t *f[kMaxPeers] = {nullptr};
    for (int r = 0; r < world; ++r) f[r] = fp[r];
    k_gather_signal<<<1, 32, 0, st>>>(f[0], f[1], f[2], f[3], f[4], f[5], f[6], f[7], world);
    return cudaGetLastError() == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
}

int launch_gather_wait(uint32_t *flag, uint32_t *state, int world, int32_t *err, uint32_t timeout_us, cudaStream_t st) {
    k_gather_wait<<<1, 1, 0, st>>>(flag, state, world, err, timeout_us);
    return cudaGetLastError() == cudaSuccess ? SPINFER_OK : SPINFER_ECUDA;
}

}  // namespace spinfer
