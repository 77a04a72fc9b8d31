#!/usr/bin/env python3
"""bench.py — TCA-BME SpMM (SpInfer hot path) on B200: one JSON line on rank 0.

Workload (BASELINE.json configs[1]): Y = W X with W fp16 M x K = 28672 x 8192 at
50% unstructured sparsity stored in TCA-BME, X fp16 K x N = 8192 x 16, fp32
accumulation. A "step" is one spinfer_spmm call (the whole hot path: bulk-async
staging, SMBD decode, tensor-core MMA, split-K fix-up) over that input.

Metric: algorithmic HBM GB/s = (TCA-BME bytes + X bytes + Y bytes) / kernel time
(SURVEY §8(d)(iii)); also µs per SpMM and the cuBLAS fp16 dense GEMM on the same
shape. L2 is flushed (256 MiB memset + 256 MiB read) before every timed step, outside the
events. Multi-GPU (torchrun): weak scaling — every rank owns its own 28672-row
shard of an (N_gpus*28672) x 8192 row-partitioned weight (seeded seed+rank), no
data-path collective (SURVEY §8(e), config 4 pattern); value = sum of all ranks'
bytes / max over ranks of the time.

--impl reference: the CPU oracle (oracle/, single-threaded fp64 C) timed on the
host on a bounded row sample of the same workload; rank 0 only.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "SpMM µs & HBM GB/s vs cuBLAS fp16, M/K/N=28K/8K/16, 30-70% sparsity"
UNIT = "GB/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--M", type=int, default=28672)
    ap.add_argument("--K", type=int, default=8192)
    ap.add_argument("--N", type=int, default=16)
    ap.add_argument("--sparsity", type=float, default=0.5)
    ap.add_argument("--seed", type=int, default=20250330)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-cublas", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--profile", action="store_true", help="minimal run for ncu (no flush, no baselines)")
    ap.add_argument("--json-out", default=None)
    return ap.parse_args()


def workload_name(a):
    return f"spmm_tca_bme M/K/N={a.M}/{a.K}/{a.N} s={a.sparsity}"


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", 6650.0)), "measured"
    return 6650.0, "fallback"


def algorithmic_bytes(M, K, N, n_values):
    """TCA-BME storage (eq. (9), with padded value count) + X + Y (fp16)."""
    return 4 * ((M // 64) * (K // 64) + 1) + 8 * (M * K // 64) + 2 * n_values + 2 * K * N + 2 * M * N


def cpu_info():
    model = "unknown"
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return model, os.cpu_count()


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """Samples SM clock and throttle reasons via NVML every ~1 ms during the timed region
    (falls back to nvidia-smi polling if NVML is unavailable)."""

    REASONS = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
               "sw_power_cap": 0x4, "hw_power_brake_slowdown": 0x80}

    def __init__(self, index: int, uuid: str | None = None):
        self.index = index
        self.uuid = uuid
        self.sm = []
        self.max_sm = None
        self.reasons = set()
        self._stop = threading.Event()
        self._t = None

    def _run(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            h = None
            if self.uuid:
                try:
                    h = pynvml.nvmlDeviceGetHandleByUUID(self.uuid)
                except Exception:
                    h = None
            if h is None:
                h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.max_sm = float(pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM))
            while not self._stop.is_set():
                self.sm.append(float(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)))
                try:
                    r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
                except AttributeError:
                    r = pynvml.nvmlDeviceGetCurrentClocksThrottleReasons(h)
                for name, bit in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
                time.sleep(0.0005)
        except Exception as e:  # pragma: no cover - NVML missing
            self.reasons.add(f"nvml unavailable: {type(e).__name__}")

    def __enter__(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        # NVML initialisation can outlast a short timed region: wait for the first sample, then
        # count only the samples taken from here on (the region itself)
        t0 = time.time()
        while not self.sm and not self.reasons and time.time() - t0 < 5.0:
            time.sleep(0.001)
        self._mark = len(self.sm)
        return self

    def __exit__(self, *exc):
        self._stop.set()
        if self._t:
            self._t.join(timeout=10)

    def summary(self):
        sm = self.sm[getattr(self, "_mark", 0):]
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": self.max_sm,
                "reasons": sorted(self.reasons), "samples": len(sm)}


# ----------------------------------------------------------------------------- reference arm
def run_reference(a, rank):
    """The CPU oracle as it stands, on a bounded sample: each step = oracle SpMM of
    the first `rows` rows of the workload's W (fp64, single-threaded)."""
    if rank != 0:
        return None
    import oracle
    import synth
    rows = 1024
    W = synth.weight(rows, a.K, a.sparsity, seed=a.seed)   # rows 0..1023 of the full W (same generator indices)
    X = synth.activation(a.K, a.N, seed=a.seed + 1)
    T = oracle.encode(W)
    b = algorithmic_bytes(rows, a.K, a.N, T.n_values)
    for _ in range(a.warmup):
        oracle.spmm_f64(T, X)
    ts = []
    for _ in range(a.steps):
        t0 = time.perf_counter()
        oracle.spmm_f64(T, X)
        ts.append(time.perf_counter() - t0)
    dt = statistics.mean(ts)
    v = b / dt / 1e9
    model, ncpu = cpu_info()
    sample = f"first {rows} of {a.M} rows of W (all {a.K} cols), N={a.N}, oracle.spmm_f64 (TCA-BME walk, fp64)"
    return {
        "impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": a.gpus, "steps": a.steps,
        "warmup": a.warmup, "ms_per_step": dt * 1e3, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": workload_name(a), "sample_rows": rows, "seed": a.seed},
        "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample,
                         "cpu_model": model, "host_cpus": ncpu},
        "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }


# ----------------------------------------------------------------------------- our arm
def run_ours(a, rank, world, local_rank):
    import torch
    import torch.distributed as dist
    import synth
    import paper_conf_eurosys_fanydlgww025_b200 as sp

    dev = torch.device("cuda", local_rank)
    torch.cuda.set_device(dev)
    M, K, N = a.M, a.K, a.N
    seed = a.seed + rank
    W = synth.weight(M, K, a.sparsity, seed=seed)
    X = synth.activation(K, N, seed=a.seed + 1)
    Wd = torch.from_numpy(W.view(np.int16)).to(dev)
    Xd = torch.from_numpy(X.view(np.int16)).to(dev).view(torch.float16)
    T = sp.encode(Wd)
    ws = sp.workspace(M, K, N, dev)
    Yd = torch.empty((M, N), dtype=torch.float16, device=dev)
    stream = torch.cuda.current_stream()
    nbytes = algorithmic_bytes(M, K, N, T.n_values)
    flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=dev)
    flush_rd = torch.zeros(64 * 1024 * 1024, dtype=torch.float32, device=dev)   # 256 MiB

    def flush_l2():
        # write a buffer larger than L2 (126 MB), then read another one: the timed kernel starts
        # with a cold L2 that holds no dirty lines (otherwise it pays the flush's write-backs)
        flush.zero_()
        flush_rd.sum()

    def barrier():
        if world > 1:
            dist.barrier()

    def timed(fn, steps, do_flush=True):
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
        barrier()
        torch.cuda.synchronize()
        # ~1 ms of device-side spin ahead of the loop, outside every event pair: the host gets
        # ahead of the device, so no step's events also time a host-side launch gap (without it
        # the first timed step read 257-384 us against 84-86 us for the others, profiles/r1_steps)
        torch.cuda._sleep(2_000_000)
        for _ in range(2):   # untimed lead-in steps in the same burst (the first step after a host
            if do_flush:     # synchronize also ran slow: profiles/r1_steps.txt)
                flush_l2()
            fn()
        for i in range(steps):
            if do_flush:
                flush_l2()
            evs[i][0].record(stream)
            fn()
            evs[i][1].record(stream)
        torch.cuda.synchronize()
        barrier()
        return [s.elapsed_time(e) for s, e in evs]

    def step():
        sp.spmm(T, Xd, Yd, ws)

    for _ in range(max(a.warmup, 3)):
        step()
    torch.cuda.synchronize()

    if a.profile:
        for _ in range(a.steps):
            step()
        torch.cuda.synchronize()
        return None

    try:
        uuid = "GPU-" + str(torch.cuda.get_device_properties(dev).uuid)
    except Exception:
        uuid = None
    with ClockSampler(local_rank, uuid) as clk:
        t_ms = timed(step, a.steps, do_flush=True)
    kern_ms = statistics.mean(t_ms)
    kern_med = statistics.median(t_ms)

    # max over ranks
    tt = torch.tensor([kern_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    kmax = float(tt.item())
    total_bytes = nbytes * world
    value = total_bytes / (kmax * 1e-3) / 1e9

    peak, peak_kind = load_peaks()
    achieved = nbytes / (kern_ms * 1e-3) / 1e9

    # e2e through the public API with host buffers: H2D X (pinned) + SpMM + D2H Y (pinned)
    e2e = None
    if not a.no_e2e:
        Xh = torch.from_numpy(X.view(np.int16)).pin_memory()
        Yh = torch.empty((M, N), dtype=torch.int16).pin_memory()
        Xe = torch.empty((K, N), dtype=torch.int16, device=dev)

        def e2e_step():
            Xe.copy_(Xh, non_blocking=True)
            sp.spmm(T, Xe, Yd, ws)
            Yh.copy_(Yd.view(torch.int16), non_blocking=True)

        for _ in range(3):
            e2e_step()
        e_ms = timed(e2e_step, a.steps, do_flush=True)
        em = torch.tensor([statistics.mean(e_ms)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(em, op=dist.ReduceOp.MAX)
        e2e = {"value": total_bytes / (float(em.item()) * 1e-3) / 1e9, "unit": UNIT,
               "h2d_bytes_per_step": int(Xh.numel() * 2), "d2h_bytes_per_step": int(Yh.numel() * 2),
               "ms_per_step": float(em.item())}
        # e2e result must equal the device-resident result
        assert torch.equal(Yh, Yd.view(torch.int16).cpu())

    # cuBLAS fp16 dense GEMM on the same shape, same protocol
    cublas = None
    if not a.no_cublas and rank == 0:
        torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
        Wdense = sp.decode(T)
        Yc = torch.empty((M, N), dtype=torch.float16, device=dev)

        def cub():
            torch.mm(Wdense, Xd, out=Yc)

        for _ in range(3):
            cub()
        c_ms = timed(cub, a.steps, do_flush=True) if world == 1 else None
        if c_ms:
            cm = statistics.mean(c_ms)
            cublas = {"us": cm * 1e3, "dense_bytes": 2 * M * K + 2 * K * N + 2 * M * N,
                      "gbs_dense": (2 * M * K + 2 * K * N + 2 * M * N) / (cm * 1e-3) / 1e9,
                      "speedup_spmm_vs_cublas": cm / kern_ms}
        del Wdense

    cpu = None
    if not a.no_cpu_baseline and rank == 0 and world == 1:
        import oracle
        rows = 8192
        Wc = W[:rows]
        Tc = oracle.encode(Wc)
        t0 = time.perf_counter()
        oracle.spmm_f64(Tc, X)
        dt = time.perf_counter() - t0
        model, ncpu = cpu_info()
        cpu = {"value": algorithmic_bytes(rows, K, N, Tc.n_values) / dt / 1e9, "unit": UNIT, "cores": 1,
               "kind": "oracle", "seconds": dt, "cpu_model": model, "host_cpus": ncpu,
               "sample": f"first {rows} of {M} rows of W (all {K} cols), N={N}: oracle.spmm_f64, single thread"}

    # ncu DRAM traffic for this kernel/config, if a committed capture exists
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        try:
            d = json.load(open(tp))
            traffic = d.get(workload_name(a))
        except Exception:
            traffic = None

    if rank != 0:
        return None
    return {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps, "warmup": a.warmup,
        "ms_per_step": kmax, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "f16 in / f32 acc", "data": "synthetic",
        "config": {"workload": workload_name(a), "M": M, "K": K, "N": N, "sparsity": a.sparsity,
                   "nnz": T.nnz, "n_values": T.n_values, "seed": a.seed, "l2": "flushed before each step: 256 MiB memset, then a 256 MiB read (cold, clean L2)",
                   "parallelism": f"row-partitioned x{world} (weak, no collective)" if world > 1 else "1 GPU"},
        "us_per_spmm": kmax * 1e3, "us_median": kern_med * 1e3, "us_steps": [round(x * 1e3, 1) for x in t_ms],
        "tflops_dense_equiv": 2 * M * K * N / (kern_ms * 1e-3) / 1e12,
        "frac_of_8tbs": achieved / 8000.0,
        "cublas_fp16": cublas,
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                     "peak_kind": peak_kind, "bytes_per_launch": nbytes, "traffic": traffic},
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": a.steps,
        "clocks": clk.summary(),
    }


def main():
    a = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if a.impl == "reference":
        out = run_reference(a, rank)
    else:
        if world > 1:
            import torch
            import torch.distributed as dist
            torch.cuda.set_device(local_rank)
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        out = run_ours(a, rank, world, local_rank)
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()
    if out is not None and rank == 0:
        line = json.dumps(out)
        print(line, flush=True)
        if a.json_out:
            with open(a.json_out, "w") as f:
                f.write(line + "\n")


if __name__ == "__main__":
    main()
