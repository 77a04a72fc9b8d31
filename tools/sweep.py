"""Config 3 (BASELINE.json configs[2]): sparsity sweep x N on the OPT linear-layer shapes, 1 x B200.

For every (model, layer, s, N) point: seeded synthetic W (SURVEY.md §8(d)(i) recipe) encoded to
TCA-BME on the GPU, the SpMM timed with CUDA events on the launching stream (L2 flushed before
every timed launch: 256 MiB memset + 256 MiB read, as in bench.py), cuBLAS fp16 dense GEMM
(torch.mm on the decoded W) timed identically, and a parity check of 128 sampled output rows
against an fp64 product of the generator's dense W (north_star tolerance
|Y - Y_ref| <= 2e-3 (|W||X|) + 1e-3). Prints one JSON line per point and a summary table.

Usage: python tools/sweep.py [--models 13b,30b,66b] [--s 0.3,0.4,0.5,0.6,0.7] [--N 8,16,32]
                             [--steps 10] [--out profiles/r1_sweep.jsonl]
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_eurosys_fanydlgww025_b200 as sp

# OPT linear shapes (M = output features, K = input features): SURVEY.md §8(d)(i)
OPT = {
    "13b": {"h": 5120, "ffn": 20480},
    "30b": {"h": 7168, "ffn": 28672},
    "66b": {"h": 9216, "ffn": 36864},
}


# Other model families of the paper's Fig. 10 (external: the public model configs):
# gated MLPs (gate and up projections fused as one 2*ffn x h weight), grouped-query attention
# (QKV = h + 2 * kv_heads * head_dim rows). Every M and K is a multiple of 64.
GATED = {
    "llama2-7b": {"h": 4096, "ffn": 11008, "kv": 4096},
    "llama2-70b": {"h": 8192, "ffn": 28672, "kv": 2 * 8 * 128 // 2},
    "llama3-8b": {"h": 4096, "ffn": 14336, "kv": 8 * 128},
    "qwen2-7b": {"h": 3584, "ffn": 18944, "kv": 4 * 128},
    "mixtral-8x7b-expert": {"h": 4096, "ffn": 14336, "kv": 8 * 128},
}


def layers(m):
    if m in GATED:
        h, f, kv = GATED[m]["h"], GATED[m]["ffn"], GATED[m]["kv"]
        return {"QKV": (h + 2 * kv, h), "O": (h, h), "GateUp": (2 * f, h), "Down": (h, f)}
    h, f = OPT[m]["h"], OPT[m]["ffn"]
    return {"QKV": (3 * h, h), "O": (h, h), "FC1": (f, h), "FC2": (h, f)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--models", default="13b,30b,66b")
    ap.add_argument("--s", default="0.3,0.4,0.5,0.6,0.7")
    ap.add_argument("--N", default="8,16,32")
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
    peak = None
    try:
        peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                           "MEASURED_PEAKS.json")))["hbm_gbs"]
    except Exception:
        pass
    stream = torch.cuda.current_stream()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    flush_rd = torch.zeros(64 << 20, dtype=torch.float32, device=dev)

    def timed(fn, steps):
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
        torch.cuda.synchronize()
        torch.cuda._sleep(2_000_000)   # device-side lead-in, as in bench.py (no host gap inside a step's events)
        for _ in range(2):
            flush.zero_()
            flush_rd.sum()
            fn()
        for i in range(steps):
            flush.zero_()
            flush_rd.sum()
            evs[i][0].record(stream)
            fn()
            evs[i][1].record(stream)
        torch.cuda.synchronize()
        return [s.elapsed_time(e) * 1e3 for s, e in evs]   # us

    out = open(a.out, "a") if a.out else None
    rows = []
    gen = np.random.default_rng(7)
    for m in a.models.split(","):
        for lname, (M, K) in layers(m).items():
            for s in (float(x) for x in a.s.split(",")):
                W = synth.weight(M, K, s, seed=synth.DEFAULT_SEED)
                Wd = torch.from_numpy(W.view(np.int16)).to(dev)
                T = sp.encode(Wd)
                Wdense = Wd.view(torch.float16)
                del W
                for N in (int(x) for x in a.N.split(",")):
                    X = synth.activation(K, N, seed=synth.DEFAULT_SEED + 1)
                    Xd = torch.from_numpy(X.view(np.int16)).to(dev).view(torch.float16)
                    Y = torch.empty((M, N), dtype=torch.float16, device=dev)
                    ws = sp.workspace(M, K, N, dev)
                    for _ in range(3):
                        sp.spmm(T, Xd, Y, ws)
                    t = timed(lambda: sp.spmm(T, Xd, Y, ws), a.steps)
                    # parity on sampled rows (fp64 on the GPU, from the generator's dense W)
                    ridx = torch.from_numpy(gen.choice(M, size=min(128, M), replace=False)).to(dev)
                    Wr = Wdense[ridx].double()
                    Xf = Xd.double()
                    ref = Wr @ Xf
                    bound = 2e-3 * (Wr.abs() @ Xf.abs()) + 1e-3
                    err = (Y[ridx].double() - ref).abs()
                    ok = bool((err <= bound).all())
                    Yc = torch.empty((M, N), dtype=torch.float16, device=dev)
                    for _ in range(3):
                        torch.mm(Wdense, Xd, out=Yc)
                    tc = timed(lambda: torch.mm(Wdense, Xd, out=Yc), a.steps)
                    nbytes = sp.algorithmic_bytes(T, N)
                    us, usc = statistics.median(t), statistics.median(tc)
                    gbs = nbytes / (us * 1e-6) / 1e9
                    rec = {"model": f"OPT-{m.upper()}" if m in OPT else m, "layer": lname, "M": M, "K": K, "N": N, "sparsity": s,
                           "us_median": us, "us_mean": statistics.mean(t), "gbs": gbs,
                           "frac_measured_peak": gbs / peak if peak else None, "frac_8tbs": gbs / 8000.0,
                           "tflops_dense_equiv": 2 * M * K * N / (us * 1e-6) / 1e12,
                           "cublas_us_median": usc, "speedup_vs_cublas": usc / us, "parity_ok": ok,
                           "parity_max_err_over_bound": float((err - bound).max()),
                           "algorithmic_bytes": nbytes}
                    rows.append(rec)
                    line = json.dumps(rec)
                    print(line, flush=True)
                    if out:
                        out.write(line + "\n")
                        out.flush()
                    del Y, Yc, ws, Xd
                del T, Wd, Wdense
                torch.cuda.empty_cache()
    print(f"{'model':8s} {'layer':4s} {'M':>6s} {'K':>6s} {'N':>3s} {'s':>4s} {'us':>8s} {'GB/s':>7s} "
          f"{'frac':>5s} {'cuBLAS':>8s} {'x':>5s} ok")
    for r in rows:
        print(f"{r['model']:8s} {r['layer']:4s} {r['M']:6d} {r['K']:6d} {r['N']:3d} {r['sparsity']:4.1f} "
              f"{r['us_median']:8.1f} {r['gbs']:7.0f} {r['frac_measured_peak'] or 0:5.2f} {r['cublas_us_median']:8.1f} "
              f"{r['speedup_vs_cublas']:5.2f} {'ok' if r['parity_ok'] else 'FAIL'}")
    bad = [r for r in rows if not r["parity_ok"]]
    if bad:
        print(f"PARITY FAILURES: {len(bad)}")
        sys.exit(1)


if __name__ == "__main__":
    main()
