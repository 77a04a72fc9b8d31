"""Wide-N (prefill) kernel: parity on small shapes and timing vs cuBLAS on the config-2 shape
(development aid). Usage: python tools/wide_quick.py [parity|time|all]"""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle, synth
import paper_conf_eurosys_fanydlgww025_b200 as sp
from tests.helpers import to_dev, f16_bits, north_star_bound, assert_within


def parity(M, K, N, s=0.5, mode="uniform", seed=1):
    W = synth.weight(M, K, s, seed=seed, mode=mode); X = synth.activation(K, N, seed=seed + 1, mode=mode)
    T = sp.encode(to_dev(W)); ws = sp.workspace(M, K, N)
    Y = sp.spmm(T, to_dev(X), ws=ws); torch.cuda.synchronize()
    err = sp.check(ws)
    R = oracle.encode(W); Yref = oracle.spmm_f64(R, X)
    if mode == "int":
        exp = Yref.astype(np.float16).view(np.uint16); got = f16_bits(Y)
        print(f"int {M}x{K}x{N}: bitexact={np.array_equal(got, exp)} mism={int(np.count_nonzero(got != exp))} err={err}", flush=True)
    else:
        try:
            assert_within(f16_bits(Y), Yref, north_star_bound(W, X), f"{M}x{K}x{N}")
            print(f"ok {M}x{K}x{N} err={err}", flush=True)
        except AssertionError as e:
            print(f"FAIL {M}x{K}x{N}: {str(e)[:300]}", flush=True)


def timeit(M, K, N, s=0.5, steps=10):
    W = synth.weight(M, K, s, seed=7); X = synth.activation(K, N, seed=8)
    T = sp.encode(to_dev(W)); Xd = to_dev(X).view(torch.float16); ws = sp.workspace(M, K, N)
    Y = torch.empty((M, N), dtype=torch.float16, device="cuda")
    Wd = sp.decode(T); Yc = torch.empty_like(Y)
    torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
    def tm(fn):
        for _ in range(2): fn()
        torch.cuda.synchronize(); ts = []
        for _ in range(steps):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); fn(); b.record(); ts.append((a, b))
        torch.cuda.synchronize()
        return statistics.median([x.elapsed_time(y) * 1e3 for x, y in ts])
    t_s = tm(lambda: sp.spmm(T, Xd, Y, ws=ws)); t_c = tm(lambda: torch.mm(Wd, Xd, out=Yc))
    tf = 2 * M * K * N / t_s / 1e6
    d = (Y.float() - Yc.float()).abs().max().item()
    print(f"time {M}x{K}x{N}: spmm {t_s:.1f} us ({tf:.0f} TFLOP/s dense-equiv), cuBLAS {t_c:.1f} us, ratio {t_c / t_s:.3f}, max|dY| {d:.3g}", flush=True)


if __name__ == "__main__":
    what = sys.argv[1] if len(sys.argv) > 1 else "all"
    for a in sys.argv[2:]:   # name=value library options
        k, v = a.split("=")
        sp.set_option(k, v if k == "kernel" else int(v))
    if what in ("all", "parity"):
        for M, K, N in [(128, 64, 64), (256, 256, 64), (1024, 1024, 128), (1000, 700, 100), (384, 2048, 512),
                        (256, 512, 600), (512, 512, 40), (200, 330, 37), (1024, 1024, 1024)]:
            parity(M, K, N, seed=M + N)
        parity(1024, 4096, 256, mode="int", seed=5)
        parity(640, 2048, 520, mode="int", seed=6)
    if what in ("all", "time"):
        for N in (64, 128, 256, 512, 1024, 2048, 4096, 8192):
            timeit(28672, 8192, N)
