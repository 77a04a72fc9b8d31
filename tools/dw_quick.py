"""Quick parity + timing of the default SpMM path on a few shapes (GPU box, development aid)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle, synth
import paper_conf_eurosys_fanydlgww025_b200 as sp
from tests.helpers import to_dev, f16_bits, north_star_bound, assert_within

def parity(M, K, N, s, seed=1, mode="uniform"):
    W = synth.weight(M, K, s, seed=seed, mode=mode); X = synth.activation(K, N, seed=seed + 1, mode=mode)
    T = sp.encode(to_dev(W)); Y = sp.spmm(T, to_dev(X)); torch.cuda.synchronize()
    R = oracle.encode(W); Yref = oracle.spmm_f64(R, X)
    if mode == "int":
        exp = Yref.astype(np.float16).view(np.uint16); ok = np.array_equal(f16_bits(Y), exp)
        print(f"int {M}x{K}x{N}: bitexact={ok} mism={int(np.count_nonzero(f16_bits(Y) != exp))}", flush=True)
    else:
        assert_within(f16_bits(Y), Yref, north_star_bound(oracle.decode(R), X), f"{M}x{K}x{N}")
        print(f"ok {M}x{K}x{N} s={s}", flush=True)

def timeit(M, K, N, s, steps=20):
    W = synth.weight(M, K, s, seed=7); X = synth.activation(K, N, seed=8)
    T = sp.encode(to_dev(W)); Xd = to_dev(X).view(torch.float16); ws = sp.workspace(M, K, N)
    Y = torch.empty((M, N), dtype=torch.float16, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(3): sp.spmm(T, Xd, Y, ws)
    torch.cuda.synchronize()
    ts = []
    for _ in range(steps):
        flush.zero_(); a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
        a.record(); sp.spmm(T, Xd, Y, ws); b.record(); torch.cuda.synchronize(); ts.append(a.elapsed_time(b) * 1e3)
    nb = sp.algorithmic_bytes(T, N)
    med = float(np.median(ts))
    print(f"time {M}x{K}x{N} s={s} kernel={sp.get_option('kernel')}: median {med:.1f} us mean {np.mean(ts):.1f} -> {nb/med/1e3:.0f} GB/s", flush=True)
    return Y

if __name__ == "__main__":
    what = sys.argv[1] if len(sys.argv) > 1 else "all"
    for a in sys.argv[2:]:   # name=value library options, e.g. kernel=tc stage_s=2
        k, v = a.split("=")
        sp.set_option(k, v if k == "kernel" else int(v))
    if what in ("all", "parity"):
        for (M, K, N) in [(256, 256, 8), (256, 256, 16), (64, 64, 16), (128, 4096, 16), (192, 320, 16), (1024, 1024, 16), (4096, 2048, 8), (320, 1472, 16), (100, 70, 5)]:
            parity(M, K, N, 0.5, seed=M + K + N)
        parity(384, 2048, 16, 0.5, seed=101, mode="int")
        for ctas in (3, 7, 16):
            sp.set_option("max_ctas", ctas)
            parity(384, 2048, 16, 0.5, seed=101, mode="int")
            parity(576, 1472, 8, 0.5, seed=102, mode="int")
            parity(192, 4160, 13, 0.5, seed=7)
        sp.set_option("max_ctas", 0)
    if what in ("all", "time"):
        for s in (0.5, 0.3, 0.7):
            timeit(28672, 8192, 16, s)
        timeit(28672, 8192, 8, 0.5)
