"""Time the SpMM on a list of shapes (development aid): median µs with a cold L2 (flush before
each call) and back to back (warm L2), plus the library options given as name=value args.
Usage: python tools/shape_time.py MxKxN[,MxKxN...] [s=0.5] [name=value ...]"""
import os, sys, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import synth
import paper_conf_eurosys_fanydlgww025_b200 as sp
from tests.helpers import to_dev

shapes = [tuple(int(x) for x in t.split("x")) for t in sys.argv[1].split(",")]
s = 0.5
for a in sys.argv[2:]:
    k, v = a.split("=")
    if k == "s":
        s = float(v)
    else:
        sp.set_option(k, v if k == "kernel" else int(v))
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for (M, K, N) in shapes:
    T = sp.encode(to_dev(synth.weight(M, K, s, seed=3)))
    X = to_dev(synth.activation(K, N, seed=4)).view(torch.float16)
    Y = torch.empty((M, N), dtype=torch.float16, device="cuda")
    ws = sp.workspace(M, K, N)
    for _ in range(5):
        sp.spmm(T, X, Y, ws=ws)
    res = {}
    for mode in ("cold", "warm"):
        ts = []
        torch.cuda.synchronize()
        torch.cuda._sleep(2_000_000)
        for i in range(30):
            if mode == "cold":
                flush.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); sp.spmm(T, X, Y, ws=ws); b.record()
            ts.append((a, b))
        torch.cuda.synchronize()
        res[mode] = statistics.median([x.elapsed_time(y) * 1e3 for x, y in ts[5:]])
    nb = sp.algorithmic_bytes(T, N)
    print(f"{M}x{K}x{N} s={s}: cold {res['cold']:.1f} us ({nb / res['cold'] / 1e3:.0f} GB/s), warm {res['warm']:.1f} us", flush=True)
