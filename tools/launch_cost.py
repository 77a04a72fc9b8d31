"""Experiment: event-timed cost of the SpMM launch itself (debug build, SPINFER_DEBUG_MODE=16 = exit after
set-up) after an L2 flush and back to back, next to the full kernel. Usage: python tools/launch_cost.py"""
import os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
os.environ.setdefault("SPINFER_LIB", os.path.join(ROOT, "paper_conf_eurosys_fanydlgww025_b200", "libspinfer_dbg.so"))
import numpy as np, torch
import synth
import paper_conf_eurosys_fanydlgww025_b200 as sp
M, K, N = 28672, 8192, 16
T = sp.encode(torch.from_numpy(synth.weight(M, K, 0.5).view(np.int16)).cuda())
X = torch.from_numpy(synth.activation(K, N).view(np.int16)).cuda()
Y = torch.empty((M, N), dtype=torch.float16, device="cuda"); ws = sp.workspace(M, K, N, "cuda")
fl = torch.empty(256 << 20, dtype=torch.uint8, device="cuda"); fr = torch.zeros(64 << 20, device="cuda")
s = torch.cuda.current_stream()
def t(mode, flush, n=25):
    os.environ["SPINFER_DEBUG_MODE"] = str(mode)
    r = []
    for i in range(n):
        if flush:
            fl.zero_(); fr.sum()
        a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
        a.record(s); sp.spmm(T, X, Y, ws); b.record(s)
        torch.cuda.synchronize()
        if i >= 5: r.append(a.elapsed_time(b) * 1e3)
    return statistics.median(r)
for k in (os.environ.get("SPINFER_KERNEL", "tc"),):
    print(k, "launch-only after flush %.2f us, back-to-back %.2f us; full after flush %.2f, back-to-back %.2f" %
          (t(16, True), t(16, False), t(0, True), t(0, False)))
# host-side cost of one spmm call (no GPU wait)
import time
os.environ["SPINFER_DEBUG_MODE"] = "16"
torch.cuda.synchronize(); t0 = time.perf_counter()
for _ in range(200): sp.spmm(T, X, Y, ws)
t1 = time.perf_counter(); torch.cuda.synchronize()
print("host time per spmm call: %.1f us" % ((t1 - t0) / 200 * 1e6))
