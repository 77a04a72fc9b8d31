"""Per-warp stage timeline of one config-2 SpMM (instrumented build, SPINFER_TRACE).

Layout written by the kernel: trace[CTA 0..3][stage 0..63][warp 0..19][ev 0..3] (clock64);
stage 63 holds kernel-level events (entry, after __syncthreads, main loop done, exit).
Prints, per CTA, where each consumer warp's time goes and the scan/producer timing.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
os.environ.setdefault("SPINFER_LIB", os.path.join(ROOT, "paper_conf_eurosys_fanydlgww025_b200", "libspinfer_instr.so"))
os.environ.setdefault("SPINFER_TRACE", "/tmp/spinfer_trace.bin")
import paper_conf_eurosys_fanydlgww025_b200 as sp  # noqa: E402

M, K, N = 28672, 8192, 16
W = synth.weight(M, K, 0.5)
X = synth.activation(K, N)
T = sp.encode(torch.from_numpy(W.view(np.int16)).cuda())
Xd = torch.from_numpy(X.view(np.int16)).cuda()
for _ in range(3):
    sp.spmm(T, Xd)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
flush.zero_()
torch.cuda.synchronize()
sp.spmm(T, Xd)
torch.cuda.synchronize()
tr = np.fromfile(os.environ["SPINFER_TRACE"], dtype=np.int64)[:4 * 64 * 20 * 4].reshape(4, 64, 20, 4)

NCW = 16
for p in range(2):
    k = tr[p, 63]
    t0 = k[:, 0][k[:, 0] > 0].min()
    rel = lambda v: (v - t0) if v > 0 else -1  # noqa: E731
    nst = int(max(np.count_nonzero(tr[p, :63, w, 3]) for w in range(NCW)))
    print(f"=== CTA {p}: {nst} stages; kernel: entry {rel(k[0,0])} sync {rel(k[0,1])} "
          f"loop-done(w0) {rel(k[0,2])} exit max {max(rel(v) for v in k[:, 3])}")
    print("warp  start   wait   work  epi+rel  gap   end   (cycles; sums over stages)")
    for w in range(NCW):
        a = tr[p, :nst, w, :]
        wait = int(np.sum(a[:, 1] - a[:, 0]))
        work = int(np.sum(a[:, 2] - a[:, 1]))
        epi = int(np.sum(a[:, 3] - a[:, 2]))
        gap = int(np.sum(a[1:, 0] - a[:-1, 3]))
        print(f"{w:4d} {rel(a[0,0]):6d} {wait:6d} {work:6d} {epi:7d} {gap:6d} {rel(k[w,3]):6d}")
    for w in (17, 18):   # scan warps (warp 16 = fix-up, 19 = producer)
        a = tr[p, :nst, w, :]
        wait = int(np.sum(a[:, 1] - a[:, 0]))
        busy = int(np.sum(a[:, 3] - a[:, 1]))
        pre = int(np.sum(a[:, 2] - a[:, 1]))
        print(f"scan {w}: wait {wait} scan {busy} per-stage scan {busy / max(nst, 1):.0f} "
              f"(load+prefix {pre / max(nst, 1):.0f}, stores+publish {(busy - pre) / max(nst, 1):.0f})")
    a = tr[p, :nst, 19, :]
    print(f"producer: first issue {rel(a[0,1])}, wait-on-empty sum {int(np.sum(a[:,1]-a[:,0]))}")
    print("stage  prod_issued  scan_full(17)  scan_done(17)  cons_wait_end(min..max over warps)  rel(max)")
    for i in range(0, nst, max(1, nst // 16)):
        c1 = tr[p, i, :NCW, 1]
        print(f"{i:4d} {rel(tr[p,i,19,1]):10d} {rel(tr[p,i,17,1]):10d} {rel(tr[p,i,17,3]):10d} "
              f"{rel(c1.min()):10d}..{rel(c1.max()):<10d} {rel(tr[p,i,:NCW,3].max()):10d}")

# per-stage release latency (decode done -> slot released) of a few consumer warps: segment
# ends (epilogue) stand out
for p in range(1):
    k = tr[p, 63]
    t0 = k[:, 0][k[:, 0] > 0].min()
    nst = int(max(np.count_nonzero(tr[p, :63, w, 3]) for w in range(NCW)))
    print(f"=== CTA {p} epilogue scan (ev3-ev2 per stage, cycles) for warps 0, 1, 8, 15")
    for i in range(nst):
        v = [int(tr[p, i, w, 3] - tr[p, i, w, 2]) for w in (0, 1, 8, 15)]
        if max(v) > 1500:
            print(f"stage {i:3d} start {int(tr[p, i, 0, 0] - t0):7d}  epi {v}  decode-done w0..w15 spread "
                  f"{int(tr[p, i, :NCW, 2].max() - tr[p, i, :NCW, 2].min())}")
