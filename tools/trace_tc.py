"""Per-stage timeline of the tcgen05 SpMM kernel (instrumented build libspinfer_instr.so, SPINFER_TRACE).

trace[CTA 0..3][stage 0..63][warp 0..19][ev 0..3] = clock64; stage 63 = kernel-level events.
Warps: 0-15 decode (ev0 wait-scan start, ev1 scanned seen, ev2 A published, ev3 after epilogue),
16 MMA (ev0 wait-full start, ev1 full seen, ev2 all A seen + MMAs issued, ev3 commits issued),
17-18 scan (ev0 wait start, ev1 full seen, ev3 table published), 19 producer (ev0 before the
empty wait, ev1 copies issued). Usage: python tools/trace_tc.py [M K N]
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
os.environ.setdefault("SPINFER_KERNEL", "tc")
import paper_conf_eurosys_fanydlgww025_b200 as sp  # noqa: E402

M, K, N = (int(x) for x in sys.argv[1:4]) if len(sys.argv) > 3 else (28672, 8192, 16)
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

PW = 16   # producer warp (decode warps 0-15; k-team leaders issue the MMAs)
for p in range(2):
    k = tr[p, 63]
    t0 = k[:, 0][k[:, 0] > 0].min()
    R = lambda v: int(v - t0) if v > 0 else -1  # noqa: E731
    nst = int(np.count_nonzero(tr[p, :63, PW, 1]))
    print(f"=== CTA {p}: {nst} stages; entry..sync {R(k[:,1].max())}, exit max {max(R(v) for v in k[:, 3])}")
    print(" st  prodW  issued  dataSeen(min..max)  MMAissued(min..max)")
    for i in range(nst):
        c = tr[p, i]
        cw1 = c[:16, 1]; cw2 = c[:16, 2]
        print(f"{i:3d} {R(c[PW,0]):7d} {R(c[PW,1]):7d} {R(cw1.min()):8d}..{R(cw1.max()):<8d} {R(cw2.min()):7d}..{R(cw2.max()):<7d}")
    a = tr[p, :nst, :16, :]
    wait = (a[:, :, 1] - a[:, :, 0]).sum(0)
    work = (a[:, :, 2] - a[:, :, 1]).sum(0)
    epi = (a[1:, :, 0] - a[:-1, :, 2]).sum(0)
    print("decode warps: wait-data sum", wait.tolist())
    print("              decode sum   ", work.tolist())
    print("              between sum  ", epi.tolist())
