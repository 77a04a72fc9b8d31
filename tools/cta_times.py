"""Per-CTA entry / exit times of one config-2 SpMM on the global ns timer (instrumented build):
launch-to-first-CTA is not visible here, but the spread of entries (launch skew), of exits (load
imbalance / fix-up tail) and the event-timed kernel duration are. Usage: python tools/cta_times.py [N]"""
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

N = int(sys.argv[1]) if len(sys.argv) > 1 else 16
M, K = 28672, 8192
T = sp.encode(torch.from_numpy(synth.weight(M, K, 0.5).view(np.int16)).cuda())
Xd = torch.from_numpy(synth.activation(K, N).view(np.int16)).cuda()
for _ in range(3):
    sp.spmm(T, Xd)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
rd = torch.zeros(64 << 20, device="cuda")
base = 4 * 64 * 20 * 4
for rep in range(3):
    flush.zero_(); rd.sum()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); sp.spmm(T, Xd); e1.record()
    torch.cuda.synchronize()
    tr = np.fromfile(os.environ["SPINFER_TRACE"], dtype=np.int64)
    g = tr[base:base + 2 * 1024].reshape(1024, 2)
    smid = tr[base + 2 * 1024:base + 3 * 1024]
    live = g[:, 0] > 0
    g, smid = g[live], smid[live]
    t0 = g[:, 0].min()
    ent, ex = (g[:, 0] - t0) / 1e3, (g[:, 1] - t0) / 1e3
    print(f"rep {rep}: event {e0.elapsed_time(e1)*1e3:.1f} us; CTAs {len(g)}; entry spread {ent.max():.2f} us; "
          f"exit min/med/max {ex.min():.1f}/{np.median(ex):.1f}/{ex.max():.1f} us; "
          f"latest 5 exits (CTA: us) {[(int(i), round(float(ex[i]),1)) for i in np.argsort(-ex)[:5]]}")
    if rep == 2:
        order = np.argsort(smid)
        print("exit (us) by SM id:", " ".join(f"{int(smid[i])}:{ex[i]:.1f}" for i in order))
