"""Per-warp cycle breakdown of the decoupled-warp kernel (instrumented build; development aid).

Runs config 2 once with SPINFER_LIB=libspinfer_instr.so SPINFER_PROF=<file> and prints, per warp
role, the mean cycles waiting for data / scanning / decoding / flushing, GTs decoded, first-data
and exit times (clock64 of the SM)."""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("SPINFER_LIB", None) if False else None
os.environ["SPINFER_LIB"] = os.environ.get("SPINFER_PROF_LIB") or os.path.join(ROOT, "paper_conf_eurosys_fanydlgww025_b200", "libspinfer_instr.so")
out = os.path.join(ROOT, "gpurun_out", "dw_prof.bin")
import numpy as np
import torch
import synth
import paper_conf_eurosys_fanydlgww025_b200 as sp
from tests.helpers import to_dev

M, K, N = (int(a) for a in sys.argv[1:4]) if len(sys.argv) > 3 else (28672, 8192, 16)
s = float(sys.argv[4]) if len(sys.argv) > 4 else 0.5
W = synth.weight(M, K, s, seed=7); X = synth.activation(K, N, seed=8)
T = sp.encode(to_dev(W)); Xd = to_dev(X); ws = sp.workspace(M, K, N)
Y = torch.empty((M, N), dtype=torch.float16, device="cuda")
for _ in range(3): sp.spmm(T, Xd, Y, ws)
torch.cuda.synchronize()
os.environ["SPINFER_PROF"] = out
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda"); flush.zero_(); torch.cuda.synchronize()
sp.spmm(T, Xd, Y, ws); torch.cuda.synchronize()
raw = np.fromfile(out, dtype=np.int64)
P = len(torch.zeros(1)) and int(os.environ.get("DW_P", "148"))
a = raw[:1024 * 20 * 8].reshape(1024, 20, 8)[:P]
tr = raw[1024 * 20 * 8:1024 * 20 * 8 + 1024].reshape(256, 4).view(np.uint64)
nst = int(np.count_nonzero(tr[:, 0]))
names = ["wait", "scan", "decode", "flush", "GTs", "first", "exit", "arrive"]
cons = a[:, :16, :]
print(f"P={P} CTAs; consumer warps (mean over CTAs and warps; cycles):")
for k, n in enumerate(names):
    print(f"  {n:7s} mean {cons[:, :, k].mean():10.0f}  min {cons[:, :, k].min():10.0f}  max {cons[:, :, k].max():10.0f}")
print(f"producer: wait-empty mean {a[:, 16:, 0].mean():.0f}  issue {a[:, 16:, 1].mean():.0f}  exit mean {a[:, 16:, 6].mean():.0f} max {a[:, 16:, 6].max():.0f}")
ex = cons[:, :, 6].max(axis=1)
print(f"CTA exit: min {ex.min()} median {np.median(ex):.0f} max {ex.max()}")
per = cons[:, :, 2].sum(axis=1) / np.maximum(cons[:, :, 4].sum(axis=1), 1)
print(f"decode cycles per GT per warp: {per.mean():.0f}  scan per GT: {(cons[:, :, 1].sum(axis=1) / np.maximum(cons[:, :, 4].sum(axis=1), 1)).mean():.0f}")
print("CTA 0 stage trace (cycles from entry): i  prod_wait_start  issued  first_wake  released  | land-issue  release-wake")
for i in range(min(nst, 256)):
    w = int(~tr[i, 1]) if tr[i, 1] else 0
    print(f"  {i:3d} {int(tr[i,3]):7d} {int(tr[i,0]):7d} {w:7d} {int(tr[i,2]):7d}   | {w - int(tr[i,0]):6d} {int(tr[i,2]) - w:6d}")
print("CTA 0 warps:")
for w in range(20):
    print("  w%2d " % w + " ".join(f"{n}={a[0, w, k]}" for k, n in enumerate(names)))
ev = raw[1024 * 20 * 8 + 256 * 4:1024 * 20 * 8 + 256 * 4 + 16 * 64 * 6].reshape(16, 64, 6)
for w in (0, 5):
    print(f"warp {w} events (cycles): own-stage k: wait_start +wait +header/seg +scan +decode +arrive")
    for k in range(64):
        e = ev[w, k]
        if e[0] == 0 and e[1] == 0: continue
        d = [e[1] - e[0], e[2] - e[1], (e[3] - e[2]) if e[3] else 0, (e[4] - e[3]) if e[4] else 0, (e[5] - e[4]) if e[5] else 0]
        print(f"  {k:2d} t={e[0]:7d} " + " ".join(f"{x:6d}" for x in d))
# CTA entry / exit (globaltimer ns) relative to the first CTA entry
kGtOff = 1024 * 20 * 8 + 256 * 4 + 16 * 64 * 6
gt = raw[kGtOff:kGtOff + 1024 * 4].reshape(1024, 4)[:P].astype(np.int64)
t0 = gt[:, 0].min()
ent = (gt[:, 0] - t0) / 1e3
ex_c, ex_p, ex_r = (gt[:, 1] - t0) / 1e3, (gt[:, 2] - t0) / 1e3, (gt[:, 3] - t0) / 1e3
print(f"CTA entry (us after first): min {ent.min():.2f} median {np.median(ent):.2f} max {ent.max():.2f}")
print(f"consumer exit (us): min {ex_c.min():.2f} median {np.median(ex_c):.2f} max {ex_c.max():.2f}; producer max {ex_p.max():.2f}; reducer max {ex_r.max():.2f}")
o = np.argsort(ent)
print("latest entries:", [(int(i), round(float(ent[i]), 2)) for i in o[-8:]])
