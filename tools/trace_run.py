"""Run one config-2 SpMM with SPINFER_TRACE and print the per-stage timeline of a few CTAs."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
os.environ.setdefault("SPINFER_LIB", os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "paper_conf_eurosys_fanydlgww025_b200", "libspinfer_instr.so"))
import paper_conf_eurosys_fanydlgww025_b200 as sp
M, K, N = 28672, 8192, 16
W = synth.weight(M, K, 0.5); X = synth.activation(K, N)
T = sp.encode(torch.from_numpy(W.view(np.int16)).cuda())
Xd = torch.from_numpy(X.view(np.int16)).cuda()
for _ in range(3): sp.spmm(T, Xd)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda"); flush.zero_(); torch.cuda.synchronize()
path = os.environ["SPINFER_TRACE"]
sp.spmm(T, Xd); torch.cuda.synchronize()
tr = np.fromfile(path, dtype=np.int64).reshape(4, 64, 16)
for p in range(2):
    t0 = tr[p, 0, 0]
    print(f"CTA {p}: columns = prod_issue | scan_full | scan_tbl | scan_done | cons_full | cons_scan | cons_rel | cons_done (cycles from first issue)")
    for i in range(0, 50):
        row = tr[p, i, :12]
        if row[0] == 0 and row[7] == 0 and i > 0: break
        print(i, " ".join(f"{(v - t0) if v else -1:8d}" for v in row))
