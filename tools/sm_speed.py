"""Per-SM decode speed of the decoupled-warp kernel, twice (instrumented build; development aid):
is the CTA-to-CTA spread a property of the SM it runs on?"""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ["SPINFER_LIB"] = os.path.join(ROOT, "paper_conf_eurosys_fanydlgww025_b200", "libspinfer_instr.so")
import numpy as np, torch, synth
import paper_conf_eurosys_fanydlgww025_b200 as sp
from tests.helpers import to_dev
M, K, N = 28672, 8192, 16
T = sp.encode(to_dev(synth.weight(M, K, 0.5, seed=7))); X = to_dev(synth.activation(K, N, seed=8))
ws = sp.workspace(M, K, N); Y = torch.empty((M, N), dtype=torch.float16, device="cuda")
out = os.path.join(ROOT, "gpurun_out", "sm_speed.bin")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
kGtOff = 1024 * 20 * 8 + 256 * 4 + 16 * 64 * 6
res = []
for rep in range(4):
    sp.spmm(T, X, Y, ws=ws); flush.zero_(); torch.cuda.synchronize()
    os.environ["SPINFER_PROF"] = out
    sp.spmm(T, X, Y, ws=ws); torch.cuda.synchronize()
    del os.environ["SPINFER_PROF"]
    raw = np.fromfile(out, dtype=np.int64)
    a = raw[:1024 * 20 * 8].reshape(1024, 20, 8)[:148]
    smid = raw[kGtOff + 4096: kGtOff + 4096 + 148]
    dec = a[:, :16, 2].mean(1)          # consumer decode cycles per CTA
    ex = a[:, :16, 6].max(1)            # exit
    per_sm = np.zeros(148); per_sm[smid] = dec
    per_sm_exit = np.zeros(148); per_sm_exit[smid] = ex
    res.append((per_sm, per_sm_exit))
    print(f"rep {rep}: decode min {dec.min():.0f} max {dec.max():.0f}; exit min {ex.min()} max {ex.max()}")
for i in range(1, 4):
    print(f"corr(rep0, rep{i}) decode per SM {np.corrcoef(res[0][0], res[i][0])[0,1]:.3f}  exit per SM {np.corrcoef(res[0][1], res[i][1])[0,1]:.3f}")
m = np.mean([r[0] for r in res], axis=0)
o = np.argsort(m)
print("fastest SMs", o[:10].tolist(), "slowest", o[-10:].tolist())
print("per-SM mean decode by SM id (TPC pairs):", np.round(m.reshape(-1, 2)[:20] / 1000, 1).tolist())
