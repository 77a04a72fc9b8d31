"""Per-warp-role cycle breakdown of the wide kernel (instrumented build; development aid).
Usage: python tools/wide_prof.py M K N"""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ["SPINFER_LIB"] = os.path.join(ROOT, "paper_conf_eurosys_fanydlgww025_b200", "libspinfer_instr.so")
import numpy as np, torch, synth
import paper_conf_eurosys_fanydlgww025_b200 as sp
from tests.helpers import to_dev
M, K, N = (int(x) for x in sys.argv[1:4])
T = sp.encode(to_dev(synth.weight(M, K, 0.5, seed=7))); X = to_dev(synth.activation(K, N, seed=8)).view(torch.float16)
ws = sp.workspace(M, K, N); Y = torch.empty((M, N), dtype=torch.float16, device="cuda")
sp.spmm(T, X, Y, ws=ws); torch.cuda.synchronize()
out = os.path.join(ROOT, "gpurun_out", "wide_prof.bin")
os.environ["SPINFER_PROF"] = out
sp.spmm(T, X, Y, ws=ws); torch.cuda.synchronize()
a = np.fromfile(out, dtype=np.int64).reshape(1024, 32, 4)
P = int(np.count_nonzero(a[:, 0, 3]))
a = a[:P]
roles = {"W prod": [0], "X prod": [1], "MMA": [2], "epilogue": [4, 5, 6, 7, 24, 25, 26, 27], "decode": list(range(8, 24))}
print(f"{M}x{K}x{N}: {P} CTAs; cycles (mean over CTAs): in-wait / out-wait / work / total")
for name, ws_ in roles.items():
    v = a[:, ws_, :].mean(axis=(0, 1))
    print(f"  {name:9s} {v[0]:10.0f} {v[1]:10.0f} {v[2]:10.0f} {v[3]:10.0f}")
