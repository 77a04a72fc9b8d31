"""One wide-kernel launch for ncu (development aid): python tools/wide_one.py M K N"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_eurosys_fanydlgww025_b200 as sp
from tests.helpers import to_dev
M, K, N = (int(x) for x in sys.argv[1:4])
T = sp.encode(to_dev(synth.weight(M, K, 0.5, seed=7))); X = to_dev(synth.activation(K, N, seed=8)).view(torch.float16)
ws = sp.workspace(M, K, N); Y = torch.empty((M, N), dtype=torch.float16, device="cuda")
for _ in range(3):
    sp.spmm(T, X, Y, ws=ws)
torch.cuda.synchronize()
