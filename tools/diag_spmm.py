"""Diagnostic: compare spinfer SpMM with cuBLAS fp32 on the decoded W; report bad rows by rowblock/CTA."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_eurosys_fanydlgww025_b200 as sp

def run(M, K, N, s, max_ctas=None):
    if max_ctas: os.environ["SPINFER_MAX_CTAS"] = str(max_ctas)
    else: os.environ.pop("SPINFER_MAX_CTAS", None)
    W = synth.weight(M, K, s); X = synth.activation(K, N)
    Wd = torch.from_numpy(W.view(np.int16)).cuda(); Xd = torch.from_numpy(X.view(np.int16)).cuda().view(torch.float16)
    T = sp.encode(Wd)
    Y = sp.spmm(T, Xd, ws=torch.zeros(sp.workspace_bytes(M, K, N) + 256, dtype=torch.uint8, device="cuda")).float()
    Dw = sp.decode(T).float()
    Yr = Dw @ Xd.float()
    bound = 2e-3 * (Dw.abs() @ Xd.float().abs()) + 1e-3
    bad = ((Y - Yr).abs() > bound).any(dim=1).cpu().numpy()
    KG = K // 64; MG = M // 64; nRB = (MG + 1) // 2; U = nRB * KG
    P = min(int(max_ctas or 148), U)
    badrows = np.flatnonzero(bad)
    rbs = sorted(set((badrows // 128).tolist()))
    print(f"M/K/N={M}/{K}/{N} s={s} P={P} U={U} upc={U/P:.1f}: bad rows {len(badrows)}/{M}; bad rowblocks {len(rbs)}/{nRB}", flush=True)
    def owner(u): return ((u + 1) * P - 1) // U
    for rb in rbs[:12]:
        pf, pl = owner(rb * KG), owner((rb + 1) * KG - 1)
        rows_in = badrows[(badrows // 128) == rb]
        print(f"   rb {rb}: contributors {pf}..{pl} ({'complete' if pf == pl else 'split'}); bad rows in rb: {len(rows_in)} first {rows_in[:4].tolist()}")
    return len(badrows)

for args in [(4096, 2048, 16, 0.5, None), (1024, 4096, 16, 0.5, 4), (1024, 4096, 16, 0.5, 3), (256, 8192, 16, 0.5, 2),
             (2048, 2048, 16, 0.5, 1), (28672, 8192, 16, 0.5, None)]:
    run(*args)
