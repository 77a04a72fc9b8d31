"""One SpMM call per (kernel, shape) for compute-sanitizer: config 1 and
1024 x 1024, N = 8 / 16 (decoupled-warp kernel) and N = 32 (tcgen05; and the decoupled-warp
kernel's half-GroupTile mode, kernel option 1), plus a split-rowblock case (grid capped at 3 CTAs)
and a ragged shape. Checks the result against the oracle too."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle, synth
import paper_conf_eurosys_fanydlgww025_b200 as sp
from tests.helpers import to_dev, f16_bits, north_star_bound, assert_within

cases = [(256, 256, 8, 0, 0), (256, 256, 32, 0, 0), (1024, 1024, 16, 0, 0), (1024, 1024, 32, 0, 0),
         (1024, 1024, 16, 3, 0), (1024, 1024, 32, 3, 0), (200, 330, 13, 0, 0),
         (256, 256, 32, 0, 1), (1024, 1024, 32, 3, 1), (200, 330, 27, 0, 1)]
for M, K, N, ctas, kern in cases:
    sp.set_option("max_ctas", ctas)
    sp.set_option("kernel", kern)
    W = synth.weight(M, K, 0.5, seed=M + N); X = synth.activation(K, N, seed=1)
    T = sp.encode(to_dev(W))
    Y = sp.spmm(T, to_dev(X)); torch.cuda.synchronize()
    R = oracle.encode(W)
    assert np.array_equal(T.bitmap.cpu().numpy().view(np.uint64), R.bitmap)
    assert_within(f16_bits(Y), oracle.spmm_f64(R, X), north_star_bound(W, X), f"{M}x{K}x{N}")
    print(f"ok {M}x{K}x{N} ctas={ctas} kernel={kern}", flush=True)
sp.set_option("max_ctas", 0)
sp.set_option("kernel", 0)
