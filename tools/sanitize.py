"""One SpMM call per (kernel, shape) for compute-sanitizer: config 1 and
1024 x 1024, N = 8 / 16 (decoupled-warp kernel) and N = 32 (tcgen05), plus a split-rowblock
case (grid capped at 3 CTAs) and a ragged shape. Checks the result against the oracle too."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import oracle, synth
import paper_conf_eurosys_fanydlgww025_b200 as sp
from tests.helpers import to_dev, f16_bits, north_star_bound, assert_within

cases = [(256, 256, 8, 0), (256, 256, 32, 0), (1024, 1024, 16, 0), (1024, 1024, 32, 0), (1024, 1024, 16, 3),
         (1024, 1024, 32, 3), (200, 330, 13, 0)]
for M, K, N, ctas in cases:
    sp.set_option("max_ctas", ctas)
    W = synth.weight(M, K, 0.5, seed=M + N); X = synth.activation(K, N, seed=1)
    T = sp.encode(to_dev(W))
    Y = sp.spmm(T, to_dev(X)); torch.cuda.synchronize()
    R = oracle.encode(W)
    assert np.array_equal(T.bitmap.cpu().numpy().view(np.uint64), R.bitmap)
    assert_within(f16_bits(Y), oracle.spmm_f64(R, X), north_star_bound(W, X), f"{M}x{K}x{N}")
    print(f"ok {M}x{K}x{N} ctas={ctas}", flush=True)
sp.set_option("max_ctas", 0)
