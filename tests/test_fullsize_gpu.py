"""Bit-exact parity at BASELINE.json's full sizes (-m gpu), through the C ABI, every output.

Integer inputs (synth "int" mode: W in {-2,-1,1,2}, X in {-1,0,1}) make every fp32 partial sum
exact in any order, and |Y| <= 2048 makes every output exactly representable in fp16, so the
GPU result must equal the fp64 oracle bit for bit (P-S2) — a dropped, duplicated or misplaced
product changes an output by >= 1, far above fp16's ulp at these magnitudes, and fails here
(the north_star tolerance at K = 8192 is ~2.0 absolute and would not see it).

One oracle run per shape serves every kernel and N: X has 32 columns, the N-column cases use
its first N (Y[:, :N] = W X[:, :N]). The grid caps force many units per CTA (3584 at 8 CTAs on
config 2: long stage walks, large descriptor/segment counts, 32-bit unit arithmetic) and
unaligned stream-K splits (147 CTAs).
"""
import numpy as np
import pytest

import oracle
import synth
from tests.helpers import f16_bits, max_ctas, to_dev, use_kernel

pytestmark = pytest.mark.gpu


def _case(M, K, seed):
    W = synth.weight(M, K, 0.5, seed=seed, mode="int")
    X = synth.activation(K, 32, seed=seed + 1, mode="int")
    Yref = oracle.spmm_f64(oracle.encode(W), X)
    assert np.abs(Yref).max() <= 2048 and np.array_equal(Yref, np.round(Yref))
    return W, X, Yref.astype(np.float16).view(np.uint16)


@pytest.fixture(scope="module")
def config2():
    """BASELINE.json configs[1]: M/K = 28672/8192 (OPT-30B FC1-like), s = 0.5."""
    return _case(28672, 8192, 2002)


@pytest.fixture(scope="module")
def opt66_fc2():
    """OPT-66B FC2 (M/K = 9216/36864), the longest K of the paper's models."""
    return _case(9216, 36864, 6602)


def _run(W, X, N, kernel, ctas):
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    use_kernel(kernel, N)
    if ctas:
        max_ctas(ctas)
    T = sp.encode(to_dev(W))
    Xd = to_dev(np.ascontiguousarray(X[:, :N]))
    ws = sp.workspace(T.M, T.K, N)
    Y = f16_bits(sp.spmm(T, Xd, ws=ws))
    torch.cuda.synchronize()
    assert sp.check(ws) == 0
    return Y


@pytest.mark.parametrize("kernel,N,ctas", [
    ("default", 16, 0), ("default", 32, 0), ("dw", 8, 0), ("tc", 16, 0), ("default", 24, 0),
    ("dw", 16, 8), ("tc", 32, 8), ("dw", 16, 147), ("tc", 32, 147), ("dw", 13, 0), ("tc", 27, 0),
    ("dw", 32, 0), ("dw", 24, 147), ("dw", 32, 8)])
def test_config2_bit_exact(config2, kernel, N, ctas):
    W, X, exp = config2
    Y = _run(W, X, N, kernel, ctas)
    bad = np.count_nonzero(Y != exp[:, :N])
    assert bad == 0, f"{kernel} N={N} ctas={ctas}: {bad} of {Y.size} outputs differ"


@pytest.mark.parametrize("kernel,N", [("dw", 16), ("tc", 16), ("tc", 32), ("dw", 32)])
def test_opt66_fc2_bit_exact(opt66_fc2, kernel, N):
    W, X, exp = opt66_fc2
    Y = _run(W, X, N, kernel, 0)
    bad = np.count_nonzero(Y != exp[:, :N])
    assert bad == 0, f"{kernel} N={N}: {bad} of {Y.size} outputs differ"
