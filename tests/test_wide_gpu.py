"""GPU parity of the wide-X (N > 32, prefill) kernel against the fp64 oracle, through the C ABI.

The kernel decodes each 128 x 64 W tile into shared memory and multiplies it on tcgen05 with up to
two 256-column sub-tiles per output tile, so the cases cover: one sub-tile (N <= 256), two equal
sub-tiles (256 < N <= 512), several column tiles (N > 512), N not a multiple of 16 / 64 (TMA
zero-fill past N, masked stores) and not a multiple of 8 (the zero-padded X copy), ragged M and K,
a grid capped below the tile count (persistent CTAs walking several tiles, accumulator reuse), the
fused bias / ReLU epilogue, and corrupt input (reported, not faulting). Integer inputs make the
result exact (P-S2): compared bit for bit.
"""
import numpy as np
import pytest

import oracle
import synth
from tests.helpers import assert_within, f16_bits, max_ctas, north_star_bound, to_dev

pytestmark = pytest.mark.gpu


def _run(M, K, N, s=0.5, mode="uniform", seed=1, bias=None, act=None):
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    W = synth.weight(M, K, s, seed=seed, mode=mode)
    X = synth.activation(K, N, seed=seed + 1, mode=mode)
    T = sp.encode(to_dev(W))
    ws = sp.workspace(M, K, N)
    Y = sp.spmm(T, to_dev(X), ws=ws, bias=bias, act=act)
    torch.cuda.synchronize()
    assert sp.check(ws) == 0
    return W, X, f16_bits(Y)


@pytest.mark.parametrize("M,K,N", [(128, 64, 64), (256, 256, 48), (1024, 1024, 128), (1000, 700, 100), (384, 2048, 512),
                                   (256, 512, 600), (512, 512, 40), (200, 330, 37), (1024, 1024, 1024),
                                   (130, 1000, 257), (64, 4096, 33), (640, 576, 1100)])
def test_wide_parity(M, K, N):
    W, X, Y = _run(M, K, N, seed=M + N)
    Yref = oracle.spmm_f64(oracle.encode(W), X)
    assert_within(Y, Yref, north_star_bound(W, X), f"wide {M}x{K}x{N}")


@pytest.mark.parametrize("M,K,N,ctas", [(1024, 4096, 256, 0), (640, 2048, 520, 0), (768, 1024, 1536, 5),
                                        (2048, 512, 384, 3)])
def test_wide_integer_exact(M, K, N, ctas):
    if ctas:
        max_ctas(ctas)
    W, X, Y = _run(M, K, N, mode="int", seed=M + K + N)
    Yref = oracle.spmm_f64(oracle.encode(W), X)
    assert np.abs(Yref).max() <= 2048
    exp = Yref.astype(np.float16).view(np.uint16)
    assert np.array_equal(Y, exp), f"{int(np.count_nonzero(Y != exp))} mismatches"


@pytest.mark.parametrize("s", [0.0, 0.3, 0.7, 0.95])
def test_wide_sparsities(s):
    W, X, Y = _run(512, 768, 320, s=s, seed=int(1000 * s) + 3)
    Yref = oracle.spmm_f64(oracle.encode(W), X)
    assert_within(Y, Yref, north_star_bound(W, X), f"wide s={s}")


@pytest.mark.parametrize("act", [None, "relu"])
def test_wide_bias_act(act):
    import torch
    M, K, N = 300, 640, 200
    b = synth.activation(M, 1, seed=9).reshape(M)
    W, X, Y = _run(M, K, N, seed=11, bias=to_dev(b).view(torch.float16), act=act)
    Yref = oracle.spmm_f64(oracle.encode(W), X) + b.view(np.float16).astype(np.float64)[:, None]
    if act == "relu":
        Yref = np.maximum(Yref, 0.0)
    assert_within(Y, Yref, north_star_bound(W, X) + 1e-3, f"wide bias act={act}")


def test_wide_config2_sampled_rows():
    """The config-2 weight (28672 x 8192, s = 0.5) at N = 1024, integer inputs: every output of
    64 sampled rows (first / last rows, rowblock and tile boundaries) bit-exact."""
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    M, K, N = 28672, 8192, 1024
    W = synth.weight(M, K, 0.5, seed=4242, mode="int")
    X = synth.activation(K, N, seed=4243, mode="int")
    T = sp.encode(to_dev(W))
    Y = f16_bits(sp.spmm(T, to_dev(X)))
    torch.cuda.synchronize()
    rng = np.random.default_rng(1)
    rows = np.unique(np.concatenate([[0, 127, 128, 2047, 2048, M - 129, M - 128, M - 1],
                                     rng.integers(0, M, 56)])).astype(np.int32)
    Yref = oracle.spmm_rows_f64(oracle.encode(W), X, rows)
    assert np.abs(Yref).max() <= 2048
    exp = Yref.astype(np.float16).view(np.uint16)
    assert np.array_equal(Y[rows], exp), f"{int(np.count_nonzero(Y[rows] != exp))} mismatches"


def test_wide_corrupt_input_reported():
    import dataclasses
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    M, K, N = 256, 512, 128
    W = synth.weight(M, K, 0.5, seed=5, mode="int")
    X = to_dev(synth.activation(K, N, seed=6, mode="int"))
    T = sp.encode(to_dev(W))
    ws = sp.workspace(M, K, N)
    for bad in (dataclasses.replace(T, max_gt_values=8),
                dataclasses.replace(T, bitmap=T.bitmap.clone().index_fill_(0, torch.arange(64, 128, device="cuda"), -1))):
        sp.spmm(bad, X, ws=ws)
        torch.cuda.synchronize()
        assert sp.check(ws) != 0
    Y = f16_bits(sp.spmm(T, X, ws=ws))
    torch.cuda.synchronize()
    assert sp.check(ws) == 0
    exp = oracle.spmm_f64(oracle.encode(W), synth.activation(K, N, seed=6, mode="int")).astype(np.float16).view(np.uint16)
    assert np.array_equal(Y, exp)
