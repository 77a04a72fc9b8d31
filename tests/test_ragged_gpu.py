"""Shapes that are not multiples of 64 (DESIGN reading A8: zero-padded to
whole GroupTiles) on the GPU path: encode bit-exact vs the oracle, decode round trip, SpMM parity on
both kernels (including K not a multiple of 8, N not a multiple of 8, split-K fix-up on a ragged
last rowblock), a write-past-Y canary, and the row partition with a ragged tail."""
import numpy as np
import pytest

import oracle
import synth
from tests.helpers import use_kernel, max_ctas, assert_within, f16_bits, north_star_bound, to_dev

pytestmark = pytest.mark.gpu

SHAPES = [(100, 70), (65, 64), (64, 65), (200, 1000), (1, 300), (333, 777), (1000, 130)]


@pytest.mark.parametrize("M,K", SHAPES)
def test_ragged_encode_bit_exact_and_decode(M, K):
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    W = synth.weight(M, K, 0.5, seed=M * 7 + K)
    T = sp.encode(to_dev(W))
    R = oracle.encode(W)
    assert (T.n_values, T.nnz) == (R.n_values, R.nnz)
    assert np.array_equal(T.gtile_offset.cpu().numpy(), R.gtile_offset)
    assert np.array_equal(T.bitmap.cpu().numpy().view(np.uint64), R.bitmap)
    assert np.array_equal(T.values[:T.n_values].cpu().view(torch.int16).numpy().view(np.uint16), R.values)
    Wd = f16_bits(sp.decode(T))
    W0 = W.copy()
    W0[(W0 & 0x7FFF) == 0] = 0
    assert np.array_equal(Wd, W0)


@pytest.mark.parametrize("kernel", ["dw", "tc"])
@pytest.mark.parametrize("N", [3, 16, 32])
@pytest.mark.parametrize("M,K", SHAPES)
def test_ragged_spmm(M, K, N, kernel, monkeypatch):
    use_kernel(kernel, locals().get("N", 16), monkeypatch)
    max_ctas(3)          # split rowblocks, ragged last one included
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    W = synth.weight(M, K, 0.5, seed=M + K + N)
    X = synth.activation(K, N, seed=N)
    T = sp.encode(to_dev(W))
    guard = torch.full((M * N + 64,), 0x7777, dtype=torch.int16, device="cuda")
    Y = guard[: M * N].view(M, N).view(torch.float16)
    sp.spmm(T, to_dev(X), Y)
    torch.cuda.synchronize()
    assert bool((guard[M * N:] == 0x7777).all()), "write past Y"
    Yref = oracle.spmm_f64(oracle.encode(W), X)
    assert_within(f16_bits(Y), Yref, north_star_bound(W, X), f"{M}x{K}x{N} {kernel}")


@pytest.mark.parametrize("world", [2, 3, 4])
def test_ragged_tp_rows(world):
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    M, K, N = 1000, 300, 16                               # 16 GT rows, the last one 40 rows tall
    W = synth.weight(M, K, 0.5, seed=world)
    X = synth.activation(K, N, seed=1)
    T = sp.encode(to_dev(W))
    Y = torch.full((M, N), float("nan"), dtype=torch.float16, device="cuda")
    tot = 0
    for r in range(world):
        b, c = sp.tp_rows(M, world, r)
        assert (b, c) == oracle.tp_rows(M, world, r)
        tot += c
        sp.spmm_tp(T.shard(b, c), to_dev(X).view(torch.float16), Y, M, world, r)
    torch.cuda.synchronize()
    assert tot == M
    assert_within(f16_bits(Y), oracle.spmm_f64(oracle.encode(W), X), north_star_bound(W, X), f"tp {world}")


@pytest.mark.parametrize("kernel,N", [("dw", 16), ("tc", 32), ("default", 100)])
@pytest.mark.parametrize("act", [None, "relu"])
def test_ragged_bias_act(kernel, N, act):
    """Fused bias / ReLU with a ragged M (rows past M are padding: they read no bias and are not
    stored), for the three kernels (N = 100: the wide kernel)."""
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    use_kernel(kernel, N)
    M, K = 100, 70
    W = synth.weight(M, K, 0.5, seed=77)
    X = synth.activation(K, N, seed=78)
    b = synth.activation(M, 1, seed=79).reshape(M)
    T = sp.encode(to_dev(W))
    bias = to_dev(b).view(torch.float16)
    Y = f16_bits(sp.spmm(T, to_dev(X), bias=bias, act=act))
    torch.cuda.synchronize()
    Yref = oracle.spmm_f64(oracle.encode(W), X) + b.view(np.float16).astype(np.float64)[:, None]
    if act == "relu":
        Yref = np.maximum(Yref, 0.0)
    assert_within(Y, Yref, north_star_bound(W, X) + 1e-3, f"ragged bias {kernel} N={N} act={act}")
