"""GPU SpMM parity against the fp64 CPU oracle (-m gpu), through the C ABI.

Tolerance (BASELINE.json north_star): |Y_gpu - Y_ref| <= 2e-3 (|W||X|)_ij + 1e-3.
Bit-exact where the mathematics fixes the result (integer inputs, identity, s = 1).
"""
import numpy as np
import pytest

import oracle
import synth
from tests.helpers import use_kernel, max_ctas, assert_within, f16_bits, f64, north_star_bound, to_dev

pytestmark = pytest.mark.gpu


def _sp():
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    return sp


def run_case(M, K, N, s, seed=1, mode="uniform"):
    import torch
    sp = _sp()
    W = synth.weight(M, K, s, seed=seed, mode=mode)
    X = synth.activation(K, N, seed=seed + 1, mode=mode)
    T = sp.encode(to_dev(W))
    Y = sp.spmm(T, to_dev(X))
    torch.cuda.synchronize()
    R = oracle.encode(W)
    return W, X, f16_bits(Y), oracle.spmm_f64(R, X)


# Shapes chosen to exercise: one GT; a single rowblock split across many CTAs
# (long K); an odd number of GT rows (last rowblock has one GT row); several
# rowblocks with stream-K boundaries inside rowblocks; ragged stages (KG % G != 0).
SHAPES = [(64, 64), (256, 256), (128, 4096), (192, 320), (1024, 1024), (4096, 2048), (320, 1472)]


@pytest.mark.parametrize("kernel", ["default", "dw", "tc"])
@pytest.mark.parametrize("M,K", SHAPES)
@pytest.mark.parametrize("N", [8, 16, 24, 32])
def test_spmm_shapes(M, K, N, kernel, monkeypatch):
    """Both sm_100a kernels (mma.sync and tcgen05; the library picks by N) on every shape."""
    use_kernel(kernel, N, monkeypatch)
    W, X, Y, Yref = run_case(M, K, N, 0.5, seed=M + K + N)
    assert_within(Y, Yref, north_star_bound(oracle.decode(oracle.encode(W)), X), f"{M}x{K}x{N} {kernel}")


@pytest.mark.parametrize("kernel", ["dw", "tc"])
@pytest.mark.parametrize("N", [8, 16, 24, 32])
def test_spmm_integer_exact_both_kernels(N, kernel, monkeypatch):
    """P-S2 bit-exactness for each kernel explicitly (split-K fix-up included: 4 CTAs on a
    long K force rowblocks split across CTAs)."""
    use_kernel(kernel, locals().get("N", 16), monkeypatch)
    max_ctas(4)
    M, K = 384, 2048
    for seed in range(100, 200):
        W = synth.weight(M, K, 0.5, seed=seed, mode="int")
        X = synth.activation(K, N, seed=seed + 1, mode="int")
        R = oracle.encode(W)
        Yref = oracle.spmm_f64(R, X)
        if np.abs(Yref).max() <= 2048:
            break
    import torch
    sp = _sp()
    Y = f16_bits(sp.spmm(sp.encode(to_dev(W)), to_dev(X)))
    torch.cuda.synchronize()
    exp = Yref.astype(np.float16).view(np.uint16)
    assert np.array_equal(Y, exp), f"{kernel} N={N}: {int(np.count_nonzero(Y != exp))} mismatches"


@pytest.mark.parametrize("s", [0.0, 0.3, 0.4, 0.6, 0.7, 0.95])
def test_spmm_sparsities(s):
    W, X, Y, Yref = run_case(1024, 768, 16, s, seed=int(s * 1000))
    assert_within(Y, Yref, north_star_bound(W, X), f"s={s}")


def test_spmm_config1():
    W, X, Y, Yref = run_case(256, 256, 8, 0.5, seed=synth.DEFAULT_SEED)
    assert_within(Y, Yref, north_star_bound(W, X), "config 1")


@pytest.mark.parametrize("N", [8, 16, 32])
def test_spmm_integer_exact(N):
    """P-S2: integer W, X with |Y| <= 2048 -> every fp32 partial sum is exact and Y is
    representable in fp16, so the GPU result must equal the oracle bit for bit."""
    W, X, Y, Yref = run_case(1024, 1024, N, 0.5, seed=77, mode="int")
    assert np.max(np.abs(Yref)) <= 2048
    assert np.array_equal(Yref, np.round(Yref))      # integers, exactly representable in fp16
    exp = Yref.astype(np.float16).view(np.uint16)
    assert np.array_equal(Y, exp)


def test_spmm_identity_and_empty():
    import torch
    sp = _sp()
    I = np.zeros((512, 512), dtype=np.uint16)
    I[np.arange(512), np.arange(512)] = 0x3C00
    X = synth.activation(512, 16, seed=5)
    Y = f16_bits(sp.spmm(sp.encode(to_dev(I)), to_dev(X)))
    assert np.array_equal(Y, X)                      # W = I -> Y = X exactly
    T1 = sp.encode(to_dev(np.zeros((256, 512), dtype=np.uint16)))
    assert T1.n_values == 0
    Y1 = f16_bits(sp.spmm(T1, to_dev(X)))
    assert np.all(Y1 == 0)                           # s = 1 -> Y = +0.0
    torch.cuda.synchronize()


def test_spmm_deterministic_and_workspace_reusable():
    """Repeated calls reuse one workspace (the fix-up counters return to zero) and
    give identical bits (fixed summation order of split-K partials)."""
    sp = _sp()
    W = synth.weight(2048, 2048, 0.5, seed=9)
    T = sp.encode(to_dev(W))
    X1 = to_dev(synth.activation(2048, 16, seed=1))
    X2 = to_dev(synth.activation(2048, 16, seed=2))
    a = f16_bits(sp.spmm(T, X1))
    b = f16_bits(sp.spmm(T, X2))
    c = f16_bits(sp.spmm(T, X1))
    assert np.array_equal(a, c) and not np.array_equal(a, b)
    ws = sp.workspace(2048, 2048, 16)
    cnt = ws[: 65536].view(dtype=__import__("torch").int32)
    assert int(cnt.abs().sum()) == 0


@pytest.mark.parametrize("N", [16, 32])
def test_spmm_config2_sampled_rows(N):
    """Full-size config 2 (M/K = 28672/8192, s = 0.5) in the launch bench.py times (N = 16:
    mma.sync kernel; N = 32: tcgen05 kernel); parity on sampled rows (incl. first/last rows
    and rowblock/CTA boundaries)."""
    import torch
    sp = _sp()
    M, K = 28672, 8192
    W = synth.weight(M, K, 0.5)
    X = synth.activation(K, N)
    T = sp.encode(to_dev(W))
    Y = f16_bits(sp.spmm(T, to_dev(X)))
    torch.cuda.synchronize()
    R = oracle.encode(W)
    rng = np.random.default_rng(0)
    rows = np.unique(np.concatenate([[0, 63, 64, 127, 128, M - 65, M - 64, M - 1],
                                     rng.integers(0, M, 120)])).astype(np.int32)
    Yref = oracle.spmm_rows_f64(R, X, rows)
    bound = 2e-3 * (np.abs(f64(W[rows])) @ np.abs(f64(X))) + 1e-3
    assert_within(Y[rows], Yref, bound, "config 2 sampled rows")
    # property at any size: every row against a cuBLAS fp32 product of the decoded W
    Wd = sp.decode(T).float()
    Yc = (Wd @ to_dev(X).view(torch.float16).float()).double().cpu().numpy()
    full_bound = 2e-3 * (Wd.abs() @ to_dev(X).view(torch.float16).float().abs()).double().cpu().numpy() + 1e-3
    assert np.all(np.abs(f64(Y) - Yc) <= full_bound + 1e-6 * np.abs(Yc))


@pytest.mark.parametrize("kernel", ["default", "dw", "tc"])
@pytest.mark.parametrize("N", [1, 2, 3, 5, 7, 12, 20, 31])
@pytest.mark.parametrize("M,K", [(256, 512), (320, 1472)])
def test_spmm_any_N(M, K, N, kernel, monkeypatch):
    """N not a multiple of 8: X is zero-padded to a multiple of 8 in the
    workspace, only the N real columns of Y are written (odd row strides included)."""
    use_kernel(kernel, N, monkeypatch)
    import torch
    sp = _sp()
    W = synth.weight(M, K, 0.5, seed=N)
    X = synth.activation(K, N, seed=N + 1)
    T = sp.encode(to_dev(W))
    guard = torch.full((M * N + 64,), 0x7777, dtype=torch.int16, device="cuda")   # canary after Y
    Y = guard[: M * N].view(M, N).view(torch.float16)
    sp.spmm(T, to_dev(X), Y)
    torch.cuda.synchronize()
    assert bool((guard[M * N:] == 0x7777).all()), "write past Y"
    Yref = oracle.spmm_f64(oracle.encode(W), X)
    assert_within(f16_bits(Y), Yref, north_star_bound(W, X), f"{M}x{K}x{N} {kernel}")


@pytest.mark.parametrize("N", [1, 5, 13])
def test_spmm_any_N_integer_exact(N):
    W, X, Y, Yref = run_case(384, 1024, N, 0.5, seed=300 + N, mode="int")
    assert np.max(np.abs(Yref)) <= 2048
    assert np.array_equal(Y, Yref.astype(np.float16).view(np.uint16))


@pytest.mark.parametrize("kernel", ["dw", "tc"])
@pytest.mark.parametrize("act", [None, "relu"])
@pytest.mark.parametrize("N", [5, 16, 32])
def test_spmm_bias_act(N, act, kernel, monkeypatch):
    """spinfer_spmm_ex: act(W X + bias) fused into the epilogue, on complete rowblocks and (4 CTAs
    on a long K) split rowblocks finished by the split-K fix-up; vs the oracle's C7 epilogue."""
    use_kernel(kernel, locals().get("N", 16), monkeypatch)
    max_ctas(4)
    import torch
    sp = _sp()
    M, K = 384, 2048
    W = synth.weight(M, K, 0.5, seed=N + 11)
    X = synth.activation(K, N, seed=N + 12)
    bias = synth.activation(M, 1, seed=N + 13).reshape(M)
    T = sp.encode(to_dev(W))
    Y = sp.spmm(T, to_dev(X), bias=to_dev(bias).view(torch.float16), act=act)
    torch.cuda.synchronize()
    Yref = oracle.bias_act_f64(oracle.spmm_f64(oracle.encode(W), X), bias, act)
    assert_within(f16_bits(Y), Yref, north_star_bound(W, X), f"bias act={act} N={N} {kernel}")
    if act == "relu":
        assert (f16_bits(Y) & 0x8000).sum() == 0 or np.all(f64(f16_bits(Y)) >= 0)


@pytest.mark.parametrize("kernel", ["dw", "tc"])
def test_spmm_bias_relu_integer_exact(kernel, monkeypatch):
    use_kernel(kernel, locals().get("N", 16), monkeypatch)
    max_ctas(4)
    import torch
    sp = _sp()
    M, K, N = 384, 2048, 16
    W = synth.weight(M, K, 0.5, seed=5, mode="int")
    X = synth.activation(K, N, seed=6, mode="int")
    bias = np.array([oracle.f64_to_f16(float((i % 9) - 4)) for i in range(M)], dtype=np.uint16)
    Y = sp.spmm(sp.encode(to_dev(W)), to_dev(X), bias=to_dev(bias).view(torch.float16), act="relu")
    torch.cuda.synchronize()
    Yref = oracle.bias_act_f64(oracle.spmm_f64(oracle.encode(W), X), bias, "relu")
    assert np.abs(Yref).max() <= 2048
    assert np.array_equal(f16_bits(Y), Yref.astype(np.float16).view(np.uint16))


def test_spmm_errors():
    import torch
    sp = _sp()
    T = sp.encode(to_dev(synth.weight(128, 128, 0.5)))
    X = torch.zeros((128, 65537), dtype=torch.float16, device="cuda")   # N > 65536
    with pytest.raises(sp.SpinferError) as e:
        sp.spmm(T, X)
    assert e.value.status == -1
    X = torch.zeros((128, 16), dtype=torch.float16, device="cuda")
    with pytest.raises(sp.SpinferError) as e:
        sp.spmm(T, X, ws=torch.zeros(16, dtype=torch.uint8, device="cuda"))
    assert e.value.status == -2
    Xbig = torch.zeros((128 * 16 + 8), dtype=torch.float16, device="cuda")
    with pytest.raises(sp.SpinferError) as e:
        sp.spmm(T, Xbig[1:1 + 128 * 16].view(128, 16))   # misaligned by 2 bytes
    assert e.value.status == -1
    cs = T.c_struct()
    import ctypes
    ws = sp.workspace(128, 128, 16)
    rc = sp.lib().spinfer_spmm_ex(ctypes.byref(cs), X.data_ptr(), X.data_ptr(), 128, 128, 16, None, 7,
                                  ws.data_ptr(), ws.numel(), None)
    assert rc == -1                                     # unknown activation
