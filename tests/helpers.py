"""Shared test helpers: device transfer of fp16 bit arrays and the north_star tolerance."""
import numpy as np


def to_dev(a: np.ndarray, device="cuda"):
    import torch
    return torch.from_numpy(np.ascontiguousarray(a).view(np.int16)).to(device)


def f16_bits(t) -> np.ndarray:
    """torch fp16/int16 tensor -> numpy uint16 bit patterns."""
    import torch
    if t.dtype == torch.float16:
        t = t.view(torch.int16)
    return t.cpu().numpy().view(np.uint16)


def f64(a_bits: np.ndarray) -> np.ndarray:
    return a_bits.view(np.float16).astype(np.float64)


def north_star_bound(W_bits: np.ndarray, X_bits: np.ndarray) -> np.ndarray:
    """|Y_gpu - Y_ref| <= 2e-3 * (|W| |X|)_ij + 1e-3 (BASELINE.json north_star)."""
    return 2e-3 * (np.abs(f64(W_bits)) @ np.abs(f64(X_bits))) + 1e-3


def assert_within(Y_gpu_bits: np.ndarray, Y_ref: np.ndarray, bound: np.ndarray, what=""):
    y = f64(Y_gpu_bits)
    err = np.abs(y - Y_ref)
    bad = ~(err <= bound)
    if np.any(bad):
        idx = np.argwhere(bad)[:5]
        raise AssertionError(f"{what}: {int(bad.sum())} outputs out of tolerance, e.g. "
                             + ", ".join(f"{tuple(i)} gpu={y[tuple(i)]} ref={Y_ref[tuple(i)]} bound={bound[tuple(i)]:.3g}"
                                         for i in idx))


def use_kernel(kernel: str, N: int, monkeypatch=None):
    """Select the SpMM kernel for this test (spinfer_set_option SPINFER_OPT_KERNEL; the conftest
    fixture resets every option after the test): "default" = the library's choice, "dw" = the
    decoupled-warp mma.sync kernel (N <= 32; half-GroupTile mode above 16), "tc" = the tcgen05
    kernel."""
    import pytest
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    if kernel == "default":
        return
    if kernel == "dw" and N > 32:
        pytest.skip("the decoupled-warp kernel serves N <= 32")
    sp.set_option("kernel", kernel)


def max_ctas(n: int):
    """Cap the persistent grid (forces split rowblocks on small shapes)."""
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    sp.set_option("max_ctas", n)
