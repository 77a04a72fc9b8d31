"""Structured sparsity patterns and corrupt-input robustness of the SpMM (-m gpu, C ABI).

Patterns (bit-exact, integer inputs): the kernels' work per GroupTile varies with its value
count (stage byte counts, PopCount prefix, MaskedPopCount addresses), so uniform
random masks alone never reach the extremes: a completely dense GroupTile (4096 values, the
max_gt_values = 4096 stage size) next to an empty one (0 values: zero-byte copies), GT columns
alternating dense / empty, one dense row or column in a very sparse matrix, a GroupTile whose
only non-zero is its last bit, and fully dense / fully empty matrices.

Robustness (include/spinfer.h spinfer_spmm_check): a TCA-BME struct that contradicts its arrays
(max_gt_values understated, gtile_offset decreasing or past n_values, bitmaps with more set bits
than the values) must not fault or read out of bounds: the call completes, the workspace's error
word reports it, and the next valid call on the same workspace is exact with a clean word.
"""
import numpy as np
import pytest

import oracle
import synth
from tests.helpers import f16_bits, max_ctas, to_dev, use_kernel

pytestmark = pytest.mark.gpu

M, K = 384, 1024   # 6 GT rows x 16 GT columns


def _pattern(name):
    W = synth.weight(M, K, 0.0, seed=31, mode="int")           # dense integer values
    keep = synth.weight(M, K, 0.9, seed=32, mode="int") != 0   # 10% random background
    if name == "dense_next_to_empty":
        keep[0:64, 0:64] = True
        keep[0:64, 64:128] = False
        keep[64:128, 512:576] = True
    elif name == "alternating_gt_columns":
        for j in range(K // 64):
            keep[:, 64 * j: 64 * j + 64] = (j % 2 == 0)
    elif name == "dense_row":
        keep[:] = False
        keep[77, :] = True
        keep[200, 5] = True
    elif name == "dense_column":
        keep[:] = False
        keep[:, 1023] = True
        keep[:, 64] = True
    elif name == "last_bit_only":
        keep[:] = False
        keep[63::64, 63::64] = True      # the last position of every GroupTile (bit 63 of BT 63)
    elif name == "all_dense":
        keep[:] = True
    elif name == "all_empty":
        keep[:] = False
    W[~keep] = 0
    return W


PATTERNS = ["dense_next_to_empty", "alternating_gt_columns", "dense_row", "dense_column", "last_bit_only",
            "all_dense", "all_empty"]


@pytest.mark.parametrize("kernel", ["dw", "tc"])
@pytest.mark.parametrize("ctas", [0, 3])
@pytest.mark.parametrize("pattern", PATTERNS)
def test_structured_pattern_bit_exact(pattern, kernel, ctas):
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    N = 16
    use_kernel(kernel, N)
    if ctas:
        max_ctas(ctas)
    W = _pattern(pattern)
    X = synth.activation(K, N, seed=33, mode="int")
    R = oracle.encode(W)
    Yref = oracle.spmm_f64(R, X)
    assert np.abs(Yref).max() <= 2048
    T = sp.encode(to_dev(W))
    assert T.n_values == R.n_values and T.max_gt_values == R.max_gt_values
    ws = sp.workspace(M, K, N)
    Y = f16_bits(sp.spmm(T, to_dev(X), ws=ws))
    torch.cuda.synchronize()
    assert sp.check(ws) == 0
    exp = Yref.astype(np.float16).view(np.uint16)
    assert np.array_equal(Y, exp), f"{pattern} {kernel}: {int(np.count_nonzero(Y != exp))} mismatches"


def _corrupt(T, how):
    import dataclasses
    import torch
    off, bm = T.gtile_offset.clone(), T.bitmap.clone()
    mx = T.max_gt_values
    if how == "max_gt_understated":
        mx = 8
    elif how == "offset_decreasing":
        off[5] = off[4] - 8
    elif how == "offset_past_end":
        off[-2] = T.n_values + 4096
    elif how == "extra_bits":
        bm[64 * 3: 64 * 3 + 64] = -1          # every bit of GroupTile 3 set: 4096 > its values
    return dataclasses.replace(T, gtile_offset=off, bitmap=bm, max_gt_values=mx)


@pytest.mark.parametrize("kernel", ["dw", "tc"])
@pytest.mark.parametrize("how", ["max_gt_understated", "offset_decreasing", "offset_past_end", "extra_bits"])
def test_corrupt_input_is_reported_not_faulting(how, kernel):
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    N = 16
    use_kernel(kernel, N)
    W = synth.weight(M, K, 0.5, seed=41, mode="int")
    X = synth.activation(K, N, seed=42, mode="int")
    T = sp.encode(to_dev(W))
    Xd = to_dev(X)
    ws = sp.workspace(M, K, N)
    assert sp.check(ws) == 0
    Tb = _corrupt(T, how)
    sp.spmm(Tb, Xd, ws=ws)
    torch.cuda.synchronize()              # no fault, no hang
    flags = sp.check(ws)
    assert flags != 0, f"{how}: corrupt input not reported"
    # the workspace is clean again: the next valid call is exact and reports nothing
    Y = f16_bits(sp.spmm(T, Xd, ws=ws))
    torch.cuda.synchronize()
    assert sp.check(ws) == 0
    exp = oracle.spmm_f64(oracle.encode(W), X).astype(np.float16).view(np.uint16)
    assert np.array_equal(Y, exp)
