"""Pins of the CPU oracle against what the paper and the mathematics fix (-m "not gpu").

Each pin is chosen so that a plausible mistake in the oracle (wrong TCTile /
BitmapTile order, wrong bit order, missing padding, transposed operand, dropped
term) fails at least one of them. None of them re-types the oracle's own loops:
they use hand-derived fixtures (tests/golden), closed forms from the paper's
equations, the PTX ISA m16n8k16 fragment table, numpy library routines and
brute force on tiny inputs.
"""
import json
import os

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def canon(W):
    """-0.0 is not a non-zero (reading A7): decode yields +0.0."""
    W = W.copy()
    W[(W & 0x7FFF) == 0] = 0
    return W


def closed_form_bt(r, c, K):
    """Global BitmapTile index and bit of element (r, c) — SURVEY §8(c) closed form,
    derived from P:192 (BTs column-major in a TT), P:194 (TTs column-major in a GT,
    GTs row-major) and P:287 (bit b <-> (b/8, b%8))."""
    g = (r // 64) * (-(-K // 64)) + c // 64     # K/64 rounded up: ragged shapes are zero-padded (A8)
    tt = ((c % 64) // 16) * 4 + (r % 64) // 16
    bt = ((c % 16) // 8) * 2 + (r % 16) // 8
    return (g * 16 + tt) * 4 + bt, (r % 8) * 8 + c % 8


# ---------------------------------------------------------------- fp16 helpers

def test_f16_to_f64_matches_numpy_all_patterns():
    bits = np.arange(65536, dtype=np.uint16)
    ref = bits.view(np.float16).astype(np.float64)
    got = np.array([oracle.f16_to_f64(int(b)) for b in bits])
    fin = np.isfinite(ref)
    assert np.array_equal(got[fin], ref[fin])
    assert np.all(np.isnan(got[np.isnan(ref)]))
    assert np.array_equal(got[np.isinf(ref)], ref[np.isinf(ref)])


def test_f64_to_f16_rne_matches_numpy():
    rng = np.random.default_rng(1)
    xs = np.concatenate([rng.uniform(-3000, 3000, 200), rng.uniform(-1e-4, 1e-4, 100),
                         np.array([0.5, 1.5, 2.5, 2049.0, 2051.0, -2049.0, 65504.0, 1e-8])])
    for x in xs:
        assert oracle.f64_to_f16(float(x)) == int(np.float16(x).view(np.uint16)), x


# ---------------------------------------------------------------- worked example

def test_worked_example_64x64():
    g = json.load(open(os.path.join(GOLD, "worked_64x64.json")))
    W = np.zeros((64, 64), dtype=np.uint16)
    for r, c, v in g["nonzeros"]:
        W[r, c] = int(v, 16)
    T = oracle.encode(W)
    assert T.gtile_offset.tolist() == g["gtile_offset"]
    exp_bm = np.zeros(64, dtype=np.uint64)
    for k, v in g["bitmap_nonzero"].items():
        exp_bm[int(k)] = np.uint64(int(v, 16))
    assert np.array_equal(T.bitmap, exp_bm)
    assert [hex(int(v)) for v in T.values] == [hex(int(v, 16)) for v in g["values"]]
    for case in g["smbd"]:
        tt = case["tctile"]
        bm4 = T.bitmap[tt * 4: tt * 4 + 4]
        base = int(sum(bin(int(b)).count("1") for b in T.bitmap[: tt * 4]))
        ra = oracle.smbd_tctile(bm4, T.values[base:], case["lane"])
        assert ra == [int(x, 16) for x in case["ra"]], case["why"]


# ---------------------------------------------------------------- P-E1 brute force

@pytest.mark.parametrize("M,K", [(64, 64), (64, 128), (128, 64)])
def test_single_nonzero_brute_force(M, K):
    """Every position (r, c) alone: exactly one bitmap bit, at the closed-form index."""
    for r in range(M):
        for c in range(K):
            W = np.zeros((M, K), dtype=np.uint16)
            W[r, c] = 0x3C00 + (r * 7 + c) % 512
            T = oracle.encode(W)
            nz = np.flatnonzero(T.bitmap)
            bt, bit = closed_form_bt(r, c, K)
            assert nz.tolist() == [bt], (r, c)
            assert int(T.bitmap[bt]) == 1 << bit, (r, c)
            g = bt // 64
            assert int(T.values[T.gtile_offset[g]]) == int(W[r, c])
            assert T.n_values == 8 and T.nnz == 1


def test_row_byte_patterns_exhaustive():
    """All 256 byte patterns in one BT row land in bits 8*row .. 8*row+7."""
    for row in (0, 3, 7):
        for pat in range(256):
            W = np.zeros((64, 64), dtype=np.uint16)
            for c in range(8):
                if pat >> c & 1:
                    W[row, c] = 0x3C00 + c
            T = oracle.encode(W)
            assert int(T.bitmap[0]) == pat << (8 * row)
            exp = [0x3C00 + c for c in range(8) if pat >> c & 1]
            assert T.values[: len(exp)].tolist() == exp


# ---------------------------------------------------------------- P-E4 PTX fragment layout

def ptx_m16n8k16_a_fragment(lane, j):
    """PTX ISA, mma.m16n8k16 .f16 A fragment (row-major A 16x16): a_j of lane:
    groupID = lane >> 2, threadID_in_group = lane % 4;
    row = groupID (+8 for a2,a3,a6,a7), col = 2*tig + (j & 1) (+8 for a4..a7)."""
    g, t = lane >> 2, lane % 4
    row = g + (8 if j in (2, 3, 6, 7) else 0)
    col = 2 * t + (j & 1) + (8 if j >= 4 else 0)
    return row, col


def test_smbd_matches_ptx_fragment_layout():
    """The SMBD emulator (Alg. 2 + two-phase decode) fed with the
    oracle's encoding puts every element where the ISA's A fragment expects it."""
    rng = np.random.default_rng(7)
    for trial in range(300):
        s = rng.choice([0.0, 0.3, 0.5, 0.7, 0.95, 1.0])
        W = synth.weight(64, 64, s, seed=1000 + trial)
        T = oracle.encode(W)
        cum = np.concatenate([[0], np.cumsum([bin(int(b)).count("1") for b in T.bitmap])])
        tt = int(rng.integers(16))
        tr, tc = tt % 4, tt // 4
        tile = canon(W)[tr * 16: tr * 16 + 16, tc * 16: tc * 16 + 16]
        base = int(cum[tt * 4])
        for lane in range(32):
            ra = oracle.smbd_tctile(T.bitmap[tt * 4: tt * 4 + 4], T.values[base:], lane)
            halves = []
            for r in ra:
                halves += [r & 0xFFFF, r >> 16]
            for j in range(8):
                row, col = ptx_m16n8k16_a_fragment(lane, j)
                assert halves[j] == int(tile[row, col]), (trial, tt, lane, j)


def test_masked_popcount_alg2():
    rng = np.random.default_rng(3)
    for _ in range(200):
        b = int(rng.integers(0, 2**63)) * 2 + int(rng.integers(0, 2))
        for lane in range(32):
            assert oracle.masked_popcount(b, lane) == sum((b >> i) & 1 for i in range(2 * lane))


# ---------------------------------------------------------------- P-E2 / P-E3

def _roundtrip_and_counts(W):
    T = oracle.encode(W)
    M, K = W.shape
    Wc = canon(W)
    assert np.array_equal(oracle.decode(T), Wc)
    nz = (Wc & 0x7FFF) != 0
    assert T.nnz == int(nz.sum())
    assert sum(bin(int(b)).count("1") for b in T.bitmap) == T.nnz
    # per-GT counts from the dense matrix directly (GT = 64x64 block, row-major)
    blocks = nz.reshape(M // 64, 64, K // 64, 64).sum(axis=(1, 3)).reshape(-1)
    padded = (blocks + 7) // 8 * 8
    assert np.array_equal(np.diff(T.gtile_offset.astype(np.int64)), padded)
    assert T.gtile_offset[0] == 0 and T.gtile_offset[-1] == T.n_values
    assert T.max_gt_values == int(padded.max())
    # padding is +0.0
    for g in range(len(blocks)):
        a = int(T.gtile_offset[g]) + int(blocks[g])
        assert np.all(T.values[a: int(T.gtile_offset[g + 1])] == 0)
    # buffer sizes = eq. (9) with the padded count
    nbytes = T.gtile_offset.nbytes + T.bitmap.nbytes + T.values.nbytes
    assert nbytes == oracle.storage_bytes(M, K, T.n_values)
    assert T.n_values - T.nnz <= 7 * oracle.ngt(M, K)
    return T


@pytest.mark.parametrize("s", [0.0, 0.3, 0.4, 0.5, 0.6, 0.7, 0.95, 1.0])
def test_roundtrip_random(s):
    _roundtrip_and_counts(synth.weight(256, 192, s, seed=11))


def test_roundtrip_structured():
    M, K = 128, 192
    r, c = np.indices((M, K))
    pats = {
        "diag": r == c,
        "rows": (r % 17) == 3,
        "cols": (c % 13) == 5,
        "single_bt": (r // 8 == 5) & (c // 8 == 9),
        "upper": r <= c,
        "dense_gt": (r < 64) & (c < 64),
    }
    for name, m in pats.items():
        W = np.where(m, 0x3C00 + (r * K + c) % 1000, 0).astype(np.uint16)
        _roundtrip_and_counts(W)


def test_negative_zero_dropped_nan_inf_kept():
    W = np.zeros((64, 64), dtype=np.uint16)
    W[0, 0] = 0x8000          # -0.0: not a non-zero (A7)
    W[1, 1] = 0x7C00          # +inf kept
    W[2, 2] = 0x7E00          # NaN kept
    W[3, 3] = 0x0001          # smallest subnormal kept
    T = _roundtrip_and_counts(W)
    assert T.nnz == 3


@settings(max_examples=40, deadline=None)
@given(mg=st.integers(1, 3), kg=st.integers(1, 3), s=st.floats(0.0, 1.0), seed=st.integers(0, 2**31))
def test_roundtrip_hypothesis(mg, kg, s, seed):
    _roundtrip_and_counts(synth.weight(64 * mg, 64 * kg, s, seed=seed))


def test_invalid_shapes():
    with pytest.raises(oracle.OracleError):
        oracle.spmm_f64(oracle.encode(np.ones((64, 64), dtype=np.uint16)), np.zeros((64, 0), dtype=np.uint16))
    with pytest.raises(oracle.OracleError):
        oracle.tp_rows(0, 1, 0)


@pytest.mark.parametrize("M,K", [(1, 1), (65, 64), (64, 96), (70, 100), (130, 9)])
def test_ragged_shapes_single_nonzero_brute_force(M, K):
    """Reading A8: a shape that is not a multiple of 64 is zero-padded to whole GroupTiles. Every
    single-non-zero position lands on the closed-form BT and bit (with K/64 rounded up), the
    padding holds no bit, NGT = ceil(M/64) ceil(K/64), NBT = 64 NGT, and decode returns W."""
    ngt = (-(-M // 64)) * (-(-K // 64))
    for r in range(M):
        for c in range(0, K, max(1, K // 7)):
            W = np.zeros((M, K), dtype=np.uint16)
            W[r, c] = 0x3C00
            T = oracle.encode(W)
            assert T.gtile_offset.shape == (ngt + 1,) and T.bitmap.shape == (64 * ngt,)
            bt, bit = closed_form_bt(r, c, K)
            nz = np.flatnonzero(T.bitmap)
            assert nz.tolist() == [bt] and int(T.bitmap[bt]) == 1 << bit
            assert np.array_equal(oracle.decode(T), W)


def test_ragged_round_trip_and_product():
    rng = np.random.default_rng(9)
    for M, K in [(100, 70), (200, 130), (64, 65), (1, 300)]:
        W = synth.weight(M, K, 0.5, seed=M * 1000 + K)
        X = synth.activation(K, 5, seed=K)
        T = oracle.encode(W)
        assert np.array_equal(oracle.decode(T), canon(W))
        assert int(sum(bin(int(b)).count("1") for b in T.bitmap)) == T.nnz == int(np.count_nonzero(W & 0x7FFF))
        ref = W.view(np.float16).astype(np.float64) @ X.view(np.float16).astype(np.float64)
        assert np.array_equal(oracle.spmm_f64(T, X), ref)
        rows = rng.choice(M, size=min(M, 5), replace=False).astype(np.int32)
        assert np.array_equal(oracle.spmm_rows_f64(T, X, rows), ref[rows])
        assert oracle.storage_bytes(M, K, T.n_values) == 4 * (oracle.ngt(M, K) + 1) + 8 * 64 * oracle.ngt(M, K) + 2 * T.n_values


# ---------------------------------------------------------------- checkerboard / eq. (9)

def test_checkerboard_worked_example():
    g = json.load(open(os.path.join(GOLD, "checkerboard.json")))
    for case in g["cases"]:
        M, K = case["M"], case["K"]
        nnz = M * K // 2
        assert oracle.storage_bytes(M, K, nnz) == case["storage_bytes"]
        assert abs(oracle.compression_ratio(M, K, nnz) - case["cr"]) < 5e-6
        if M * K <= 4096 * 4096:
            r, c = np.indices((M, K))
            W = np.where((r + c) % 2 == 0, 0x3C00, 0).astype(np.uint16)
            T = oracle.encode(W)
            assert np.all(T.bitmap == np.uint64(int(g["bitmap_every_bt"], 16)))
            assert np.all(np.diff(T.gtile_offset) == g["nnz_per_gt"])
            assert T.storage_bytes() == case["storage_bytes"]


def test_cr_above_one_beyond_6_25_percent():
    """Derived from eq. (9): CR > 1 iff 2MK > 4(NGT+1) + MK/8 + 2MK(1-s), i.e. s > ~1/16
    (TCA-BME keeps CR > 1 even at low sparsity)."""
    M = K = 4096
    for s in np.linspace(0.07, 0.99, 20):
        assert oracle.compression_ratio(M, K, int(M * K * (1 - s))) > 1.0
    for s in (0.0, 0.03, 0.06):
        assert oracle.compression_ratio(M, K, int(M * K * (1 - s))) < 1.0


# ---------------------------------------------------------------- SpMM

def test_spmm_matches_dense_definition_and_numpy():
    for (M, K, N, s) in [(64, 64, 8, 0.5), (128, 192, 16, 0.3), (192, 128, 24, 0.7), (64, 256, 32, 0.0)]:
        W = synth.weight(M, K, s, seed=5)
        X = synth.activation(K, N, seed=6)
        T = oracle.encode(W)
        Yt = oracle.spmm_f64(T, X)
        Yd = oracle.gemm_f64(oracle.decode(T), X)
        Wn = W.view(np.float16).astype(np.float64)
        Xn = X.view(np.float16).astype(np.float64)
        Yn = Wn @ Xn
        scale = np.abs(Wn) @ np.abs(Xn) + 1e-300
        assert np.max(np.abs(Yt - Yn) / scale) < 1e-13
        assert np.max(np.abs(Yd - Yn) / scale) < 1e-13
        rows = [0, M // 2, M - 1]
        assert np.max(np.abs(oracle.spmm_rows_f64(T, X, rows) - Yn[rows]) / scale[rows]) < 1e-13


def test_spmm_integer_exact():
    """P-S2: integer inputs give exactly representable integer results."""
    W = synth.weight(128, 256, 0.5, seed=9, mode="int")
    X = synth.activation(256, 16, seed=9, mode="int")
    Y = oracle.spmm_f64(oracle.encode(W), X)
    Wi = W.view(np.float16).astype(np.int64)
    Xi = X.view(np.float16).astype(np.int64)
    assert np.array_equal(Y, (Wi @ Xi).astype(np.float64))


def test_spmm_special_cases():
    X = synth.activation(128, 8, seed=4)
    T1 = oracle.encode(synth.weight(128, 128, 1.0, seed=1))      # s = 1: all zero
    assert T1.n_values == 0 and not np.any(T1.bitmap)
    assert np.all(oracle.spmm_f64(T1, X) == 0)
    I = np.zeros((128, 128), dtype=np.uint16)
    I[np.arange(128), np.arange(128)] = 0x3C00                   # W = I -> Y = X
    Y = oracle.spmm_f64(oracle.encode(I), X)
    assert np.array_equal(Y, X.view(np.float16).astype(np.float64))


# ---------------------------------------------------------------- TP rows / P-E5

@pytest.mark.parametrize("M", [64, 256, 1152, 9216, 28672, 36864])
@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_tp_rows_partition(M, world):
    spans = [oracle.tp_rows(M, world, r) for r in range(world)]
    pos = 0
    for b, c in spans:
        assert b == pos and b % 64 == 0 and c % 64 == 0
        pos += c
    assert pos == M
    sizes = [c for _, c in spans]
    assert max(sizes) - min(sizes) <= 64


def test_shard_is_slice_of_encoding():
    W = synth.weight(448, 192, 0.5, seed=21)
    T = oracle.encode(W)
    for world in (2, 3, 4):
        for r in range(world):
            b, c = oracle.tp_rows(448, world, r)
            S = oracle.shard(T, b, c)
            E = oracle.encode(W[b: b + c])
            assert np.array_equal(S.gtile_offset, E.gtile_offset)
            assert np.array_equal(S.bitmap, E.bitmap)
            assert np.array_equal(S.values, E.values)


@pytest.mark.parametrize("M,K", [(1000, 300), (130, 65), (64, 100), (577, 1)])
def test_shard_is_slice_of_encoding_ragged(M, K):
    """P-E5 on ragged shapes (reading A8): the shard of every rank, including the one holding the
    partial last GT row, equals the encoding of its own rows of W, array for array."""
    W = synth.weight(M, K, 0.5, seed=M + K)
    T = oracle.encode(W)
    for world in (1, 2, 3, 5):
        for r in range(world):
            b, c = oracle.tp_rows(M, world, r)
            if c == 0:
                continue
            S = oracle.shard(T, b, c)
            E = oracle.encode(W[b: b + c])
            assert S.M == E.M == c
            assert np.array_equal(S.gtile_offset, E.gtile_offset), (M, K, world, r)
            assert np.array_equal(S.bitmap, E.bitmap)
            assert np.array_equal(S.values, E.values)
            assert S.n_values == E.n_values and S.nnz == E.nnz


def test_bias_act_worked_example():
    """C7 fused FC epilogue, values worked by hand: act(Y + b) with b = (1.0, -0.5)."""
    Y = np.array([[-1.5, 2.0], [0.25, -0.25]])
    b = np.array([0x3C00, 0xB800], dtype=np.uint16)             # fp16 1.0, -0.5
    assert np.array_equal(oracle.bias_act_f64(Y, b, None), [[-0.5, 3.0], [-0.25, -0.75]])
    assert np.array_equal(oracle.bias_act_f64(Y, b, "relu"), [[0.0, 3.0], [0.0, 0.0]])
    assert np.array_equal(oracle.bias_act_f64(Y, None, "relu"), [[0.0, 2.0], [0.25, 0.0]])
    assert np.array_equal(oracle.bias_act_f64(Y), Y)


def test_bias_act_identity_weight():
    """W = I: the SpMM returns X exactly, so the fused epilogue must give max(X + b, 0) with the
    hand-checkable fp16 inputs below (X row i = (i - 2, 2 - i) halves, b_i = -0.5 i)."""
    M = 64
    W = np.zeros((M, M), dtype=np.uint16)
    W[np.arange(M), np.arange(M)] = 0x3C00
    X = np.array([[oracle.f64_to_f16(i - 2.0), oracle.f64_to_f16(2.0 - i)] for i in range(M)], dtype=np.uint16)
    b = np.array([oracle.f64_to_f16(-0.5 * i) for i in range(M)], dtype=np.uint16)
    Y = oracle.bias_act_f64(oracle.spmm_f64(oracle.encode(W), X), b, "relu")
    i = np.arange(M, dtype=np.float64)
    exp = np.stack([np.maximum(i - 2.0 - 0.5 * i, 0.0), np.maximum(2.0 - i - 0.5 * i, 0.0)], axis=1)
    assert np.array_equal(Y, exp)
