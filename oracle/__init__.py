"""CPU oracle for the TCA-BME SpMM hot path — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package. It never imports the product package
(paper_conf_eurosys_fanydlgww025_b200) and the product never imports it.

Thin ctypes marshalling over oracle/spinfer_oracle.c (plain single-threaded C,
fp64); every function there cites the PAPER.md passage it follows.
Arrays are numpy: fp16 as uint16 bit patterns, bitmaps uint64, offsets int32.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

GT = 64  # GroupTile edge (reading A1)


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "spinfer_oracle.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        import subprocess
        # -O2, no OpenMP, no -ffast-math: single-threaded IEEE fp64.
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", src, "-o", _LIB_PATH])
    return _LIB_PATH


def _P(t):
    return ctypes.POINTER(t)


def _load():
    global _lib
    if _lib is not None:
        return _lib
    build()
    L = ctypes.CDLL(_LIB_PATH)
    i32, i64, u16, u64, dbl = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint16, ctypes.c_uint64, ctypes.c_double
    L.oracle_f16_to_f64.argtypes = [u16]; L.oracle_f16_to_f64.restype = dbl
    L.oracle_f64_to_f16.argtypes = [dbl]; L.oracle_f64_to_f16.restype = u16
    L.oracle_ngt.argtypes = [ctypes.c_int, ctypes.c_int]; L.oracle_ngt.restype = i64
    L.oracle_nbt.argtypes = [ctypes.c_int, ctypes.c_int]; L.oracle_nbt.restype = i64
    L.oracle_storage_bytes.argtypes = [ctypes.c_int, ctypes.c_int, i64]; L.oracle_storage_bytes.restype = i64
    L.oracle_compression_ratio.argtypes = [ctypes.c_int, ctypes.c_int, i64]; L.oracle_compression_ratio.restype = dbl
    L.oracle_encode_count.argtypes = [_P(u16), ctypes.c_int, ctypes.c_int, _P(i64), _P(i64), _P(i32)]
    L.oracle_encode.argtypes = [_P(u16), ctypes.c_int, ctypes.c_int, _P(i32), _P(u64), _P(u16)]
    L.oracle_decode.argtypes = [_P(i32), _P(u64), _P(u16), ctypes.c_int, ctypes.c_int, _P(u16)]
    L.oracle_gemm_f64.argtypes = [_P(u16), _P(u16), ctypes.c_int, ctypes.c_int, ctypes.c_int, _P(dbl)]
    L.oracle_gemm_f64.restype = None
    L.oracle_spmm_tca_f64.argtypes = [_P(i32), _P(u64), _P(u16), _P(u16), ctypes.c_int, ctypes.c_int,
                                      ctypes.c_int, _P(dbl)]
    L.oracle_spmm_tca_rows_f64.argtypes = [_P(i32), _P(u64), _P(u16), _P(u16), ctypes.c_int, ctypes.c_int,
                                           ctypes.c_int, _P(i32), ctypes.c_int, _P(dbl)]
    L.oracle_masked_popcount.argtypes = [u64, ctypes.c_int]; L.oracle_masked_popcount.restype = ctypes.c_int
    L.oracle_smbd_lane.argtypes = [u64, _P(u16), ctypes.c_int, _P(u16), _P(u16)]
    L.oracle_smbd_lane.restype = None
    L.oracle_smbd_tctile.argtypes = [_P(u64), _P(u16), ctypes.c_int, _P(ctypes.c_uint32)]
    L.oracle_smbd_tctile.restype = None
    L.oracle_bias_act_f64.argtypes = [_P(dbl), ctypes.c_int, ctypes.c_int, _P(u16), ctypes.c_int]
    L.oracle_tp_rows.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, _P(ctypes.c_int), _P(ctypes.c_int)]
    _lib = L
    return L


def _ptr(a: np.ndarray, t):
    assert a.flags.c_contiguous
    return a.ctypes.data_as(_P(t))


class OracleError(RuntimeError):
    pass


def _check(rc: int, what: str):
    if rc != 0:
        raise OracleError(f"{what} failed with status {rc}")


@dataclass
class TCA:
    """TCA-BME arrays as produced by the oracle encoder."""
    M: int
    K: int
    gtile_offset: np.ndarray  # int32 [NGT+1]
    bitmap: np.ndarray        # uint64 [NBT]
    values: np.ndarray        # uint16 fp16 bits [n_values]
    nnz: int
    max_gt_values: int

    @property
    def n_values(self) -> int:
        return int(self.values.shape[0])

    def storage_bytes(self) -> int:
        return storage_bytes(self.M, self.K, self.n_values)


def f16_to_f64(h: int) -> float:
    return float(_load().oracle_f16_to_f64(h))


def f64_to_f16(d: float) -> int:
    return int(_load().oracle_f64_to_f16(d))


def ngt(M: int, K: int) -> int:
    return int(_load().oracle_ngt(M, K))


def nbt(M: int, K: int) -> int:
    return int(_load().oracle_nbt(M, K))


def storage_bytes(M: int, K: int, n_values: int) -> int:
    """eq. (9), with the (padded) value count."""
    return int(_load().oracle_storage_bytes(M, K, n_values))


def compression_ratio(M: int, K: int, n_values: int) -> float:
    """eq. (1)."""
    return float(_load().oracle_compression_ratio(M, K, n_values))


def encode_count(W: np.ndarray):
    L = _load()
    M, K = W.shape
    nnz, nv, mx = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int32()
    _check(L.oracle_encode_count(_ptr(W, ctypes.c_uint16), M, K, ctypes.byref(nnz), ctypes.byref(nv),
                                 ctypes.byref(mx)), "oracle_encode_count")
    return int(nnz.value), int(nv.value), int(mx.value)


def encode(W: np.ndarray) -> TCA:
    """C1: dense fp16 W [M][K] -> TCA-BME."""
    W = np.ascontiguousarray(W, dtype=np.uint16)
    M, K = W.shape
    nnz, nv, mx = encode_count(W)
    off = np.empty(ngt(M, K) + 1, dtype=np.int32)
    bm = np.empty(nbt(M, K), dtype=np.uint64)
    vals = np.empty(max(nv, 1), dtype=np.uint16)
    _check(_load().oracle_encode(_ptr(W, ctypes.c_uint16), M, K, _ptr(off, ctypes.c_int32),
                                 _ptr(bm, ctypes.c_uint64), _ptr(vals, ctypes.c_uint16)), "oracle_encode")
    return TCA(M, K, off, bm, vals[:nv].copy(), nnz, mx)


def decode(T: TCA) -> np.ndarray:
    """C2: TCA-BME -> dense fp16 W (unset bits -> +0.0)."""
    out = np.empty((T.M, T.K), dtype=np.uint16)
    vals = T.values if T.values.size else np.zeros(1, dtype=np.uint16)
    _check(_load().oracle_decode(_ptr(T.gtile_offset, ctypes.c_int32), _ptr(T.bitmap, ctypes.c_uint64),
                                 _ptr(vals, ctypes.c_uint16), T.M, T.K, _ptr(out, ctypes.c_uint16)),
           "oracle_decode")
    return out


def gemm_f64(W: np.ndarray, X: np.ndarray) -> np.ndarray:
    """The plain definition Y = W X in fp64."""
    W = np.ascontiguousarray(W, dtype=np.uint16)
    X = np.ascontiguousarray(X, dtype=np.uint16)
    M, K = W.shape
    K2, N = X.shape
    assert K == K2
    Y = np.empty((M, N), dtype=np.float64)
    _load().oracle_gemm_f64(_ptr(W, ctypes.c_uint16), _ptr(X, ctypes.c_uint16), M, K, N,
                            _ptr(Y, ctypes.c_double))
    return Y


def spmm_f64(T: TCA, X: np.ndarray) -> np.ndarray:
    """SpMM walking the TCA-BME arrays, fp64 accumulation."""
    X = np.ascontiguousarray(X, dtype=np.uint16)
    N = X.shape[1]
    Y = np.empty((T.M, N), dtype=np.float64)
    vals = T.values if T.values.size else np.zeros(1, dtype=np.uint16)
    _check(_load().oracle_spmm_tca_f64(_ptr(T.gtile_offset, ctypes.c_int32), _ptr(T.bitmap, ctypes.c_uint64),
                                       _ptr(vals, ctypes.c_uint16), _ptr(X, ctypes.c_uint16), T.M, T.K, N,
                                       _ptr(Y, ctypes.c_double)), "oracle_spmm_tca_f64")
    return Y


def bias_act_f64(Y: np.ndarray, bias=None, act: str | None = None) -> np.ndarray:
    """C7: the fused FC epilogue act(Y + bias) on an fp64 product (returns a new array)."""
    Y = np.array(Y, dtype=np.float64, order="C", copy=True)
    M, N = Y.shape
    b = None if bias is None else np.ascontiguousarray(bias, dtype=np.uint16)
    if b is not None and b.shape != (M,):
        raise ValueError("bias must be fp16 bits [M]")
    a = {None: 0, "none": 0, "relu": 1}[act]
    _check(_load().oracle_bias_act_f64(_ptr(Y, ctypes.c_double), M, N,
                                       _ptr(b, ctypes.c_uint16) if b is not None else None, a), "oracle_bias_act_f64")
    return Y


def spmm_rows_f64(T: TCA, X: np.ndarray, rows) -> np.ndarray:
    """fp64 SpMM for a subset of output rows (sampled parity at full size)."""
    X = np.ascontiguousarray(X, dtype=np.uint16)
    rows = np.ascontiguousarray(np.asarray(rows, dtype=np.int32))
    N = X.shape[1]
    Y = np.empty((rows.shape[0], N), dtype=np.float64)
    vals = T.values if T.values.size else np.zeros(1, dtype=np.uint16)
    _check(_load().oracle_spmm_tca_rows_f64(_ptr(T.gtile_offset, ctypes.c_int32), _ptr(T.bitmap, ctypes.c_uint64),
                                            _ptr(vals, ctypes.c_uint16), _ptr(X, ctypes.c_uint16), T.M, T.K, N,
                                            _ptr(rows, ctypes.c_int32), rows.shape[0], _ptr(Y, ctypes.c_double)),
           "oracle_spmm_tca_rows_f64")
    return Y


def masked_popcount(b: int, lane: int) -> int:
    """Alg. 2."""
    return int(_load().oracle_masked_popcount(b, lane))


def smbd_lane(bitmap: int, bt_values: np.ndarray, lane: int):
    """Two-phase decode of one lane's .f16x2 register."""
    v = np.ascontiguousarray(bt_values, dtype=np.uint16)
    if v.size == 0:
        v = np.zeros(1, dtype=np.uint16)
    a0, a1 = ctypes.c_uint16(), ctypes.c_uint16()
    _load().oracle_smbd_lane(bitmap, _ptr(v, ctypes.c_uint16), lane, ctypes.byref(a0), ctypes.byref(a1))
    return int(a0.value), int(a1.value)


def smbd_tctile(bm4, tt_values: np.ndarray, lane: int):
    """Ra0..Ra3 (.f16x2, low half = a0) of one lane for one TCTile."""
    bm = np.ascontiguousarray(np.asarray(bm4, dtype=np.uint64))
    v = np.ascontiguousarray(tt_values, dtype=np.uint16)
    if v.size == 0:
        v = np.zeros(1, dtype=np.uint16)
    ra = (ctypes.c_uint32 * 4)()
    _load().oracle_smbd_tctile(_ptr(bm, ctypes.c_uint64), _ptr(v, ctypes.c_uint16), lane, ra)
    return [int(x) for x in ra]


def tp_rows(M: int, world: int, rank: int):
    b, c = ctypes.c_int(), ctypes.c_int()
    _check(_load().oracle_tp_rows(M, world, rank, ctypes.byref(b), ctypes.byref(c)), "oracle_tp_rows")
    return int(b.value), int(c.value)


def shard(T: TCA, row_begin: int, row_count: int) -> TCA:
    """Row shard of an encoding as a contiguous slice of all three arrays with
    GTileOffset rebased: GT rows [a, b) are GTs [a*KG, b*KG).
    Ragged shapes are zero-padded to whole GroupTiles (A8): KG = ceil(K / 64) and a
    shard ending at a ragged M owns the partial last GT row, b = ceil((row_begin + row_count) / 64)."""
    if row_begin % GT or (row_count % GT and row_begin + row_count != T.M):
        raise ValueError("shard rows must be whole GT rows (except a ragged tail ending at M)")
    KG = -(-T.K // GT)
    a, b = row_begin // GT, -(-(row_begin + row_count) // GT)
    off = T.gtile_offset[a * KG: b * KG + 1].astype(np.int64)
    base = int(off[0])
    vals = T.values[base: int(off[-1])].copy()
    bm = T.bitmap[a * KG * 64: b * KG * 64].copy()
    offs = (off - base).astype(np.int32)
    mx = int(np.max(np.diff(offs))) if offs.size > 1 else 0
    nnz = int(sum(bin(int(x)).count("1") for x in bm)) if bm.size < 100000 else -1
    return TCA(row_count, T.K, offs, bm, vals, nnz, mx)
