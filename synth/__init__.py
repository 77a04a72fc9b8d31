"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the CPU oracle.

Holds none of the method's arithmetic: it only draws W (fp16, unstructured
keep-mask at sparsity s) and X (fp16, dense). The recipe is documented in
synth.c and DESIGN.md ("Input recipe"). Arrays are numpy uint16 fp16 bit patterns.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libsynth.so")
_lib = None

DEFAULT_SEED = 20250330


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "synth.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        import subprocess
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-pthread",
                               src, "-o", _LIB_PATH, "-lm"])
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        u16p = ctypes.POINTER(ctypes.c_uint16)
        lib.synth_weight.argtypes = [u16p, ctypes.c_int64, ctypes.c_int64, ctypes.c_uint64,
                                     ctypes.c_double, ctypes.c_int, ctypes.c_int]
        lib.synth_weight_rows.argtypes = [u16p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_uint64,
                                          ctypes.c_double, ctypes.c_int, ctypes.c_int]
        lib.synth_activation.argtypes = [u16p, ctypes.c_int64, ctypes.c_int64, ctypes.c_uint64,
                                         ctypes.c_int, ctypes.c_int]
        lib.synth_hash.argtypes = [ctypes.c_uint64] * 3
        lib.synth_hash.restype = ctypes.c_uint64
        lib.synth_splitmix64.argtypes = [ctypes.c_uint64]
        lib.synth_splitmix64.restype = ctypes.c_uint64
        lib.synth_f64_to_f16.argtypes = [ctypes.c_double]
        lib.synth_f64_to_f16.restype = ctypes.c_uint16
        _lib = lib
    return _lib


def _threads() -> int:
    return max(1, min(64, os.cpu_count() or 1))


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint16))


def weight(M: int, K: int, sparsity: float, seed: int = DEFAULT_SEED, mode: str = "uniform",
           out: np.ndarray | None = None, row0: int = 0) -> np.ndarray:
    """Dense fp16 W [M][K] (uint16 bits) with an i.i.d. Bernoulli(1-s) keep-mask. row0 > 0: rows
    [row0, row0 + M) of the matrix drawn with the same seed (a row shard, identical elements)."""
    lib = _load()
    W = out if out is not None else np.empty((M, K), dtype=np.uint16)
    assert W.dtype == np.uint16 and W.shape == (M, K) and W.flags.c_contiguous
    rc = lib.synth_weight_rows(_ptr(W), row0, M, K, seed, float(sparsity), 1 if mode == "int" else 0, _threads())
    if rc != 0:
        raise ValueError("synth_weight failed")
    return W


def activation(K: int, N: int, seed: int = DEFAULT_SEED, mode: str = "uniform") -> np.ndarray:
    """Dense fp16 X [K][N] (uint16 bits)."""
    lib = _load()
    X = np.empty((K, N), dtype=np.uint16)
    rc = lib.synth_activation(_ptr(X), K, N, seed, 1 if mode == "int" else 0, _threads())
    if rc != 0:
        raise ValueError("synth_activation failed")
    return X


def hash64(seed: int, tag: int, idx: int) -> int:
    return int(_load().synth_hash(seed, tag, idx))


def splitmix64(x: int) -> int:
    return int(_load().synth_splitmix64(x))


def f64_to_f16(d: float) -> int:
    return int(_load().synth_f64_to_f16(d))
