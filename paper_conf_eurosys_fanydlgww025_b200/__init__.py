"""spinfer-b200: TCA-BME SpMM (SpInfer, EuroSys '25) for B200 / sm_100a.

Thin Python binding over the C ABI in include/spinfer.h (libspinfer.so, built
in-tree by build.py). This module only marshals arguments: every step of the
path (encode, decode, SpMM, split-K fix-up) runs in the library's CUDA kernels.
PyTorch supplies device memory, streams and (in tp.py) process groups. There is
no CPU fallback: if the library or a CUDA device is missing, calls raise.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import torch

__all__ = ["TCA", "SpinferError", "encode", "decode", "spmm", "spmm_tp", "spmm_tp_gather", "gather_wait", "tp_rows",
           "workspace",
           "workspace_bytes", "storage_bytes", "algorithmic_bytes", "check", "set_option", "get_option",
           "lib", "LIB_PATH"]

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SPINFER_LIB") or os.path.join(_PKG, "libspinfer.so")   # SPINFER_LIB: experiments only
GT = 64

_STATUS = {0: "SPINFER_OK", -1: "SPINFER_EINVAL", -2: "SPINFER_ENOSPC", -3: "SPINFER_EOVERFLOW",
           -4: "SPINFER_ECUDA", -5: "SPINFER_ENODEV"}


class SpinferError(RuntimeError):
    def __init__(self, status: int, what: str):
        self.status = status
        super().__init__(f"{what}: {_STATUS.get(status, status)} ({status})")


class _Tca(ctypes.Structure):
    _fields_ = [("M", ctypes.c_int32), ("K", ctypes.c_int32), ("gt_h", ctypes.c_int32), ("gt_w", ctypes.c_int32),
                ("nnz", ctypes.c_int64), ("n_values", ctypes.c_int64), ("max_gt_values", ctypes.c_int32),
                ("reserved", ctypes.c_int32), ("gtile_offset", ctypes.c_void_p), ("bitmap", ctypes.c_void_p),
                ("values", ctypes.c_void_p)]


_lib = None

# Exported symbols (must match include/spinfer.h; checked by tests/test_abi.py).
SYMBOLS = ["spinfer_encode_count", "spinfer_encode_fill", "spinfer_decode", "spinfer_spmm_workspace_bytes",
           "spinfer_spmm", "spinfer_spmm_ex", "spinfer_tp_rows", "spinfer_tca_shard", "spinfer_spmm_tp",
           "spinfer_spmm_tp_gather", "spinfer_gather_wait", "spinfer_spmm_check",
           "spinfer_set_option", "spinfer_get_option", "spinfer_status_str", "spinfer_version"]

# spinfer.h SPINFER_OPT_* / SPINFER_KERNEL_*
OPTIONS = {"kernel": 0, "max_ctas": 1, "stage_g": 2, "stage_s": 3, "wide_bn": 4, "pdl": 5}
KERNELS = {"auto": 0, "dw": 1, "tc": 2}


def lib() -> ctypes.CDLL:
    """Load libspinfer.so (raises if it was not built: no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'` "
                           "(nvcc, sm_100a). There is no CPU fallback.")
    L = ctypes.CDLL(LIB_PATH)
    vp, i32, i64, sz = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_size_t
    P = ctypes.POINTER
    L.spinfer_encode_count.argtypes = [vp, i32, i32, vp, P(ctypes.c_int64), P(ctypes.c_int64), P(ctypes.c_int32), vp]
    L.spinfer_encode_fill.argtypes = [vp, P(_Tca), vp]
    L.spinfer_decode.argtypes = [P(_Tca), vp, vp]
    L.spinfer_spmm_workspace_bytes.argtypes = [i32, i32, i32]
    L.spinfer_spmm_workspace_bytes.restype = sz
    L.spinfer_spmm.argtypes = [P(_Tca), vp, vp, i32, i32, i32, vp, sz, vp]
    L.spinfer_spmm_ex.argtypes = [P(_Tca), vp, vp, i32, i32, i32, vp, i32, vp, sz, vp]
    L.spinfer_tp_rows.argtypes = [i32, i32, i32, P(ctypes.c_int), P(ctypes.c_int)]
    L.spinfer_spmm_tp.argtypes = [P(_Tca), vp, vp, i32, i32, i32, i32, i32, vp, sz, vp]
    L.spinfer_spmm_check.argtypes = [vp, P(ctypes.c_int32), vp]
    L.spinfer_tca_shard.argtypes = [P(_Tca), i32, i32, vp, P(_Tca), vp]
    L.spinfer_spmm_tp_gather.argtypes = [P(_Tca), vp, P(vp), i32, i32, i32, i32, i32, P(vp), vp, sz, vp]
    L.spinfer_gather_wait.argtypes = [vp, vp, i32, vp, ctypes.c_uint32, vp]
    L.spinfer_set_option.argtypes = [i32, i32]
    L.spinfer_get_option.argtypes = [i32]
    L.spinfer_status_str.argtypes = [i32]
    L.spinfer_status_str.restype = ctypes.c_char_p
    L.spinfer_version.restype = ctypes.c_char_p
    for f in ("spinfer_encode_count", "spinfer_encode_fill", "spinfer_decode", "spinfer_spmm", "spinfer_spmm_ex",
              "spinfer_tp_rows", "spinfer_tca_shard", "spinfer_spmm_tp", "spinfer_spmm_tp_gather", "spinfer_gather_wait",
              "spinfer_spmm_check", "spinfer_set_option", "spinfer_get_option"):
        getattr(L, f).restype = ctypes.c_int
    _lib = L
    return L


def _check(rc: int, what: str):
    if rc != 0:
        raise SpinferError(rc, what)


_raw_stream = getattr(torch._C, "_cuda_getCurrentRawStream", None)
_cur_dev = getattr(torch._C, "_cuda_getDevice", None) or torch.cuda.current_device


def _stream(stream=None) -> int:
    if stream is None and _raw_stream is not None:
        return int(_raw_stream(_cur_dev()))   # the current stream's handle without a Stream object
    s = stream if stream is not None else torch.cuda.current_stream()
    return int(s.cuda_stream)


class _NoCtx:
    def __enter__(self):
        return self

    def __exit__(self, *a):
        return False


_NOCTX = _NoCtx()
_U16 = (torch.float16, torch.int16, torch.uint16)


def _on(dev: torch.device):
    """torch.cuda.device(dev) only when it is not already current (the context switch costs
    microseconds per call)."""
    return _NOCTX if dev.index == _cur_dev() else torch.cuda.device(dev)


def _dev_u16(t: torch.Tensor, name: str) -> torch.Tensor:
    if not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor")
    if t.dtype == torch.float16:
        t = t.view(torch.int16)
    if t.dtype not in (torch.int16, torch.uint16):
        raise ValueError(f"{name} must be float16 (got {t.dtype})")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    return t


@dataclass
class TCA:
    """A TCA-BME matrix: three device tensors + sizes."""
    M: int
    K: int
    gtile_offset: torch.Tensor   # int32 [NGT+1]
    bitmap: torch.Tensor         # int64 (uint64 bits) [NBT]
    values: torch.Tensor         # float16 [max(n_values, 8)]
    n_values: int
    nnz: int
    max_gt_values: int

    def c_struct(self) -> _Tca:
        key = (self.M, self.K, self.nnz, self.n_values, self.max_gt_values, id(self.gtile_offset), id(self.bitmap),
               id(self.values))
        c = self.__dict__.get("_cs")
        if c is None or c[0] != key:   # built once per matrix (the host cost of a call matters at TP sizes)
            c = (key, _Tca(self.M, self.K, GT, GT, self.nnz, self.n_values, self.max_gt_values, 0,
                           self.gtile_offset.data_ptr(), self.bitmap.data_ptr(), self.values.data_ptr()))
            self.__dict__["_cs"] = c
        return c[1]

    def storage_bytes(self) -> int:
        return storage_bytes(self.M, self.K, self.n_values)

    def shard(self, row_begin: int, row_count: int, stream=None) -> "TCA":
        """Zero-copy row shard (spinfer_tca_shard): bitmap and values are views into this
        matrix's tensors, GTileOffset a new rebased tensor. One host synchronization."""
        KG = -(-self.K // GT)
        off = torch.empty((-(-row_count // GT)) * KG + 1, dtype=torch.int32, device=self.bitmap.device)
        cs, out = self.c_struct(), _Tca()
        with torch.cuda.device(off.device):
            _check(lib().spinfer_tca_shard(ctypes.byref(cs), row_begin, row_count, off.data_ptr(), ctypes.byref(out),
                                           _stream(stream)), "spinfer_tca_shard")
        esz = self.bitmap.element_size()
        bm0 = (out.bitmap - self.bitmap.data_ptr()) // esz
        v0 = (out.values - self.values.data_ptr()) // self.values.element_size()
        nv = int(out.n_values)
        return TCA(row_count, self.K, off, self.bitmap[bm0: bm0 + 64 * (off.numel() - 1)],
                   self.values[v0: v0 + max(nv, 8)], nv, -1, self.max_gt_values)


def storage_bytes(M: int, K: int, n_values: int) -> int:
    """Buffer bytes of a TCA-BME matrix: eq. (9) with the padded value count."""
    ngt = (-(-M // GT)) * (-(-K // GT))   # zero-padded to whole GroupTiles (reading A8)
    return 4 * (ngt + 1) + 8 * 64 * ngt + 2 * n_values


def algorithmic_bytes(T: TCA, N: int) -> int:
    """Bytes the SpMM must move: the whole TCA-BME matrix,
    X [K][N] and Y [M][N] in fp16."""
    return T.storage_bytes() + 2 * T.K * N + 2 * T.M * N


def encode(W: torch.Tensor, stream=None) -> TCA:
    """Dense fp16 W [M][K] (CUDA) -> TCA-BME on the same device (GPU encoder, bit-exact
    with the oracle). One host synchronization (the value count readback)."""
    W = _dev_u16(W, "W")
    if W.dim() != 2:
        raise ValueError("W must be 2-D")
    M, K = W.shape
    L = lib()
    st = _stream(stream)
    with torch.cuda.device(W.device):
        off = torch.empty((-(-M // GT)) * (-(-K // GT)) + 1, dtype=torch.int32,
                          device=W.device)
        nv, nz, mx = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int32()
        _check(L.spinfer_encode_count(W.data_ptr(), M, K, off.data_ptr(), ctypes.byref(nv), ctypes.byref(nz),
                                      ctypes.byref(mx), st), "spinfer_encode_count")
        bm = torch.empty(64 * (off.numel() - 1), dtype=torch.int64, device=W.device)   # NBT = 64 NGT
        vals = torch.empty(max(nv.value, 8), dtype=torch.float16, device=W.device)
        T = TCA(M, K, off, bm, vals, int(nv.value), int(nz.value), int(mx.value))
        cs = T.c_struct()
        _check(L.spinfer_encode_fill(W.data_ptr(), ctypes.byref(cs), st), "spinfer_encode_fill")
    return T


def decode(T: TCA, stream=None) -> torch.Tensor:
    """TCA-BME -> dense fp16 [M][K] (unset bits -> +0.0)."""
    out = torch.empty((T.M, T.K), dtype=torch.float16, device=T.bitmap.device)
    cs = T.c_struct()
    with torch.cuda.device(out.device):
        _check(lib().spinfer_decode(ctypes.byref(cs), out.data_ptr(), _stream(stream)), "spinfer_decode")
    return out


def workspace_bytes(M: int, K: int, N: int) -> int:
    with torch.cuda.device(torch.cuda.current_device()):
        return int(lib().spinfer_spmm_workspace_bytes(M, K, N))


_ws_cache: dict = {}


_ws_need: dict = {}


def workspace(M: int, K: int, N: int, device=None, stream=None) -> torch.Tensor:
    """A zero-filled workspace for spinfer_spmm, cached per (device, stream): calls on one stream
    are ordered, so they may share one; two streams never do (spinfer.h)."""
    dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
    with _on(dev):
        opts = tuple(int(lib().spinfer_get_option(i)) for i in (OPTIONS["max_ctas"],))
        nk = (dev, M, K, N, opts)
        need = _ws_need.get(nk)
        if need is None:
            need = _ws_need[nk] = max(int(lib().spinfer_spmm_workspace_bytes(M, K, N)), 256)
        key = (dev, _stream(stream))
    ws = _ws_cache.get(key)
    if ws is None or ws.numel() < need:
        ws = torch.zeros(need, dtype=torch.uint8, device=dev)
        _ws_cache[key] = ws
    return ws


def check(ws: torch.Tensor, stream=None) -> int:
    """The workspace's corrupt-input flags since the last check (spinfer_spmm_check; 0 = none:
    1 = gtile_offset out of range, 2 = bitmaps inconsistent with gtile_offset), then resets them."""
    flags = ctypes.c_int32()
    with torch.cuda.device(ws.device):
        _check(lib().spinfer_spmm_check(ws.data_ptr(), ctypes.byref(flags), _stream(stream)), "spinfer_spmm_check")
    return int(flags.value)


def set_option(name: str, value) -> None:
    """Process-wide library option (spinfer.h spinfer_set_option): "kernel" ("auto" | "dw" | "tc"),
    "max_ctas", "stage_g", "stage_s" (0 = default)."""
    v = KERNELS[value] if name == "kernel" and isinstance(value, str) else int(value)
    _check(lib().spinfer_set_option(OPTIONS[name], v), f"spinfer_set_option({name})")


def get_option(name: str) -> int:
    return int(lib().spinfer_get_option(OPTIONS[name]))


def _same_device(X: torch.Tensor, name: str, t: torch.Tensor):
    if t.device != X.device:
        raise ValueError(f"{name} is on {t.device}, X on {X.device}")


ACT_NONE, ACT_RELU = 0, 1   # spinfer.h SPINFER_ACT_*
_ACTS = {None: ACT_NONE, "none": ACT_NONE, "relu": ACT_RELU}


def spmm(T: TCA, X: torch.Tensor, Y: torch.Tensor | None = None, ws: torch.Tensor | None = None,
         stream=None, bias: torch.Tensor | None = None, act: str | None = None) -> torch.Tensor:
    """Y = act(W X + bias): X fp16 [K][N] (CUDA), 1 <= N <= 32; bias fp16 [M] or
    None; act None or "relu" (fused into the SpMM epilogue, spinfer_spmm_ex); returns fp16 [M][N]."""
    if not (X.is_cuda and X.dtype in _U16 and X.dim() == 2 and X.is_contiguous()):
        X = _dev_u16(X, "X")
        if X.dim() != 2:
            raise ValueError("X must be 2-D [K][N]")
    K, N = X.shape
    if K != T.K:
        raise ValueError(f"X has K={K}, W has K={T.K}")
    dev = X.device
    if T.bitmap.device != dev:
        _same_device(X, "W", T.bitmap)
    if Y is None:
        Y = torch.empty((T.M, N), dtype=torch.float16, device=dev)
    Yv = Y if (Y.is_cuda and Y.dtype in _U16 and Y.is_contiguous()) else _dev_u16(Y, "Y")
    if Yv.shape != (T.M, N):
        raise ValueError(f"Y has shape {tuple(Yv.shape)}, expected {(T.M, N)}")
    if Yv.device != dev:
        _same_device(X, "Y", Yv)
    if ws is None:
        ws = workspace(T.M, T.K, N, dev, stream)
    if ws.device != dev:
        _same_device(X, "workspace", ws)
    actc = _ACTS[act]
    bptr = None
    if bias is not None:
        bv = _dev_u16(bias, "bias")
        _same_device(X, "bias", bv)
        if bv.numel() != T.M:
            raise ValueError(f"bias has {bv.numel()} entries, W has M={T.M}")
        bptr = bv.data_ptr()
    cs = T.c_struct()
    with _on(dev):
        if bptr is None and actc == ACT_NONE:
            _check(lib().spinfer_spmm(ctypes.byref(cs), X.data_ptr(), Yv.data_ptr(), T.M, T.K, N, ws.data_ptr(),
                                      ws.numel(), _stream(stream)), "spinfer_spmm")
        else:
            _check(lib().spinfer_spmm_ex(ctypes.byref(cs), X.data_ptr(), Yv.data_ptr(), T.M, T.K, N, bptr, actc,
                                         ws.data_ptr(), ws.numel(), _stream(stream)), "spinfer_spmm_ex")
    return Y


def tp_rows(M: int, world: int, rank: int):
    b, c = ctypes.c_int(), ctypes.c_int()
    _check(lib().spinfer_tp_rows(M, world, rank, ctypes.byref(b), ctypes.byref(c)), "spinfer_tp_rows")
    return int(b.value), int(c.value)


def spmm_tp(T_shard: TCA, X: torch.Tensor, Y_full: torch.Tensor, M_full: int, world: int, rank: int,
            ws: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """Row-partitioned SpMM: writes rows tp_rows(M_full, world, rank) of Y_full [M_full][N]. No communication."""
    X = _dev_u16(X, "X")
    if X.dim() != 2:
        raise ValueError("X must be 2-D [K][N]")
    K, N = X.shape
    Yv = _dev_u16(Y_full, "Y_full")
    if tuple(Yv.shape) != (M_full, N):
        raise ValueError(f"Y_full has shape {tuple(Yv.shape)}, expected {(M_full, N)}")
    _same_device(X, "Y_full", Yv)
    _same_device(X, "W shard", T_shard.bitmap)
    if ws is None:
        ws = workspace(max(T_shard.M, GT), K, N, X.device, stream)
    _same_device(X, "workspace", ws)
    cs = T_shard.c_struct()
    with torch.cuda.device(X.device):
        _check(lib().spinfer_spmm_tp(ctypes.byref(cs), X.data_ptr(), Yv.data_ptr(), M_full, K, N, world, rank,
                                     ws.data_ptr(), ws.numel(), _stream(stream)), "spinfer_spmm_tp")
    return Y_full


def _ptr(x) -> int:
    return x.data_ptr() if isinstance(x, torch.Tensor) else int(x)


def spmm_tp_gather(T_shard: TCA, X: torch.Tensor, Y_peers, M_full: int, world: int, rank: int, flag_peers,
                   ws: torch.Tensor | None = None, stream=None):
    """Fused all-gather epilogue (spinfer_spmm_tp_gather): this rank's rows of W X are stored into every
    rank's Y_full (Y_peers[r]: tensor or device address of rank r's [M_full][N] buffer as mapped here),
    then every rank's counter (flag_peers[r]) is signalled. N <= 16."""
    X = _dev_u16(X, "X")
    if X.dim() != 2:
        raise ValueError("X must be 2-D [K][N]")
    K, N = X.shape
    if len(Y_peers) != world or len(flag_peers) != world:
        raise ValueError("one Y buffer and one counter per rank")
    if ws is None:
        ws = workspace(max(T_shard.M, GT), K, N, X.device, stream)
    yp = (ctypes.c_void_p * world)(*[_ptr(y) for y in Y_peers])
    fp = (ctypes.c_void_p * world)(*[_ptr(f) for f in flag_peers])
    cs = T_shard.c_struct()
    with torch.cuda.device(X.device):
        _check(lib().spinfer_spmm_tp_gather(ctypes.byref(cs), X.data_ptr(), yp, M_full, K, N, world, rank, fp,
                                            ws.data_ptr(), ws.numel(), _stream(stream)), "spinfer_spmm_tp_gather")


def gather_wait(flag, state, world: int, ws: torch.Tensor | None = None, timeout_us: int = 0, stream=None):
    """Stream-ordered wait until every rank signalled this rank's counter (spinfer_gather_wait)."""
    dev = flag.device if isinstance(flag, torch.Tensor) else torch.device("cuda", torch.cuda.current_device())
    with torch.cuda.device(dev):
        _check(lib().spinfer_gather_wait(_ptr(flag), _ptr(state), world, ws.data_ptr() if ws is not None else None,
                                         int(timeout_us), _stream(stream)), "spinfer_gather_wait")
