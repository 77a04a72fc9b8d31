"""Tensor-parallel (row-partitioned) SpMM driver over torch.distributed.

PAPER.md runs SpInfer inside FasterTransformer with tensor parallelism on 1/2/4
GPUs and attributes the shrinking multi-GPU gains to "rising
communication overhead associated with model parallelism". Here
the split is by output rows: rank r owns rows
spinfer_tp_rows(M, world, r) of every weight, encodes only that shard, and
computes Y[rows] = W[rows] X with spinfer_spmm_tp — no reduction is needed.
  * config 4 (independent layers): no collective at all.
  * config 5 (stacked layers): the next layer needs the full Y, so each layer
    ends with one all-gather of the row chunks of Y (NCCL over NVLink/NVSwitch
    on GPUs; gloo in the CPU tests). Y is [M][N] row-major, so a rank's rows are
    one contiguous chunk and the gather is a plain concatenation whose result
    is directly the next layer's X [M][N] = [K'][N].

Only argument plumbing lives here; the SpMM runs in libspinfer's kernels. The
`spmm_fn` hook exists so the host-side dataflow can be tested with gloo on CPU
(tests/test_tp_cpu.py injects a dense stand-in there); the default is the CUDA path.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Callable, List, Optional, Sequence

import torch
import torch.distributed as dist

GT = 64


def tp_rows(M: int, world: int, rank: int):
    """Rows [b, b + c) of rank `rank` (spinfer_tp_rows: host logic, no device needed)."""
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    if M <= 0 or world <= 0 or not (0 <= rank < world):
        raise ValueError("bad tp_rows arguments")
    return sp.tp_rows(M, world, rank)


@dataclass
class Layer:
    """One row-sharded weight: W_full is M x K; this rank holds rows [row_begin, row_begin+row_count)."""
    name: str
    M: int
    K: int
    row_begin: int
    row_count: int
    shard: object = None          # TCA (GPU) or any object spmm_fn understands
    x_rows: Optional[int] = None  # consume only the first x_rows rows of the previous output (stand-in attention)
    act: Optional[str] = None     # fused epilogue activation ("relu" for the OPT FC1 layers), spinfer_spmm_ex
    bias: object = None           # this rank's bias rows (fp16 [row_count]) or None
    ws: object = None             # preallocated SpMM workspace (None: the binding's per-stream cache)


_scratch: dict = {}


def _buffer(key, shape, like: torch.Tensor) -> torch.Tensor:
    """A scratch tensor reused across calls (no allocation in the per-layer hot loop; allocated
    on first use, so warm up once before capturing a CUDA graph)."""
    k = (key, tuple(shape), like.dtype, like.device)
    t = _scratch.get(k)
    if t is None:
        t = _scratch[k] = torch.empty(shape, dtype=like.dtype, device=like.device)
    return t


def gather_rows(Y_full: torch.Tensor, M: int, world: int, rank: int, group=None) -> torch.Tensor:
    """All-gather the row chunks of Y_full [M][N] in place (each rank has written its rows)."""
    if world == 1:
        return Y_full
    spans = [tp_rows(M, world, r) for r in range(world)]
    sizes = {c for _, c in spans}
    b, c = spans[rank]
    mine = Y_full[b:b + c]
    if len(sizes) == 1:
        # equal chunks: one all_gather_into_tensor straight into Y_full; the rank's chunk goes
        # through a reused send buffer (the input must not alias the output)
        send = _buffer("send", mine.shape, Y_full)
        send.copy_(mine)
        dist.all_gather_into_tensor(Y_full, send, group=group)
    else:
        # uneven chunks (M/64 not divisible by world): pad every chunk to the largest one and
        # gather into one buffer (all_gather with unequal sizes is not portable across backends)
        cmax = max(sizes)
        send = _buffer("send_pad", (cmax,) + tuple(Y_full.shape[1:]), Y_full)
        send[:c] = mine
        recv = _buffer("recv_pad", (world * cmax,) + tuple(Y_full.shape[1:]), Y_full)
        dist.all_gather_into_tensor(recv, send, group=group)
        for r, (bb, cc) in enumerate(spans):
            if r != rank:
                Y_full[bb:bb + cc] = recv[r * cmax: r * cmax + cc]
    return Y_full


def gpu_spmm_fn(layer: Layer, X: torch.Tensor, Y_full: torch.Tensor, world: int, rank: int):
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    if layer.act is None and layer.bias is None:
        sp.spmm_tp(layer.shard, X, Y_full, layer.M, world, rank, ws=layer.ws)
    else:
        # the rank's rows of Y_full are one contiguous [row_count][N] block: the fused-epilogue
        # SpMM writes straight into it (what spinfer_spmm_tp does for the plain SpMM)
        b, c = tp_rows(layer.M, world, rank)
        sp.spmm(layer.shard, X, Y_full[b:b + c], ws=layer.ws, bias=layer.bias, act=layer.act)


def run_stack(layers: Sequence[Layer], X: torch.Tensor, world: int, rank: int, group=None,
              spmm_fn: Callable = gpu_spmm_fn, outputs: Optional[List[torch.Tensor]] = None,
              gather: bool = True) -> torch.Tensor:
    """Config 5 dataflow: for each layer, Y_full[rows] = W[rows] X, all-gather Y_full,
    next X = Y_full (or its first x_rows rows). Returns the last gathered output."""
    cur = X
    for li, L in enumerate(layers):
        if L.x_rows is not None:
            cur = cur[:L.x_rows]
        if cur.shape[0] != L.K:
            raise ValueError(f"layer {L.name}: X has {cur.shape[0]} rows, W has K={L.K}")
        Y = outputs[li] if outputs is not None else torch.empty((L.M, X.shape[1]), dtype=X.dtype, device=X.device)
        spmm_fn(L, cur, Y, world, rank)
        if gather:
            gather_rows(Y, L.M, world, rank, group)
        cur = Y
    return cur


def run_stack_fused(layers: Sequence[Layer], X: torch.Tensor, world: int, rank: int, outputs: Sequence[torch.Tensor],
                    y_peers: Sequence[Sequence[int]], flag_peers: Sequence[int], flag, state, ws=None,
                    timeout_us: int = 0) -> torch.Tensor:
    """Config 5 with the fused all-gather epilogue (spinfer_spmm_tp_gather): each
    layer's kernel stores this rank's rows into every rank's output buffer (y_peers[li][r]: rank r's
    outputs[li] as mapped here, e.g. torch symmetric memory), then one stream-ordered wait on this
    rank's counter. No NCCL call; N <= 16, no bias / activation."""
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    cur = X
    for li, L in enumerate(layers):
        if L.x_rows is not None:
            cur = cur[:L.x_rows]
        if cur.shape[0] != L.K:
            raise ValueError(f"layer {L.name}: X has {cur.shape[0]} rows, W has K={L.K}")
        sp.spmm_tp_gather(L.shard, cur, y_peers[li], L.M, world, rank, flag_peers, ws=ws if ws is not None else L.ws)
        sp.gather_wait(flag, state, world, ws=ws if ws is not None else L.ws, timeout_us=timeout_us)
        cur = outputs[li]
    return cur


# OPT linear-layer shapes (external: OPT configs; the paper names the models)
OPT = {
    "opt-13b": (5120, 20480),
    "opt-30b": (7168, 28672),
    "opt-66b": (9216, 36864),
}


def opt_layer_shapes(model: str):
    """[(name, M, K)] for QKV (fused), O, FC1, FC2 — W is M x K."""
    h, f = OPT[model]
    return [("qkv", 3 * h, h), ("o", h, h), ("fc1", f, h), ("fc2", h, f)]


def opt_stack_layers(model: str, world: int, rank: int, relu: bool = False) -> List[Layer]:
    """Config 5 stack: QKV -> O (consumes the Q block = first h rows of QKV's output,
    the stand-in for attention) -> FC1 (-> ReLU, fused, when relu=True) -> FC2."""
    h, _ = OPT[model]
    out = []
    for name, M, K in opt_layer_shapes(model):
        b, c = tp_rows(M, world, rank)
        out.append(Layer(name, M, K, b, c, x_rows=h if name == "o" else None,
                         act="relu" if (relu and name == "fc1") else None))
    return out
