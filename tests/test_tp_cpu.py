"""Multi-process (gloo, CPU) tests of the row-partitioned TP dataflow (-m "not gpu").

The SpMM itself needs a GPU; here the per-rank compute is a dense fp64 stand-in
injected through tp.run_stack's spmm_fn hook, so what is tested is the host
logic: row partition, shard ownership, all-gather assembly, stacked-layer
wiring (config 5) and the equal/unequal chunk paths.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth
from paper_conf_eurosys_fanydlgww025_b200 import tp

MINI = [("qkv", 384, 128), ("o", 128, 128), ("fc1", 320, 128), ("fc2", 128, 320)]
H = 128


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _layers(world, rank):
    out = []
    for i, (name, M, K) in enumerate(MINI):
        W = synth.weight(M, K, 0.5, seed=100 + i).view(np.float16).astype(np.float64)
        b, c = tp.tp_rows(M, world, rank)
        L = tp.Layer(name, M, K, b, c, shard=torch.from_numpy(W[b:b + c].copy()),
                     x_rows=H if name == "o" else None)
        out.append(L)
    return out


def _dense_fn(L, X, Y, world, rank):
    Y[L.row_begin:L.row_begin + L.row_count] = L.shard @ X


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    X = torch.from_numpy(synth.activation(MINI[0][2], 16, seed=7).view(np.float16).astype(np.float64))
    out = tp.run_stack(_layers(world, rank), X, world, rank, spmm_fn=_dense_fn)
    q.put((rank, out.numpy().copy()))
    dist.barrier()
    dist.destroy_process_group()


def _run(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(world))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    return res


def _single():
    X = torch.from_numpy(synth.activation(MINI[0][2], 16, seed=7).view(np.float16).astype(np.float64))
    return tp.run_stack(_layers(1, 0), X, 1, 0, spmm_fn=_dense_fn).numpy()


@pytest.mark.parametrize("world", [2, 3])
def test_tp_stack_gloo_matches_single(world):
    ref = _single()
    res = _run(world)
    for r in range(world):
        np.testing.assert_allclose(res[r], ref, rtol=1e-12, atol=1e-12)


def test_opt_shapes_partition_multiple_of_64():
    for model in tp.OPT:
        for world in (1, 2, 4, 8):
            for name, M, K in tp.opt_layer_shapes(model):
                spans = [tp.tp_rows(M, world, r) for r in range(world)]
                assert sum(c for _, c in spans) == M
                assert all(b % 64 == 0 and c % 64 == 0 for b, c in spans)
                assert len({c for _, c in spans}) == 1   # every configured shape splits evenly
