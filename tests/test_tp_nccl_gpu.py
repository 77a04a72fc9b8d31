"""Multi-GPU test of the config-5 dataflow over NCCL: one
process per GPU, each rank encodes and multiplies only its row shard of every layer with the CUDA
kernels (spinfer_spmm_tp) and the outputs are all-gathered with NCCL (tp.gather_rows). Every rank's
gathered output of every layer must match the fp64 oracle applied to that layer's own gathered
input (errors do not compound), within the north_star bound, and all ranks must hold bit-identical
results. Needs >= 2 visible GPUs: skipped on a one-GPU box (the gloo tests in test_tp_cpu.py cover the
host logic there)."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

H, F, N, S = 256, 1024, 16, 0.6
SHAPES = [("qkv", 3 * H, H), ("o", H, H), ("fc1", F, H), ("fc2", H, F)]


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    import synth
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    from paper_conf_eurosys_fanydlgww025_b200 import tp
    from tests.helpers import to_dev
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", rank))
    try:
        layers = []
        for i, (name, M, K) in enumerate(SHAPES):
            W = synth.weight(M, K, S, seed=40 + i)
            b, c = tp.tp_rows(M, world, rank)
            shard = sp.encode(to_dev(np.ascontiguousarray(W[b:b + c]))) if c else None
            layers.append(tp.Layer(name, M, K, b, c, shard=shard, x_rows=H if name == "o" else None))
        X = to_dev(synth.activation(H, N, seed=3)).view(torch.float16)
        outs = [torch.empty((M, N), dtype=torch.float16, device="cuda") for _, M, _ in SHAPES]
        tp.run_stack(layers, X, world, rank, outputs=outs)
        torch.cuda.synchronize()
        q.put((rank, [o.cpu().view(torch.int16).numpy().view(np.uint16).copy() for o in outs], None))
    except Exception as e:   # report, do not hang the other ranks' queue reads
        q.put((rank, None, repr(e)))
    finally:
        dist.destroy_process_group()


def test_config5_stack_nccl_world():
    import torch
    import torch.multiprocessing as mp
    import oracle
    import synth
    from tests.helpers import assert_within, north_star_bound
    ngpu = torch.cuda.device_count()
    if ngpu < 2:
        pytest.skip(f"needs >= 2 GPUs for an NCCL world (this box has {ngpu})")
    world = min(ngpu, 4)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        rank, outs, err = q.get(timeout=600)
        assert err is None, f"rank {rank}: {err}"
        res[rank] = outs
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    for r in range(1, world):   # the all-gather leaves every rank with the same bits
        for li in range(len(SHAPES)):
            assert np.array_equal(res[r][li], res[0][li]), f"rank {r} layer {SHAPES[li][0]} differs from rank 0"
    cur = synth.activation(H, N, seed=3)
    for li, (name, M, K) in enumerate(SHAPES):
        if name == "o":
            cur = cur[:H]
        W = synth.weight(M, K, S, seed=40 + li)
        Yref = oracle.spmm_f64(oracle.encode(W), np.ascontiguousarray(cur))
        assert_within(res[0][li], Yref, north_star_bound(W, cur), f"world {world} layer {name}")
        cur = res[0][li]
