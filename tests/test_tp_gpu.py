"""GPU tests of the row-partitioned path through the C ABI.

One process plays every rank of a world in turn on cuda:0: each rank's spinfer_spmm_tp call
writes exactly its rows of the shared Y_full (no communication inside the library), so after all
ranks Y_full must equal the oracle's full product. The config-5 layer stack runs through
tp.run_stack with the real kernels at world size 1 (the NCCL gather itself is covered by the
gloo tests in test_tp_cpu.py; one GPU is all this harness has).
"""
import numpy as np
import pytest

import oracle
import synth
from tests.helpers import assert_within, f16_bits, north_star_bound, to_dev

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("N", [16, 32])
@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_spmm_tp_every_rank(world, N):
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    M, K = 1600, 768                       # 25 GT rows: uneven row chunks for world 2, 3, 4, 8
    W = synth.weight(M, K, 0.5, seed=world * 100 + N)
    X = synth.activation(K, N, seed=7)
    T = sp.encode(to_dev(W))
    Xd = to_dev(X).view(torch.float16)
    Y_slice = torch.full((M, N), float("nan"), dtype=torch.float16, device="cuda")
    Y_own = torch.full((M, N), float("nan"), dtype=torch.float16, device="cuda")
    covered = np.zeros(M, dtype=bool)
    for rank in range(world):
        b, c = sp.tp_rows(M, world, rank)
        assert (b, c) == oracle.tp_rows(M, world, rank)
        covered[b:b + c] = True
        sp.spmm_tp(T.shard(b, c), Xd, Y_slice, M, world, rank)          # zero-copy shard (P-E5)
        Ts = sp.encode(to_dev(np.ascontiguousarray(W[b:b + c])))         # rank encodes its own rows
        assert np.array_equal(Ts.bitmap.cpu().numpy(), T.shard(b, c).bitmap.cpu().numpy())
        sp.spmm_tp(Ts, Xd, Y_own, M, world, rank)
    torch.cuda.synchronize()
    assert covered.all()
    Yref = oracle.spmm_f64(oracle.encode(W), X)
    bound = north_star_bound(W, X)
    assert_within(f16_bits(Y_slice), Yref, bound, f"tp world={world} N={N} (slice)")
    assert np.array_equal(f16_bits(Y_slice), f16_bits(Y_own)), "shard slice and per-rank encode disagree"


def test_run_stack_world1_real_kernels():
    """Config-5 dataflow (QKV -> O on the Q block -> FC1 -> FC2) with the CUDA kernels, scaled
    down (h = 256, ffn = 1024); each layer is checked against the oracle applied to the GPU's
    own input of that layer (so errors do not compound across layers)."""
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    from paper_conf_eurosys_fanydlgww025_b200 import tp
    h, f, N, s = 256, 1024, 16, 0.6
    shapes = [("qkv", 3 * h, h), ("o", h, h), ("fc1", f, h), ("fc2", h, f)]
    Ws, layers = [], []
    for i, (name, M, K) in enumerate(shapes):
        W = synth.weight(M, K, s, seed=40 + i)
        Ws.append(W)
        layers.append(tp.Layer(name, M, K, 0, M, shard=sp.encode(to_dev(W)), x_rows=h if name == "o" else None))
    X = synth.activation(h, N, seed=3)
    outs = [torch.empty((M, N), dtype=torch.float16, device="cuda") for _, M, _ in shapes]
    tp.run_stack(layers, to_dev(X).view(torch.float16), 1, 0, outputs=outs)
    torch.cuda.synchronize()
    cur = X
    for i, (name, M, K) in enumerate(shapes):
        if name == "o":
            cur = cur[:h]
        Yref = oracle.spmm_f64(oracle.encode(Ws[i]), np.ascontiguousarray(cur))
        Y = f16_bits(outs[i])
        assert_within(Y, Yref, north_star_bound(Ws[i], cur), f"layer {name}")
        cur = Y


@pytest.mark.parametrize("N", [13, 16, 32])
@pytest.mark.parametrize("graph", [False, True])
def test_stack_pdl_matches_serial(graph, N):
    """SPINFER_OPT_PDL: the layer stack's SpMMs (one shared workspace, each layer's X the previous
    layer's Y) launched with programmatic dependent launch give the same bits as serial launches,
    eagerly and replayed from a CUDA graph; the first layer also matches the oracle."""
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    from paper_conf_eurosys_fanydlgww025_b200 import tp
    h, f, s = 256, 1024, 0.6
    shapes = [("qkv", 3 * h, h), ("o", h, h), ("fc1", f, h), ("fc2", h, f)] * 2
    ws = torch.zeros(max(sp.workspace_bytes(M, K, N) for _, M, K in shapes), dtype=torch.uint8, device="cuda")
    layers, Ws = [], []
    for i, (name, M, K) in enumerate(shapes):
        W = synth.weight(M, K, s, seed=60 + i)
        Ws.append(W)
        # FC1 with the fused ReLU epilogue (spinfer_spmm_ex); N = 13 adds the X padding kernel in between
        layers.append(tp.Layer(name, M, K, 0, M, shard=sp.encode(to_dev(W)), x_rows=h if name == "o" else None, ws=ws,
                               act="relu" if name == "fc1" else None))
    X = to_dev(synth.activation(h, N, seed=5)).view(torch.float16)

    def run(pdl):
        sp.set_option("pdl", pdl)
        outs = [torch.empty((M, N), dtype=torch.float16, device="cuda") for _, M, _ in shapes]
        if graph:
            cs = torch.cuda.Stream()
            cs.wait_stream(torch.cuda.current_stream())
            with torch.cuda.stream(cs):
                tp.run_stack(layers, X, 1, 0, outputs=outs)
            torch.cuda.current_stream().wait_stream(cs)
            torch.cuda.synchronize()
            for o in outs:
                o.fill_(0)
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                tp.run_stack(layers, X, 1, 0, outputs=outs)
            for _ in range(3):
                g.replay()
        else:
            for _ in range(3):
                tp.run_stack(layers, X, 1, 0, outputs=outs)
        torch.cuda.synchronize()
        return [f16_bits(o) for o in outs]

    ref = run(0)
    got = run(1)
    sp.set_option("pdl", 0)
    assert sp.check(ws) == 0
    for i, (a, b) in enumerate(zip(ref, got)):
        assert np.array_equal(a, b), f"layer {i} ({shapes[i][0]}): PDL result differs"
    Yref = oracle.spmm_f64(oracle.encode(Ws[0]), synth.activation(h, N, seed=5))
    assert_within(got[0], Yref, north_star_bound(Ws[0], synth.activation(h, N, seed=5)), "layer 0")
