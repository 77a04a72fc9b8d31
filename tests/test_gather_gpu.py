"""Fused all-gather epilogue (spinfer_spmm_tp_gather / spinfer_gather_wait),
on one GPU: world 1 is the loopback case; worlds 2-4 give every simulated rank its own Y buffer
and counter on the same device, and each rank's call must fill its rows of EVERY buffer and signal
every counter, so that after the waits all buffers equal the full product (the peer-store and
counter logic; NVLink peer mapping itself is exercised only on a multi-GPU node)."""
import numpy as np
import pytest

import oracle
import synth
from tests.helpers import assert_within, f16_bits, north_star_bound, to_dev

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("world", [1, 2, 3, 4])
@pytest.mark.parametrize("N", [8, 16, 13])
def test_gather_all_ranks(world, N):
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    M, K = 1600, 768                         # 25 GT rows: uneven row chunks
    W = synth.weight(M, K, 0.5, seed=world * 10 + N)
    X = synth.activation(K, N, seed=3)
    T = sp.encode(to_dev(W))
    Xd = to_dev(X)
    Ys = [torch.full((M, N), float("nan"), dtype=torch.float16, device="cuda") for _ in range(world)]
    flags = torch.zeros(world * 4, dtype=torch.int32, device="cuda")   # 16-B apart
    state = torch.zeros(world * 4, dtype=torch.int32, device="cuda")
    fp = [flags.data_ptr() + 16 * r for r in range(world)]
    for rep in range(2):                     # two exchanges: the counters keep counting
        for r in range(world):
            b, c = sp.tp_rows(M, world, r)
            sp.spmm_tp_gather(T.shard(b, c), Xd, Ys, M, world, r, fp)
        ws = sp.workspace(M, K, N)
        for r in range(world):
            sp.gather_wait(fp[r], state.data_ptr() + 16 * r, world, ws=ws, timeout_us=2_000_000)
        torch.cuda.synchronize()
        assert sp.check(ws) == 0
        assert flags.view(world, 4)[:, 0].tolist() == [world * (rep + 1)] * world
    Yref = oracle.spmm_f64(oracle.encode(W), X)
    for r in range(world):
        assert_within(f16_bits(Ys[r]), Yref, north_star_bound(W, X), f"rank {r} of {world}")
        assert np.array_equal(f16_bits(Ys[r]), f16_bits(Ys[0]))


def test_gather_wait_times_out():
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    flag = torch.zeros(4, dtype=torch.int32, device="cuda")
    state = torch.zeros(4, dtype=torch.int32, device="cuda")
    ws = sp.workspace(128, 128, 16)
    sp.gather_wait(flag, state, 2, ws=ws, timeout_us=2000)   # nobody signals
    torch.cuda.synchronize()
    assert sp.check(ws) & 4


def test_gather_rejects_wide_n():
    import torch
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    T = sp.encode(to_dev(synth.weight(128, 128, 0.5)))
    X = torch.zeros((128, 32), dtype=torch.float16, device="cuda")
    Y = torch.zeros((128, 32), dtype=torch.float16, device="cuda")
    f = torch.zeros(4, dtype=torch.int32, device="cuda")
    with pytest.raises(sp.SpinferError):
        sp.spmm_tp_gather(T, X, [Y], 128, 1, 0, [f])
