"""GPU TCA-BME encoder/decoder: bit-exact against the CPU oracle (-m gpu)."""
import numpy as np
import pytest

import oracle
import synth
from tests.helpers import f16_bits, to_dev

pytestmark = pytest.mark.gpu


def _sp():
    import paper_conf_eurosys_fanydlgww025_b200 as sp
    return sp


def check_encode(W: np.ndarray):
    import torch
    sp = _sp()
    T = sp.encode(to_dev(W))
    R = oracle.encode(W)
    assert T.n_values == R.n_values
    assert T.nnz == R.nnz
    assert T.max_gt_values == R.max_gt_values
    assert np.array_equal(T.gtile_offset.cpu().numpy(), R.gtile_offset)
    assert np.array_equal(T.bitmap.cpu().numpy().view(np.uint64), R.bitmap)
    assert np.array_equal(f16_bits(T.values[: T.n_values]), R.values)
    # decode(encode(W)) == canon(W) on the GPU
    D = f16_bits(sp.decode(T))
    assert np.array_equal(D, oracle.decode(R))
    torch.cuda.synchronize()
    return T, R


@pytest.mark.parametrize("M,K", [(64, 64), (256, 256), (192, 320), (1024, 512), (64, 4096)])
@pytest.mark.parametrize("s", [0.0, 0.3, 0.5, 0.7, 0.95, 1.0])
def test_encode_random(M, K, s):
    check_encode(synth.weight(M, K, s, seed=M * 7 + K + int(s * 100)))


def test_encode_structured():
    M, K = 256, 192
    r, c = np.indices((M, K))
    pats = [(r + c) % 2 == 0, r == c, (r % 17) == 3, (c % 13) == 5, (r // 8 == 5) & (c // 8 == 9),
            r <= c, (r < 64) & (c < 64)]
    for m in pats:
        check_encode(np.where(m, 0x3C00 + (r * K + c) % 1000, 0).astype(np.uint16))


def test_encode_special_values():
    W = synth.weight(128, 128, 0.5, seed=3)
    W[0, 0] = 0x8000   # -0.0 dropped
    W[1, 1] = 0x7C00   # +inf kept
    W[2, 2] = 0x7E00   # NaN kept
    W[3, 3] = 0x0001   # subnormal kept
    W[4, 4] = 0xFC00   # -inf kept
    check_encode(W)


def test_encode_config1_and_checkerboard_storage():
    T, R = check_encode(synth.weight(256, 256, 0.5))
    assert T.storage_bytes() == oracle.storage_bytes(256, 256, R.n_values)
    r, c = np.indices((256, 256))
    T2, _ = check_encode(np.where((r + c) % 2 == 0, 0x3C00, 0).astype(np.uint16))
    assert T2.storage_bytes() == 73796   # tests/golden/checkerboard.json


def test_encode_config2_full_size():
    """M/K = 28672/8192 at 50%: bit-exact with the oracle on the whole matrix."""
    check_encode(synth.weight(28672, 8192, 0.5))


def test_encode_invalid_shape():
    """Ragged shapes are valid (zero-padded, reading A8; tests/test_ragged_gpu.py); an empty W is not."""
    import torch
    sp = _sp()
    with pytest.raises(sp.SpinferError):
        sp.encode(torch.zeros((0, 64), dtype=torch.float16, device="cuda"))
