"""The seeded input generator (shared by both sides; holds no method arithmetic)."""
import numpy as np

import synth


def _sm64(x):
    m = (1 << 64) - 1
    z = (x + 0x9E3779B97F4A7C15) & m
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & m
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & m
    return z ^ (z >> 31)


def test_splitmix_reference_values():
    # First outputs of the SplitMix64 stream seeded with 0 (x_i = i * golden gamma).
    assert synth.splitmix64(0) == 0xE220A8397B1DCDAF
    for x in (1, 12345, 2**63 + 7):
        assert synth.splitmix64(x) == _sm64(x)
    assert synth.hash64(20250330, 2, 17) == _sm64(((_sm64(20250330) ^ _sm64(2)) + 17) % 2**64)


def test_f64_to_f16_matches_numpy():
    rng = np.random.default_rng(0)
    xs = np.concatenate([rng.uniform(-1, 1, 20000), rng.uniform(-1e-5, 1e-5, 2000),
                         np.array([0.0, -0.0, 2**-24, 2**-25, 3 * 2**-26, 0.99999])])
    got = np.array([synth.f64_to_f16(float(x)) for x in xs], dtype=np.uint16)
    assert np.array_equal(got, xs.astype(np.float16).view(np.uint16))


def test_weight_deterministic_and_sparsity():
    a = synth.weight(256, 512, 0.5, seed=3)
    b = synth.weight(256, 512, 0.5, seed=3)
    c = synth.weight(256, 512, 0.5, seed=4)
    assert np.array_equal(a, b) and not np.array_equal(a, c)
    for s in (0.0, 0.3, 0.5, 0.7, 1.0):
        W = synth.weight(512, 512, s, seed=1)
        frac_zero = float(np.mean((W & 0x7FFF) == 0))
        n = W.size
        assert abs(frac_zero - s) <= 5 * np.sqrt(s * (1 - s) / n) + 1e-12
        vals = W[(W & 0x7FFF) != 0].view(np.float16).astype(np.float64)
        if vals.size:
            assert vals.min() >= -1.0 and vals.max() <= 1.0


def test_thread_count_independent():
    import os
    a = synth.weight(300, 128, 0.4, seed=8)
    # row-split threading must not change values: compare with a 1-row-at-a-time build
    b = np.vstack([synth.weight(300, 128, 0.4, seed=8)[i:i + 1] for i in (0, 150, 299)])
    assert np.array_equal(a[[0, 150, 299]], b)


def test_int_mode_values():
    W = synth.weight(128, 128, 0.5, seed=2, mode="int")
    v = W.view(np.float16).astype(np.float64)
    assert set(np.unique(v)) <= {-2.0, -1.0, 0.0, 1.0, 2.0}
    X = synth.activation(128, 16, seed=2, mode="int")
    assert set(np.unique(X.view(np.float16).astype(np.float64))) <= {-1.0, 0.0, 1.0}


def test_weight_row_shard_equals_rows_of_full_matrix():
    """synth.weight(row0=...) draws rows [row0, row0 + M) of the same matrix (per-rank shards in
    bench.py are the rows spinfer_tp_rows assigns, without generating the whole weight)."""
    for mode in ("uniform", "int"):
        W = synth.weight(320, 200, 0.5, seed=11, mode=mode)
        for b, c in [(0, 64), (64, 128), (192, 128), (300, 20)]:
            assert np.array_equal(synth.weight(c, 200, 0.5, seed=11, mode=mode, row0=b), W[b:b + c])
