"""Host-side logic of the CUDA path that can be checked without a GPU (-m "not gpu")."""
import random

KSEL = (0x18FC, 0x6EE1, 0x2333)   # csrc/spmm.cu kSelA, kSelB, kSelC


def prmt(a, b, sel):
    """PTX prmt.b32 default mode (byte permute with sign-replicate bit)."""
    src = [(a >> (8 * i)) & 0xFF for i in range(4)] + [(b >> (8 * i)) & 0xFF for i in range(4)]
    out = 0
    for i in range(4):
        n = (sel >> (4 * i)) & 0xF
        v = src[n & 7]
        if n & 8:
            v = 0xFF if v & 0x80 else 0
        out |= v << (8 * i)
    return out


def test_selector_polynomial_matches_two_phase_decode():
    """sel(y) = y*(A + B*y) + C reproduces Phase I / Phase II of P:287 for all bit pairs."""
    A, B, C = KSEL
    rng = random.Random(0)
    for y in range(4):
        sel = (y * ((A + B * y) & 0xFFFFFFFF) + C) & 0xFFFFFFFF
        b0, b1 = y & 1, y >> 1
        for _ in range(2000):
            v0, v1 = rng.randrange(65536), rng.randrange(65536)   # V[count], V[count+1]
            lo = v0 if b0 else 0
            hi = (v1 if b0 else v0) if b1 else 0
            assert prmt(v0, v1, sel) == (hi << 16) | lo


def test_masked_popcount_as_multiply():
    """popc(w & ((1 << sh) - 1)) == popc((w * 2^(32-sh)) mod 2^32), multiplier 0 for sh = 0."""
    rng = random.Random(1)
    for _ in range(5000):
        w = rng.getrandbits(32)
        sh = 2 * rng.randrange(16)
        mul = (1 << (32 - sh)) & 0xFFFFFFFF if sh else 0
        assert bin((w * mul) & 0xFFFFFFFF).count("1") == bin(w & ((1 << sh) - 1)).count("1")


def test_stream_k_partition():
    """unit_start / unit_owner of csrc/spmm.cu: contiguous, balanced, owner inverse."""
    for U in (1, 7, 148, 1000, 28672, 41472):
        for P in (1, 3, 148, 296):
            if P > U:
                continue
            start = [p * U // P for p in range(P + 1)]
            assert start[0] == 0 and start[-1] == U
            sizes = [start[p + 1] - start[p] for p in range(P)]
            assert max(sizes) - min(sizes) <= 1 and min(sizes) >= 1
            for u in range(0, U, max(1, U // 97)):
                owner = ((u + 1) * P - 1) // U
                assert start[owner] <= u < start[owner + 1]
