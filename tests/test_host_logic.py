"""Host-side logic of the CUDA path that can be checked without a GPU (-m "not gpu")."""
import random

KSEL = (0x7F62, 0x4CBF, 0x2333)   # csrc/spmm.cu kSelA, kSelB, kSelC


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
    """sel(y) = y*(A + B*y) + C reproduces Phase I / Phase II of P:287 for all bit pairs,
    with t_lo = V[c2 - 2], t_hi = V[c2 - 1], c2 = MaskedPopCount + b0 + b1."""
    A, B, C = KSEL
    rng = random.Random(0)
    for y in range(4):
        sel = (y * ((A + B * y) & 0xFFFFFFFF) + C) & 0xFFFFFFFF
        b0, b1 = y & 1, y >> 1
        for _ in range(2000):
            V = [rng.randrange(65536) for _ in range(8)]
            cnt = rng.randrange(2, 6)                       # MaskedPopCount (values before the pair)
            c2 = cnt + b0 + b1
            t_lo, t_hi = V[c2 - 2], V[c2 - 1]
            lo = V[cnt] if b0 else 0                        # Phase I
            hi = V[cnt + b0] if b1 else 0                   # Phase II
            assert prmt(t_lo, t_hi, sel) == (hi << 16) | lo


def test_selector_search_reproduces_constants():
    import importlib.util, os
    spec = importlib.util.spec_from_file_location(
        "sel", os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools", "selector_search.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    assert KSEL in m.search()


def test_pair_count_and_bits_as_multiply():
    """z = w * 2^(30-sh) mod 2^32: z >> 30 = bits (sh, sh+1) and popc(z) = popc(w & ((4 << sh) - 1))."""
    rng = random.Random(1)
    for _ in range(5000):
        w = rng.getrandbits(32)
        sh = 2 * rng.randrange(16)
        z = (w * (1 << (30 - sh))) & 0xFFFFFFFF
        assert z >> 30 == (w >> sh) & 3
        assert bin(z).count("1") == bin(w & ((4 << sh) - 1)).count("1")


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
