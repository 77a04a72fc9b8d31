"""Exhaustive search for the SMBD selector polynomial sel(y) = y*(A + B*y) + C (mod 2^16)
used by the consumer warps (csrc/spmm.cu, kSelA/kSelB/kSelC). The final
prmt(t0, t1, sel(y)) must give (a1 << 16) | a0 with
  y = 0 -> (0, 0),  y = 1 -> (t0, 0),  y = 2 -> (0, t0),  y = 3 -> (t0, t1)
where t0, t1 are zero-extended u16 loads: zero bytes are source bytes 2, 3, 6, 7
(also in sign-replicate mode, nibbles 10, 11, 14, 15)."""
import numpy as np

Z = [2, 3, 6, 7, 10, 11, 14, 15]


def search():
    M = 1 << 16
    C_all = [a | (b << 4) | (c << 8) | (d << 12) for a in Z for b in Z for c in Z for d in Z]
    S1 = [0x10 | (c << 8) | (d << 12) for c in Z for d in Z]
    S2 = [a | (b << 4) | 0x1000 for a in Z for b in Z]
    sols = []
    for C in C_all:
        for s1 in S1:
            for s2 in S2:
                t = (s2 - C - 2 * (s1 - C)) % M
                if t & 1:
                    continue
                for B in (t // 2, t // 2 + M // 2):
                    A = (s1 - C - B) % M
                    if (3 * A + 9 * B + C) % M == 0x5410:
                        sols.append((A, B, C))
    return sols


if __name__ == "__main__":
    s = search()
    print(len(s), [tuple(hex(x) for x in t) for t in s[:5]])
