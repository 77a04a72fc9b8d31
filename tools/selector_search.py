"""Exhaustive search for the SMBD selector polynomial sel(y) = y*(A + B*y) + C (mod 2^16)
used by the consumer warps (csrc/spmm.cu, kSelA/kSelB/kSelC).

Loads: t_lo = V[c2 - 2], t_hi = V[c2 - 1] (zero-extended u16), where c2 = number of set
bits of the half-word up to and including the lane's pair. The final prmt(t_lo, t_hi, sel)
must give (a1 << 16) | a0 with (b0 = y & 1, b1 = y >> 1):
  y = 0 -> (0, 0)          y = 1 -> a0 = t_hi
  y = 2 -> a1 = t_hi        y = 3 -> a0 = t_lo, a1 = t_hi
Zero bytes: source bytes 2, 3, 6, 7 (also in sign-replicate mode: nibbles 10, 11, 14, 15)."""
Z = [2, 3, 6, 7, 10, 11, 14, 15]


def targets():
    # nibble constraints per y: list of allowed values per nibble (low nibble first)
    lo_t0, hi_t0 = 0, 1          # t_lo bytes
    lo_t1, hi_t1 = 4, 5          # t_hi bytes
    return {
        0: [Z, Z, Z, Z],
        1: [[lo_t1], [hi_t1], Z, Z],
        2: [Z, Z, [lo_t1], [hi_t1]],
        3: [[lo_t0], [hi_t0], [lo_t1], [hi_t1]],
    }


def ok(y, sel, T):
    return all(((sel >> (4 * i)) & 0xF) in T[y][i] for i in range(4))


def search():
    T = targets()
    M = 1 << 16
    import itertools
    def vals(y):
        return [a | (b << 4) | (c << 8) | (d << 12) for a in T[y][0] for b in T[y][1] for c in T[y][2] for d in T[y][3]]
    sols = []
    V0, V1, V2, V3 = vals(0), vals(1), vals(2), set(vals(3))
    for C in V0:
        for s1 in V1:
            for s2 in V2:
                t = (s2 - C - 2 * (s1 - C)) % M
                if t & 1:
                    continue
                for B in (t // 2, t // 2 + M // 2):
                    A = (s1 - C - B) % M
                    if (3 * A + 9 * B + C) % M in V3:
                        sols.append((A, B, C))
    return sols


if __name__ == "__main__":
    s = search()
    print(len(s), [tuple(hex(x) for x in t) for t in s[:5]])
