"""The exact division by a per-round divisor the one-warp SA kernels use for the bit
draw (o0 mod n, Alg. 1) and the acceptance exponent (dE div tau, Eq.(7) reading E2):
abs_round_common.cuh make_udiv / udiv (Granlund-Montgomery round-up multiply).  The
same integer steps are evaluated here on the host against Python's // for divisors and
dividends at the edges of their ranges and at random; the GPU SA parity tests then pin
the kernels that use it to the oracle's plain % and //."""
import random

MASK32 = (1 << 32) - 1


def make_udiv(d):
    l = 0
    while l < 32 and (1 << l) < d:
        l += 1
    m = ((((1 << l) - d) << 32) // d + 1) & MASK32
    return d, m, min(l, 1), max(l - 1, 0)


def udiv(x, v):
    d, m, s1, s2 = v
    t = (m * x) >> 32
    return ((t + (((x - t) & MASK32) >> s1)) & MASK32) >> s2


def test_udiv_edges_and_random():
    rng = random.Random(7)
    divisors = [1, 2, 3, 5, 7, 16, 100, 1000, 1024, 2000, 2048, 10000, 32768, 65535, 65536,
                (1 << 31) - 1, 1 << 31, (1 << 31) + 1, MASK32 - 1, MASK32]
    divisors += [rng.randrange(1, 1 << 32) for _ in range(200)] + [rng.randrange(1, 1 << 16) for _ in range(200)]
    for d in divisors:
        v = make_udiv(d)
        assert v[1] <= MASK32
        xs = [0, 1, d - 1, d, d + 1, 2 * d - 1, 2 * d, MASK32, MASK32 - 1, (MASK32 // d) * d, (MASK32 // d) * d - 1]
        xs += [rng.randrange(0, 1 << 32) for _ in range(300)]
        for x in xs:
            if 0 <= x <= MASK32:
                assert udiv(x, v) == x // d, (x, d)
