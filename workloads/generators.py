"""Workload generators (inputs only; see package docstring).

Every generator is a pure function of its arguments: numpy's counter-based
Philox bit generator keyed by (seed, stream tag, block coordinates) so a block
of W can be regenerated independently of the others and the result does not
depend on the order of generation.

Bit-vector format (the C-ABI's, include/abs.h): bit i of an n-bit vector is
bit (i & 31) of uint32 word (i >> 5); words = ceil(n / 32); bits >= n are 0.

Workload families (§4.1):
  * synthetic random QUBO  - W_ij = W_ji ~ U{-32768..32767}
  * Max-Cut                - W_ij = G_ij (i != j), W_ii = -sum_k G_ik (Eq.17)
  * TSP                    - one-hot c*c encoding, penalty A = 2*d_max (
                             encoding details are DESIGN.md reading C13)
"""
from __future__ import annotations

import math

import numpy as np

_BLOCK = 4096

# stream tags (keep generators for different families independent)
_TAG_RANDOM_QUBO = 0x52514255  # 'RQBU'
_TAG_MAXCUT = 0x4D435554       # 'MCUT'
_TAG_TSP = 0x54535020          # 'TSP '
_TAG_SOLUTIONS = 0x534F4C53    # 'SOLS'


def _rng(seed: int, tag: int, a: int = 0, b: int = 0) -> np.random.Generator:
    key = [(int(seed) & 0xFFFFFFFFFFFFFFFF), ((tag & 0xFFFFFFFF) << 32) | ((a & 0xFFFF) << 16) | (b & 0xFFFF)]
    return np.random.Generator(np.random.Philox(key=key))


def words_per_vector(n: int) -> int:
    return (int(n) + 31) // 32


def random_qubo(n: int, seed: int = 1) -> np.ndarray:
    """Synthetic random QUBO: dense symmetric int16 n x n with the
    upper triangle (incl. diagonal) i.i.d. uniform over all 65536 int16 values.

    Generated in 4096 x 4096 blocks, block (bi, bj), bi <= bj, from its own
    Philox stream, so n = 32768 (2 GiB) needs no full-size temporaries.
    """
    n = int(n)
    if n < 1:
        raise ValueError("n must be >= 1")
    W = np.empty((n, n), dtype=np.int16)
    nb = (n + _BLOCK - 1) // _BLOCK
    for bi in range(nb):
        r0, r1 = bi * _BLOCK, min(n, (bi + 1) * _BLOCK)
        for bj in range(bi, nb):
            c0, c1 = bj * _BLOCK, min(n, (bj + 1) * _BLOCK)
            U = _rng(seed, _TAG_RANDOM_QUBO, bi, bj).integers(
                -32768, 32767, size=(r1 - r0, c1 - c0), endpoint=True, dtype=np.int16)
            if bi == bj:
                up = np.triu(U)
                W[r0:r1, c0:c1] = up + np.triu(U, 1).T
            else:
                W[r0:r1, c0:c1] = U
                W[c0:c1, r0:r1] = U.T
    return W


_TAG_RQBC = 0x52514243  # 'RQBC': counter-based random QUBO (random_qubo_ctr)


def _philox4x32_10(c0, c1, c2, c3, k0: int, k1: int):
    """Philox4x32-10 (Salmon et al., SC'11) over numpy uint32 arrays of
    counters; an input generator only (the method's own draws are elsewhere)."""
    c0, c1, c2, c3 = (np.asarray(v, dtype=np.uint32) for v in (c0, c1, c2, c3))
    c0, c1, c2, c3 = np.broadcast_arrays(c0, c1, c2, c3)
    k0, k1 = np.uint32(k0 & 0xFFFFFFFF), np.uint32(k1 & 0xFFFFFFFF)
    M0, M1 = np.uint64(0xD2511F53), np.uint64(0xCD9E8D57)
    for _ in range(10):
        p0 = c0.astype(np.uint64) * M0
        p1 = c2.astype(np.uint64) * M1
        c0, c1, c2, c3 = ((p1 >> np.uint64(32)).astype(np.uint32) ^ c1 ^ k0, p1.astype(np.uint32),
                          (p0 >> np.uint64(32)).astype(np.uint32) ^ c3 ^ k1, p0.astype(np.uint32))
        k0 = np.uint32((int(k0) + 0x9E3779B9) & 0xFFFFFFFF)
        k1 = np.uint32((int(k1) + 0xBB67AE85) & 0xFFFFFFFF)
    return c0, c1, c2, c3


def random_qubo_ctr_rows(n: int, seed: int, r0: int, r1: int) -> np.ndarray:
    """Rows [r0, r1) of random_qubo_ctr(n, seed), without building the rest."""
    n = int(n)
    out = np.empty((r1 - r0, n), dtype=np.int16)
    groups = (n + 7) // 8
    k0, k1 = int(seed) & 0xFFFFFFFF, (int(seed) >> 32) & 0xFFFFFFFF
    for a in range(r0, r1, 256):
        b = min(r1, a + 256)
        rows = np.arange(a, b, dtype=np.uint32)[:, None]
        # upper part of row i (j >= i): the row's own stream
        o = _philox4x32_10(rows, np.arange(groups, dtype=np.uint32)[None, :], _TAG_RQBC, 0, k0, k1)
        up = np.stack(o, axis=-1).astype("<u4").view("<i2").reshape(b - a, groups * 8)[:, :n]
        # lower part (j < i): W_ij = W_ji = half (i & 1) of word ((i >> 1) & 3) of the stream of row j
        cols = np.arange(n, dtype=np.uint32)[None, :]
        ol = _philox4x32_10(cols, (rows >> np.uint32(3)), _TAG_RQBC, 0, k0, k1)
        words = np.stack(ol, axis=-1)                                        # [rows, n, 4]
        sel = ((np.arange(a, b) >> 1) & 3)[:, None, None]
        w = np.take_along_axis(words, np.broadcast_to(sel, (b - a, n, 1)), axis=2)[..., 0]
        half = (w >> ((np.arange(a, b, dtype=np.uint32) & 1) * 16)[:, None]).astype(np.uint16).view(np.int16)
        jj = np.arange(n)[None, :]
        ii = np.arange(a, b)[:, None]
        out[a - r0:b - r0] = np.where(jj >= ii, up, half)
    return out


def random_qubo_ctr(n: int, seed: int = 1) -> np.ndarray:
    """Synthetic random QUBO by a counter-based rule that the
    library also runs on the device (abs_random_qubo_dev, include/abs.h):
    W symmetric, upper triangle (i <= j)
        W_ij = int16 half (j & 1) of word ((j >> 1) & 3) of
               Philox4x32-10(key = (lo32 seed, hi32 seed), counter = (i, j >> 3, 'RQBC', 0)),
    i.i.d. uniform over all int16.  This host copy feeds the oracle; the GPU
    side generates its replica in HBM, so a multi-GPU run stages no 2 GiB
    host copy per rank."""
    n = int(n)
    if n < 1:
        raise ValueError("n must be >= 1")
    W = np.empty((n, n), dtype=np.int16)
    groups = (n + 7) // 8
    k0, k1 = int(seed) & 0xFFFFFFFF, (int(seed) >> 32) & 0xFFFFFFFF
    B = 512
    for r0 in range(0, n, B):
        r1 = min(n, r0 + B)
        g0 = r0 >> 3
        rows = np.arange(r0, r1, dtype=np.uint32)[:, None]
        o = _philox4x32_10(rows, np.arange(g0, groups, dtype=np.uint32)[None, :], _TAG_RQBC, 0, k0, k1)
        U = np.stack(o, axis=-1).astype("<u4").view("<i2").reshape(r1 - r0, (groups - g0) * 8)[:, :n - 8 * g0]
        # U[r, q] = value (r0 + r, 8 g0 + q) of the upper rule; keep j >= i
        c0 = r0 - 8 * g0                       # column of j = r0 inside U
        D = U[:, c0:c0 + (r1 - r0)]              # diagonal block
        W[r0:r1, r0:r1] = np.triu(D) + np.triu(D, 1).T
        if r1 < n:
            R = U[:, c0 + (r1 - r0):]
            W[r0:r1, r1:] = R
            W[r1:, r0:r1] = R.T
    return W


def maxcut_graph(n: int, m_edges: int, seed: int = 1, weights: str = "pm1"):
    """G(n, m) random graph: m distinct undirected edges drawn uniformly from
    the n(n-1)/2 pairs. weights: 'pm1' (+1/-1 equiprobable, G-set G27-like)
    or 'one' (+1, G22-like).  Returns (i, j, w) int arrays with i < j.
    The G-set edge count convention (m = 19,990 at n = 2,000) is SURVEY §8(d)
    config 3, not PAPER.md."""
    n = int(n)
    total = n * (n - 1) // 2
    if not (0 <= m_edges <= total):
        raise ValueError("bad edge count")
    rng = _rng(seed, _TAG_MAXCUT)
    idx = np.sort(rng.choice(total, size=m_edges, replace=False)).astype(np.int64)
    # map linear pair index -> (i, j), i < j, row-major over the strict upper triangle
    # row i starts at off(i) = i*(2n - i - 1)/2
    i = np.floor(((2 * n - 1) - np.sqrt((2 * n - 1) ** 2 - 8.0 * idx)) / 2).astype(np.int64)
    off = i * (2 * n - i - 1) // 2
    # fix floating point at boundaries
    too_big = off > idx
    i[too_big] -= 1
    off = i * (2 * n - i - 1) // 2
    nxt = (i + 1) * (2 * n - i - 2) // 2
    too_small = idx >= nxt
    i[too_small] += 1
    off = i * (2 * n - i - 1) // 2
    j = idx - off + i + 1
    if weights == "pm1":
        w = np.where(rng.integers(0, 2, size=m_edges) == 1, 1, -1).astype(np.int64)
    elif weights == "one":
        w = np.ones(m_edges, dtype=np.int64)
    else:
        raise ValueError(weights)
    return i, j, w


def maxcut_qubo(n: int, m_edges: int, seed: int = 1, weights: str = "pm1") -> np.ndarray:
    """Max-Cut -> QUBO by Eq.(17): W_ij = G_ij for i != j and
    W_ii = -sum_k G_ik, so E(X) = -cut(X) under Eq.(1)."""
    i, j, w = maxcut_graph(n, m_edges, seed, weights)
    G = np.zeros((n, n), dtype=np.int64)
    G[i, j] = w
    G[j, i] = w
    W = G.copy()
    W[np.arange(n), np.arange(n)] = -G.sum(axis=1)
    if W.min() < -32768 or W.max() > 32767:
        raise ValueError("Max-Cut weights do not fit int16")
    return W.astype(np.int16)


def tsp_instance(c: int, seed: int = 1, box: int = 5792):
    """c cities with integer coordinates uniform in [0, box]^2 and TSPLIB
    EUC_2D distances d = nint(sqrt(dx^2 + dy^2)).  box = 5792 keeps
    d_max <= 8191 so that A = 2 d_max and -2A fit int16 (C13)."""
    rng = _rng(seed, _TAG_TSP)
    xy = rng.integers(0, box, size=(c, 2), endpoint=True).astype(np.int64)
    dx = xy[:, None, 0] - xy[None, :, 0]
    dy = xy[:, None, 1] - xy[None, :, 1]
    d = np.floor(np.sqrt((dx * dx + dy * dy).astype(np.float64)) + 0.5).astype(np.int64)
    return xy, d


def tsp_qubo(c: int, seed: int = 1, d: np.ndarray | None = None, penalty: int | None = None) -> np.ndarray:
    """TSP -> QUBO, c*c one-hot encoding (row = city u, column = visit order t,
    bit b = u*c + t; Fig. 7 P:L462-466 layout).  Reading C13:
      * tour length: W[(u,t),(v,t+1 mod c)] = W[(v,t+1),(u,t)] = d_uv (u != v)
      * one-hot penalties A*(sum_t x_ut - 1)^2 + A*(sum_u x_ut - 1)^2 with
        A = 2*d_max ("twice as much as the maximum distance"):
        W[(u,t),(u,t')] = A (t != t'), W[(u,t),(v,t)] = A (u != v), W_ii = -2A
    Under Eq.(1) a valid tour then has E = 2*len - 2*c*A."""
    if c < 3:
        raise ValueError("need c >= 3")
    if d is None:
        _, d = tsp_instance(c, seed)
    d = np.asarray(d, dtype=np.int64)
    A = int(penalty) if penalty is not None else 2 * int(d.max())
    n = c * c
    W = np.zeros((n, n), dtype=np.int64)
    u = np.arange(c)
    for t in range(c):
        t1 = (t + 1) % c
        rows = u * c + t
        cols = u * c + t1
        # d_uv between (u,t) and (v,t+1), u != v (d_uu = 0 anyway)
        blk = d.copy()
        np.fill_diagonal(blk, 0)
        W[np.ix_(rows, cols)] += blk
        W[np.ix_(cols, rows)] += blk.T
    for x in range(c):
        row_bits = x * c + np.arange(c)          # same city, all orders
        col_bits = np.arange(c) * c + x          # same order, all cities
        W[np.ix_(row_bits, row_bits)] += A
        W[np.ix_(col_bits, col_bits)] += A
    diag = np.arange(n)
    W[diag, diag] = -2 * A
    if W.min() < -32768 or W.max() > 32767:
        raise ValueError("TSP weights do not fit int16")
    return W.astype(np.int16)


def random_solutions(count: int, n: int, seed: int = 1, p_one: float = 0.5) -> np.ndarray:
    """count random n-bit vectors in the ABI's packed format (uint32
    [count, ceil(n/32)], bits >= n zero)."""
    rng = _rng(seed, _TAG_SOLUTIONS)
    bits = rng.random((count, n)) < p_one
    return pack_bits(bits)


def pack_bits(bits: np.ndarray) -> np.ndarray:
    """bool [count, n] -> uint32 [count, ceil(n/32)] (bit i -> word i>>5, bit i&31)."""
    bits = np.atleast_2d(np.asarray(bits, dtype=bool))
    count, n = bits.shape
    words = words_per_vector(n)
    padded = np.zeros((count, words * 32), dtype=bool)
    padded[:, :n] = bits
    by = np.packbits(padded.reshape(count, words * 4, 8), axis=2, bitorder="little").reshape(count, words * 4)
    return by.view("<u4").reshape(count, words).copy()


def unpack_bits(words: np.ndarray, n: int) -> np.ndarray:
    """uint32 [count, words] -> bool [count, n]."""
    w = np.atleast_2d(np.ascontiguousarray(words, dtype="<u4"))
    by = w.view(np.uint8)
    return np.unpackbits(by, axis=1, bitorder="little")[:, :n].astype(bool)


def _selfcheck():  # pragma: no cover
    W = random_qubo(5000, 3)
    assert (W == W.T).all()
    assert math.isclose(float(W.astype(np.float64).mean()), -0.5, abs_tol=60)
