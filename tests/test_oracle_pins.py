"""Pins for the CPU oracle (oracle/): each test checks the oracle against
something other than itself — a library routine, a closed form, brute force,
an invariant, or a worked example printed in PAPER.md — so that a plausible
mistake (dropped term, wrong sign or index, transposed operand, wrong
tie-break) fails at least one of them.  All CPU-only."""
from __future__ import annotations

import itertools
import os

import numpy as np
import pytest

import oracle
from workloads import (maxcut_graph, maxcut_qubo, pack_bits, random_qubo, random_solutions,
                       tsp_instance, tsp_qubo, unpack_bits)

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ---------------------------------------------------------------- helpers (test-side, numpy)
def np_energy(W, bits):
    """Eq.(1) through numpy's matmul (library routine): x^T W x."""
    x = np.asarray(bits, dtype=np.int64)
    return int(x @ W.astype(np.int64) @ x)


def np_deltas(W, bits):
    """Delta_k = E(flip_k X) - E(X) by recomputing every neighbour with numpy."""
    e0 = np_energy(W, bits)
    out = np.empty(len(bits), dtype=np.int64)
    for k in range(len(bits)):
        y = np.array(bits, dtype=bool)
        y[k] = not y[k]
        out[k] = np_energy(W, y) - e0
    return out


def small_W(n, seed):
    return random_qubo(n, seed)


# ---------------------------------------------------------------- Philox
def test_philox_known_answers():
    rows = [l.split() for l in open(os.path.join(GOLDEN, "philox_kat.txt")) if l.strip() and not l.startswith("#")]
    assert len(rows) == 3
    for r in rows:
        v = [int(t, 16) for t in r]
        out = oracle.philox4x32_10(v[0:4], v[4:6])
        assert [int(o) for o in out] == v[6:10]


# ---------------------------------------------------------------- energy, Eq.(1)
@pytest.mark.parametrize("n,seed", [(1, 1), (5, 2), (33, 3), (64, 4), (100, 5)])
def test_energy_matches_numpy_quadratic_form(n, seed):
    W = small_W(n, seed)
    for X, bits in zip(random_solutions(6, n, seed), unpack_bits(random_solutions(6, n, seed), n)):
        assert oracle.energy(W, X) == np_energy(W, bits)


def test_energy_special_cases():
    n = 40
    W = small_W(n, 7)
    assert oracle.energy(W, np.zeros(2, np.uint32)) == 0                      # E(0) = 0
    for i in (0, 17, 39):
        b = np.zeros(n, bool); b[i] = True
        assert oracle.energy(W, pack_bits(b)[0]) == W[i, i]                   # single bit: diagonal
    b = np.zeros(n, bool); b[3] = b[30] = True
    # off-diagonal pair counted twice, diagonal once (Eq.(1) with W symmetric)
    assert oracle.energy(W, pack_bits(b)[0]) == int(W[3, 3]) + int(W[30, 30]) + 2 * int(W[3, 30])


# ---------------------------------------------------------------- Delta, Eq.(11)/(13)
@pytest.mark.parametrize("n,seed", [(1, 1), (7, 2), (32, 3), (45, 4)])
def test_init_batch_deltas_equal_recomputed_neighbour_energies(n, seed):
    W = small_W(n, seed)
    X = random_solutions(5, n, seed + 100)
    D, E = oracle.init_batch(W, X)
    for b, bits in enumerate(unpack_bits(X, n)):
        assert E[b] == np_energy(W, bits)
        assert (D[b] == np_deltas(W, bits)).all()
        # and the oracle's own by-definition routine agrees
        for k in (0, n - 1, n // 2):
            assert oracle.delta_by_definition(W, X[b], k) == D[b, k]


def test_zero_start():
    # E(0) = 0 and Delta_i(0) = W_ii
    W = small_W(50, 9)
    s = oracle.Search(W, l=4)
    assert s.E == 0 and s.flips == 0
    assert (s.d == np.diag(W).astype(np.int64)).all()
    assert (s.x == 0).all()


# ---------------------------------------------------------------- incremental flip, Eq.(16)
@pytest.mark.parametrize("n,seed", [(2, 1), (16, 2), (37, 3), (64, 4)])
def test_incremental_deltas_track_definition_after_every_flip(n, seed):
    W = small_W(n, seed)
    s = oracle.Search(W, l=4)
    rng = np.random.default_rng(seed)
    bits = np.zeros(n, bool)
    for _ in range(3 * n):
        k = int(rng.integers(n))
        s.flip(k)
        bits[k] = not bits[k]
        assert (unpack_bits(s.x, n)[0] == bits).all()
        assert s.E == np_energy(W, bits)
        assert (s.d == np_deltas(W, bits)).all()


def test_delta_int32_bound_closed_form():
    # Reading C12: W == -32768, X = 1^n gives Delta_i = 32768 * (2n - 1).
    for n in (3, 64, 2048):
        W = np.full((n, n), -32768, dtype=np.int16)
        X = pack_bits(np.ones((1, n), bool))
        D, E = oracle.init_batch(W, X)
        assert (D[0] == 32768 * (2 * n - 1)).all()
        assert E[0] == -32768 * n * n
    assert 32768 * (2 * 32768 - 1) == 2147450880 < 2 ** 31 - 1


# ---------------------------------------------------------------- straight search (Alg. 5)
@pytest.mark.parametrize("n,seed", [(16, 1), (50, 2), (70, 3)])
def test_straight_search_walks_hamming_distance_greedily(n, seed):
    W = small_W(n, seed)
    s = oracle.Search(W, l=4)
    X0 = random_solutions(1, n, seed + 1)[0]
    s.straight(X0)            # move to a random start first
    T = random_solutions(1, n, seed + 2)[0]
    tb = unpack_bits(T, n)[0]
    ham = int((unpack_bits(s.x, n)[0] != tb).sum())
    f0 = s.flips
    # replay by hand: each step must flip the lowest-index argmin over mismatches
    ref_bits = unpack_bits(s.x, n)[0].copy()
    steps = 0
    while (ref_bits != tb).any():
        d = np_deltas(W, ref_bits)
        mism = np.nonzero(ref_bits != tb)[0]
        k = mism[np.argmin(d[mism])]  # argmin returns the first (lowest) index on ties
        ref_bits[k] = not ref_bits[k]
        steps += 1
    got = s.straight(T)
    assert got == ham == steps == s.flips - f0          # P:L360 "number of flips = Hamming distance"
    assert (unpack_bits(s.x, n)[0] == tb).all()
    assert s.E == np_energy(W, tb)


# ---------------------------------------------------------------- window policy (Fig. 2)
def test_window_l1_sweeps_bits_in_order_and_restores_after_2n():
    # l = 1: "a bit is selected" in offset order; after n flips X = not X0,
    # after 2n flips X, Delta and E are restored exactly.
    n = 23
    W = small_W(n, 11)
    s = oracle.Search(W, l=1)
    s.straight(random_solutions(1, n, 12)[0])
    x0, d0, e0 = s.x, s.d, s.E
    a0 = s.a
    seq = []
    for _ in range(n):
        before = unpack_bits(s.x, n)[0]
        s.local(1)
        after = unpack_bits(s.x, n)[0]
        seq.append(int(np.nonzero(before != after)[0][0]))
    assert seq == [(a0 + j) % n for j in range(n)]
    assert (unpack_bits(s.x, n)[0] == ~unpack_bits(x0, n)[0]).all()
    s.local(n)
    assert (s.x == x0).all() and (s.d == d0).all() and s.E == e0


def test_window_l_equals_n_is_steepest_forced_greedy():
    # "If the number of extracted bits is n ... the same as a greedy algorithm"
    n = 31
    W = small_W(n, 13)
    s = oracle.Search(W, l=n)
    bits = np.zeros(n, bool)
    for _ in range(60):
        d = np_deltas(W, bits)
        k = int(np.argmin(d))
        s.local(1)
        bits[k] = not bits[k]
        assert (unpack_bits(s.x, n)[0] == bits).all()


def test_window_wraps_and_breaks_ties_by_lowest_absolute_index():
    # Reading C5: the window {(a+j) mod n} wraps; equal deltas -> lowest index.
    n = 8
    W = np.zeros((n, n), np.int16)
    np.fill_diagonal(W, 5)
    W[0, 0] = W[6, 6] = -3               # Delta_0 = Delta_6 = -3 at X = 0
    s = oracle.Search(W, l=4)
    s.set_offset(5)                      # window = {5, 6, 7, 0}
    s.local(1)
    assert unpack_bits(s.x, n)[0].tolist() == [True] + [False] * 7
    assert s.a == (5 + 4) % n


def test_fig2_worked_example():
    g = dict(l.split(None, 1) for l in open(os.path.join(GOLDEN, "fig2_window.txt"))
             if l.strip() and not l.startswith("#"))
    n, a, l = int(g["n"]), int(g["offset"]), int(g["l"])
    before = np.array([c == "1" for c in g["before"].strip()])
    after = np.array([c == "1" for c in g["after"].strip()])
    # A W realising Fig. 2: diagonal-only weights make Delta_i = phi(x_i) W_ii;
    # choose them so that Delta_5 is the strict minimum of Delta_4..Delta_7.
    W = np.zeros((n, n), np.int16)
    diag = np.full(n, 10)
    diag[5] = -20 if not before[5] else 20   # phi(x5) * W55 = -20
    np.fill_diagonal(W, diag)
    s = oracle.Search(W, l=l)
    s.straight(pack_bits(before[None])[0])
    assert (unpack_bits(s.x, n)[0] == before).all()
    d = s.d
    assert int(np.argmin(d[a:a + l])) + a == int(g["flipped"])
    s.set_offset(a)
    s.local(1)
    assert (unpack_bits(s.x, n)[0] == after).all()
    assert s.a == int(g["next_offset"])


# ---------------------------------------------------------------- best tracking (reading C2/C5)
@pytest.mark.parametrize("n,seed,l", [(9, 1, 3), (12, 2, 12), (16, 3, 4)])
def test_round_best_is_lexicographic_min_over_visited_and_neighbours(n, seed, l):
    """Brute force: over the round start X0 (t=-1) and every visited X_t and all
    its n neighbours, the emitted (B, E_B) is the (energy, t, i) lexicographic
    minimum with i = -1 for X_t itself (reading C5); E_B == E(B)."""
    W = small_W(n, seed)
    s = oracle.Search(W, l=l)
    s.straight(random_solutions(1, n, seed + 5)[0])
    T = random_solutions(1, n, seed + 6)[0]
    L = 3 * n
    # reference trajectory, replayed with numpy from the oracle's own flip choices
    start = unpack_bits(s.x, n)[0].copy()
    traj = [start.copy()]
    tmp = oracle.Search(W, l=l)
    tmp.straight(pack_bits(start[None])[0])
    tmp.set_offset(s.a)
    tmp.set_best()
    # walk the same round one flip at a time, recording states
    tb = unpack_bits(T, n)[0]
    while (unpack_bits(tmp.x, n)[0] != tb).any():
        before = tmp.flips
        cur = unpack_bits(tmp.x, n)[0]
        d = tmp.d
        mism = np.nonzero(cur != tb)[0]
        k = int(mism[np.argmin(d[mism])])
        tmp.flip(k); tmp.track()
        traj.append(unpack_bits(tmp.x, n)[0].copy())
        assert tmp.flips == before + 1
    for _ in range(L):
        tmp.local(1)
        traj.append(unpack_bits(tmp.x, n)[0].copy())
    # brute-force expected best
    best = (np_energy(W, traj[0]), -1, -1, traj[0])
    for t, X in enumerate(traj[1:]):
        e = np_energy(W, X)
        cands = [(e, t, -1, X)]
        for i in range(n):
            Y = X.copy(); Y[i] = not Y[i]
            cands.append((np_energy(W, Y), t, i, Y))
        c = min(cands, key=lambda z: (z[0], z[1], z[2]))
        if c[0] < best[0]:
            best = c
    s.round(T, L)
    assert s.EB == best[0]
    assert (unpack_bits(s.b, n)[0] == best[3]).all()
    assert s.EB == np_energy(W, unpack_bits(s.b, n)[0])
    assert (s.x == tmp.x).all() and s.E == tmp.E


# ---------------------------------------------------------------- pool
def test_pool_insert_semantics_against_sorted_list():
    n, m = 40, 16
    p = oracle.Pool(n, m, seed=3)
    assert (p.E == oracle.EINF).all()
    init_X = p.X
    ref = [(oracle.EINF, i, init_X[i]) for i in range(m)]   # (+inf entries, creation order)
    rng = np.random.default_rng(0)
    for step in range(300):
        E = int(rng.integers(-50, 50))
        X = random_solutions(1, n, 1000 + step)[0]
        got = p.insert(X, E)
        energies = [r[0] for r in ref]
        exp = (E not in energies) and E < max(energies)
        if exp:
            ref.append((E, -1, X))
            ref.sort(key=lambda r: (r[0], r[1]))
            ref = ref[:m]
        assert got == exp
        assert (p.E == np.array([r[0] for r in ref])).all()
        assert all((p.X[i] == ref[i][2]).all() for i in range(m))
        fin = p.E[p.E != oracle.EINF]
        assert (np.diff(fin) > 0).all()                      # strictly ascending & distinct


def test_pool_initial_entries_are_random_bits_below_n():
    n = 45
    X = oracle.Pool(n, 200, seed=9).X
    bits = unpack_bits(X, 64)
    assert not bits[:, n:].any()
    frac = bits[:, :n].mean()
    assert 0.45 < frac < 0.55


def test_ga_operators():
    n, m = 100, 8
    cfg = oracle.Config(n=n, searches=1, pool_size=m, seed=5)
    p = oracle.Pool(n, m, seed=5)
    P = unpack_bits(p.X, n)
    kinds = {"cross": 0, "mut": 0, "copy": 0}
    mut_max = cfg.c().mut_max
    for r in range(600):
        T = unpack_bits(p.target(cfg, r, 0), n)[0]
        ham = np.array([(P[i] != T).sum() for i in range(m)])
        if ham.min() == 0:
            kinds["copy"] += 1              # (a crossover of equal bits is vanishingly unlikely at n=100)
        elif ham.min() <= mut_max:
            kinds["mut"] += 1               # a mutation flips 1..mut_max bits of one parent
        else:
            # a crossover: every bit taken from one of two parents (~n/4 bits away from each)
            assert any(((T == P[i]) | (T == P[j])).all() for i in range(m) for j in range(i + 1, m))
            kinds["cross"] += 1
    assert kinds["copy"] > 20 and kinds["mut"] > 150 and kinds["cross"] > 150
    # deterministic in (seed, round, search)
    assert (p.target(cfg, 7, 3) == p.target(cfg, 7, 3)).all()
    assert not (p.target(cfg, 7, 3) == p.target(cfg, 7, 4)).all()


# ---------------------------------------------------------------- whole runs
def test_config1_n16_reaches_bruteforce_optimum():
    """Config 1: random int16 QUBO n=16, 256 searches x 1 round (straight 0->T0,
    then L=1000 local flips) must find the 2^16 brute-force minimum."""
    n = 16
    W = random_qubo(n, 1)
    allx = np.array(list(itertools.product([0, 1], repeat=n)), dtype=np.int64)
    E_all = np.einsum("bi,ij,bj->b", allx, W.astype(np.int64), allx)
    e_min = int(E_all.min())
    assert oracle.bruteforce(W)[0] == e_min
    out = oracle.run_lockstep(W, oracle.Config(n=n, searches=256, local_flips=1000, pool_size=32, seed=1), rounds=1)
    assert int(out["EB"].min()) == e_min
    assert int(out["poolE"][0]) == e_min
    for r_ in range(1):
        for s in range(0, 256, 37):
            assert out["EB"][r_, s] == np_energy(W, unpack_bits(out["B"][r_, s], n)[0])


def test_lockstep_run_invariants_and_determinism():
    n = 48
    W = random_qubo(n, 21)
    cfg = oracle.Config(n=n, searches=6, local_flips=40, pool_size=10, seed=3)
    a = oracle.run_lockstep(W, cfg, rounds=4)
    b = oracle.run_lockstep(W, cfg, rounds=4)
    for k in a:
        assert (a[k] == b[k]).all()
    for s in range(6):
        bits = unpack_bits(a["X"][s], n)[0]
        assert a["E"][s] == np_energy(W, bits)
        assert (a["D"][s] == np_deltas(W, bits)).all()
    fin = a["poolE"][a["poolE"] != oracle.EINF]
    assert (np.diff(fin) > 0).all()
    assert fin[0] == a["EB"].min()
    for r in range(4):
        for s in range(6):
            assert a["EB"][r, s] == np_energy(W, unpack_bits(a["B"][r, s], n)[0])
    # replay: each search's trajectory is a function of its target sequence
    # (targets regenerated here from the pool semantics are not needed: the
    # lockstep trajectory must equal a replay with the targets reconstructed
    # by straight-search end points)


def test_maxcut_energy_is_minus_cut():
    # Eq.(17): E(X) = -cut(X) for every X
    n, m = 60, 300
    i, j, w = maxcut_graph(n, m, seed=4)
    W = maxcut_qubo(n, m, seed=4)
    X = random_solutions(50, n, 44)
    for x, bits in zip(X, unpack_bits(X, n)):
        cut = int(w[bits[i] != bits[j]].sum())
        assert oracle.energy(W, x) == -cut


def test_tsp_qubo_bruteforce_minimum_is_optimal_valid_tour():
    # Reading C13: min E over all 2^16 states of the c=4 instance is
    # 2*opt - 2*c*A and is attained by a valid tour of optimal length.
    c = 4
    for seed in (1, 2, 3):
        _, d = tsp_instance(c, seed)
        W = tsp_qubo(c, seed)
        A = 2 * int(d.max())
        e_min, xmin = oracle.bruteforce(W)
        opt = min(sum(d[p[t], p[(t + 1) % c]] for t in range(c)) for p in itertools.permutations(range(c)))
        assert e_min == 2 * opt - 2 * c * A
        M = unpack_bits(xmin, c * c)[0].reshape(c, c)   # row = city, column = order (Fig. 7)
        assert (M.sum(0) == 1).all() and (M.sum(1) == 1).all()
        tour = [int(np.nonzero(M[:, t])[0][0]) for t in range(c)]
        assert sum(d[tour[t], tour[(t + 1) % c]] for t in range(c)) == opt


def test_replay_matches_lockstep_search():
    n = 40
    W = random_qubo(n, 8)
    cfg = oracle.Config(n=n, searches=1, local_flips=25, pool_size=6, seed=2)
    R = 3
    full = oracle.run_lockstep(W, cfg, rounds=R)
    # reconstruct the targets that search 0 received by re-running the GA on
    # a pool evolved from the emitted results (the pool is host-only state).
    p = oracle.Pool(n, cfg.pool_size, seed=cfg.seed)
    T = []
    for r in range(R):
        T.append(p.target(cfg, r, 0))
        p.insert(full["B"][r, 0], full["EB"][r, 0])
    rep = oracle.replay_search(W, oracle.default_ladder(n)[0], cfg.local_flips, np.array(T))
    assert (rep["X"] == full["X"][0]).all() and rep["E"][0] == full["E"][0]
    assert rep["hash"][0] == full["hash"][0] and rep["flips"][0] == full["flips"][0]
    assert (rep["EB"] == full["EB"][:, 0]).all()


def test_counter_based_random_qubo_generator():
    """workloads.random_qubo_ctr (the host copy of abs_random_qubo_dev): every
    entry follows the stated Philox rule, checked with the ORACLE's Philox
    (pinned by the Random123 vectors) on a sample; symmetric; uniform moments
    (mean -1/2, sd 65536/sqrt(12)); the row-range form equals the full matrix."""
    from workloads import random_qubo_ctr, random_qubo_ctr_rows
    n, seed = 1500, (7 << 32) | 3
    W = random_qubo_ctr(n, seed)
    assert (W == W.T).all()
    rng = np.random.default_rng(0)
    for i, j in [(0, 0), (0, n - 1), (n - 1, n - 1)] + [tuple(sorted(v)) for v in rng.integers(0, n, (40, 2))]:
        o = oracle.philox4x32_10([i, j >> 3, 0x52514243, 0], [seed & 0xFFFFFFFF, seed >> 32])
        v = (int(o[(j >> 1) & 3]) >> (16 * (j & 1))) & 0xFFFF
        assert int(W[i, j]) == (v - 65536 if v >= 32768 else v)
    assert (random_qubo_ctr_rows(n, seed, 700, 710) == W[700:710]).all()
    big = random_qubo_ctr(4096, 1).astype(np.float64)
    assert abs(big.mean() + 0.5) < 60 and abs(big.std() - 65536 / 12 ** 0.5) < 60
