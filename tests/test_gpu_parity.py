"""GPU parity: the CUDA path (libabs.so through its C ABI) against the CPU
oracle on the same seeded inputs.  Integer method -> bit-exact everywhere:
energies, Delta vectors, whole trajectories (FNV hash of the flip sequence,
flip counts, window offsets), every emitted (B, E_B), the GA targets and the
final pool."""
from __future__ import annotations

import itertools
import os
import sys
import time

import numpy as np
import pytest

import oracle
from workloads import maxcut_qubo, pack_bits, random_qubo, random_solutions, tsp_qubo

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icpp_yasudonitkyi20_b200 as abs_b200  # noqa: E402


def make(W, **kw):
    return abs_b200.Solver(W, **kw)


def ocfg(n, searches, L, pool, seed, ladder=None, mut_max=None):
    return oracle.Config(n=n, searches=searches, local_flips=L, pool_size=pool, seed=seed,
                         ladder=list(ladder or []), mut_max=mut_max)


def run_both(W, S, L, R, pool=16, seed=7, ladder=None, check_rounds=True):
    n = W.shape[0]
    s = make(W, searches=S, local_flips=L, pool_size=pool, seed=seed, ladder=ladder)
    gB, gEB, gT = [], [], []
    for _ in range(R):
        s.search(1)
        B, EB = s.round_results()
        gB.append(B)
        gEB.append(EB)
        gT.append(s.round_targets())
    o = oracle.run_lockstep(W, ocfg(n, S, L, pool, seed, ladder), R)
    return s, o, np.array(gB), np.array(gEB), np.array(gT)


def assert_same(s, o, gB, gEB, S, n, pool):
    # every emitted result, every round
    assert (gEB == o["EB"]).all(), "E_B differs"
    assert (gB == o["B"]).all(), "B differs"
    for i in range(S):
        st = s.search_state(i)
        assert st["flips"] == o["flips"][i], ("flips", i)
        assert st["hash"] == int(o["hash"][i]), ("trajectory hash", i)
        assert st["E"] == o["E"][i], ("E", i)
        assert st["a"] == o["a"][i], ("offset", i)
        assert (st["X"] == o["X"][i]).all(), ("X", i)
        assert (st["D"].astype(np.int64) == o["D"][i]).all(), ("Delta", i)
    PX, PE = s.pool(pool)
    fin = o["poolE"] != oracle.EINF
    assert (PE == o["poolE"][fin]).all()
    assert (PX == o["poolX"][fin]).all()


# ---------------------------------------------------------------- batched init
@pytest.mark.parametrize("n", [1, 16, 33, 100, 1000, 1024, 1500, 2050])
def test_batch_init_energy_and_delta(n):
    W = random_qubo(n, n)
    X = random_solutions(21, n, 5)            # spans two 16-solution tiles
    X[0] = 0
    X[1] = pack_bits(np.ones((1, n), bool))[0]  # all ones
    s = make(W, searches=1)
    Xdirty = X.copy()
    Xdirty[1] = np.iinfo(np.uint32).max       # bits >= n must be ignored
    E, D = s.energy(Xdirty, want_delta=True)
    oD, oE = oracle.init_batch(W, X)
    assert (E == oE).all()
    assert (D.astype(np.int64) == oD).all()


def test_batch_init_int32_extreme():
    # reading C12: W == -32768, X = 1^n -> Delta_i = 32768 (2n - 1), the largest |Delta|
    n = 4096
    W = np.full((n, n), -32768, np.int16)
    s = make(W, searches=1)
    X = np.full((1, n // 32), 0xFFFFFFFF, np.uint32)
    E, D = s.energy(X, want_delta=True)
    assert (D == 32768 * (2 * n - 1)).all()
    assert E[0] == -32768 * n * n


def test_zero_start_state():
    n = 1500
    W = random_qubo(n, 3)
    s = make(W, searches=3)
    for i in range(3):
        st = s.search_state(i)
        assert st["E"] == 0 and st["flips"] == 0 and st["a"] == 0
        assert (st["X"] == 0).all()
        assert (st["D"] == np.diag(W)).all()


def test_rejects_asymmetric_and_bad_n():
    W = random_qubo(40, 1)
    W[3, 5] += 1
    with pytest.raises(abs_b200.AbsError) as e:
        make(W, searches=1)
    assert e.value.rc == abs_b200.ABS_EINVAL
    with pytest.raises(abs_b200.AbsError):
        make(np.zeros((0, 0), np.int16), searches=1)


# ---------------------------------------------------------------- config 1 (n = 16)
def test_config1_n16_bitexact_and_bruteforce():
    n, S, L = 16, 256, 1000
    W = random_qubo(n, 1)
    s, o, gB, gEB, gT = run_both(W, S, L, 1, pool=32, seed=1)
    assert_same(s, o, gB, gEB, S, n, 32)
    allx = np.array(list(itertools.product([0, 1], repeat=n)), dtype=np.int64)
    e_min = int(np.einsum("bi,ij,bj->b", allx, W.astype(np.int64), allx).min())
    assert s.best()[1] == e_min


# ---------------------------------------------------------------- lockstep trajectories
@pytest.mark.parametrize("n,S,L,R,seed", [
    (5, 8, 30, 3, 1),          # tiny, ragged word
    (100, 12, 150, 3, 2),      # one warp, ragged
    (1024, 6, 1024, 2, 3),     # config-2 size, one warp, full
    (1100, 5, 300, 2, 4),      # one warp, 64 bits per thread (n_pad 2048), ragged
    (3000, 4, 500, 2, 5),      # 3 warps
    (4100, 3, 400, 2, 6),      # NT = 96 (runtime NT)
    (10000, 3, 300, 2, 7),     # NT = 160 (compile-time NT: the TSP 100-city size)
])
def test_lockstep_random_qubo_bitexact(n, S, L, R, seed):
    W = random_qubo(n, seed)
    s, o, gB, gEB, gT = run_both(W, S, L, R, pool=8, seed=seed)
    assert_same(s, o, gB, gEB, S, n, 8)


@pytest.mark.parametrize("n,extra,L,seed", [(40, 77, 24, 11), (1100, 33, 24, 12)])
def test_lockstep_split_step_full_state(n, extra, L, seed):
    """More one-warp searches than resident CTAs: a lockstep step is two launches (the
    first resident batch, then the rest on a second stream while the host builds their
    targets; DESIGN 5.7).  Every search's full state, every emitted result and the pool
    equal oracle.run_lockstep, so the split is the same round for every search."""
    S = abs_b200.device_searches(n) + extra
    W = random_qubo(n, seed)
    s, o, gB, gEB, gT = run_both(W, S, L, 2, pool=16, seed=seed)
    assert s.stats()["round_kernel_launches"] == 4  # two steps, two launches each
    assert_same(s, o, gB, gEB, S, n, 16)


def test_lockstep_maxcut_ties_bitexact():
    # Max-Cut (Eq.(17)) with +-1 weights: deltas tie constantly -> exercises
    # the lowest-index tie-break in every reduction (reading C5).
    n = 2000
    W = maxcut_qubo(n, 19990, seed=3)
    s, o, gB, gEB, gT = run_both(W, 4, 600, 3, pool=8, seed=3)
    assert_same(s, o, gB, gEB, 4, n, 8)


def test_lockstep_tsp_bitexact():
    c = 12
    W = tsp_qubo(c, seed=2)
    s, o, gB, gEB, gT = run_both(W, 6, 400, 3, pool=8, seed=2)
    assert_same(s, o, gB, gEB, 6, c * c, 8)


@pytest.mark.parametrize("ladder", [[1], [7], [64, 3], [100]])
def test_lockstep_window_edge_cases(ladder):
    # l = 1 (random-walk end), l not dividing n (wrap), l = n (greedy end)
    n = 100
    W = random_qubo(n, 11)
    s, o, gB, gEB, gT = run_both(W, 4, 250, 2, pool=8, seed=11, ladder=ladder)
    assert_same(s, o, gB, gEB, 4, n, 8)


def test_lockstep_single_local_flip():
    # L = 1: the round is almost only the straight search (Alg. 5)
    n = 300
    W = random_qubo(n, 12)
    s, o, gB, gEB, gT = run_both(W, 5, 1, 3, pool=8, seed=12)
    assert_same(s, o, gB, gEB, 5, n, 8)


def test_targets_match_oracle_ga():
    n = 200
    W = random_qubo(n, 13)
    s, o, gB, gEB, gT = run_both(W, 7, 50, 3, pool=6, seed=13)
    p = oracle.Pool(n, 6, seed=13)
    cfg = ocfg(n, 7, 50, 6, 13)
    for r in range(3):
        for i in range(7):
            assert (gT[r, i] == p.target(cfg, r, i)).all()
        for i in range(7):
            p.insert(o["B"][r, i], o["EB"][r, i])


def test_emitted_energies_are_true_energies():
    n = 777
    W = random_qubo(n, 14)
    s = make(W, searches=9, local_flips=500, pool_size=8, seed=14)
    s.search(2)
    B, EB = s.round_results()
    E = s.energy(B)
    assert (E == EB).all()
    for b in range(3):
        assert oracle.energy(W, B[b]) == EB[b]


def test_external_merge_equals_internal():
    n = 500
    W = random_qubo(n, 15)
    a = make(W, searches=6, local_flips=200, pool_size=8, seed=15)
    b = make(W, searches=6, local_flips=200, pool_size=8, seed=15, external_merge=True)
    for _ in range(3):
        a.search(1)
        b.search(1)
        B, EB = b.round_results()
        b.pool_insert(B, EB)
    assert (a.pool(8)[1] == b.pool(8)[1]).all()
    assert (a.pool(8)[0] == b.pool(8)[0]).all()


def test_sharded_ranks_equal_single_process():
    """P14 / SURVEY §8(e): 3 'ranks' (contexts with search_offset) exchanging
    all results each step reproduce the single-process oracle exactly."""
    n, Sg, R, L = 300, 4, 3, 120
    W = random_qubo(n, 16)
    ranks = [make(W, searches=Sg, search_offset=r * Sg, local_flips=L, pool_size=8, seed=16, external_merge=True)
             for r in range(3)]
    for _ in range(R):
        res = []
        for s in ranks:
            s.search(1)
            res.append(s.round_results())
        allB = np.concatenate([b for b, _ in res])
        allE = np.concatenate([e for _, e in res])
        for s in ranks:
            s.pool_insert(allB, allE)
    o = oracle.run_lockstep(W, ocfg(n, 3 * Sg, L, 8, 16), R)
    for s in ranks:
        PX, PE = s.pool(8)
        assert (PE == o["poolE"]).all() and (PX == o["poolX"]).all()
    for r, s in enumerate(ranks):
        for i in range(Sg):
            assert s.search_state(i)["hash"] == int(o["hash"][r * Sg + i])


def test_seed_pool_uses_device_energies():
    n = 250
    W = random_qubo(n, 17)
    s = make(W, searches=2, pool_size=4, seed=17)
    X = random_solutions(6, n, 17)
    s.seed_pool(X)
    PX, PE = s.pool(4)
    E_ref = np.array([oracle.energy(W, x) for x in X])
    order = np.argsort(E_ref, kind="stable")[:4]
    assert (PE == E_ref[order]).all()


# ---------------------------------------------------------------- full size (bench launch configuration)
def test_full_size_n32768_sampled():
    """n = 32768 (config 5), the kernel variant bench.py times (one 512-thread
    CTA per search, 64 bits per thread), on 2 searches with a reduced L:
    trajectory hash, Delta, E, B, E_B identical to the oracle."""
    n, S, L = 32768, 2, 64
    W = random_qubo(n, 1)
    t0 = time.time()
    s = make(W, searches=S, local_flips=L, pool_size=4, seed=5)
    s.search(1)
    B, EB = s.round_results()
    o = oracle.run_lockstep(W, ocfg(n, S, L, 4, 5), 1)
    assert (EB == o["EB"][0]).all() and (B == o["B"][0]).all()
    for i in range(S):
        st = s.search_state(i)
        assert st["hash"] == int(o["hash"][i]) and st["flips"] == o["flips"][i]
        assert st["E"] == o["E"][i]
        assert (st["D"].astype(np.int64) == o["D"][i]).all()
    assert time.time() - t0 < 600


@pytest.mark.parametrize("workload", ["random32k", "tsp100", "maxcut2k", "random1k"])
def test_bench_configuration_sampled(workload):
    """The exact step bench.py times by default for each workload: its W, seed,
    pool, searches (WAVES x co-resident CTAs, or config 2's 10,000) and L = n,
    one lockstep step.  Three sampled searches are re-run by the oracle from
    the oracle's own round-0 targets (host GA): E_B, B, final E,
    Delta, flip count and trajectory hash identical."""
    import threading

    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench

    W = bench.make_W(workload)                 # host copy (oracle)
    n = W.shape[0]
    S = bench.default_searches(workload, n, 0)
    s = make(bench.make_W_device(workload, 0), searches=S, local_flips=n, pool_size=64, seed=1)  # as bench.py
    s.search(1)
    B, EB = s.round_results()
    cfg = ocfg(n, S, n, 64, 1)
    pool = oracle.Pool(n, 64, 1)
    lad = oracle.default_ladder(n)
    sids = [0, S // 2 + 1, S - 1]
    reps = {}

    def replay(sid):
        reps[sid] = oracle.replay_search(W, lad[sid % len(lad)], n, pool.target(cfg, 0, sid))

    th = [threading.Thread(target=replay, args=(sid,)) for sid in sids]
    for x in th:
        x.start()
    for x in th:
        x.join()
    for sid in sids:
        rep, st = reps[sid], s.search_state(sid)
        assert EB[sid] == rep["EB"][0] and (B[sid] == rep["B"][0]).all()
        assert st["hash"] == int(rep["hash"][0]) and st["flips"] == int(rep["flips"][0])
        assert st["E"] == int(rep["E"][0]) and (st["X"] == rep["X"]).all()
        assert (st["D"].astype(np.int64) == rep["D"]).all()
    assert s.stats()["flips"] >= S * n


# ---------------------------------------------------------------- asynchronous mode (paper Fig. 5)
def _replay_async(W, s, L, trace_s, l):
    """Replay one search of an async run with the targets it actually used."""
    T = np.array([e[2] for e in trace_s])
    return oracle.replay_search(W, l, L, T)


@pytest.mark.parametrize("n,S,L,steps", [(300, 6, 120, 5), (1500, 4, 300, 3), (64, 6000, 40, 2),
                                         (3000, 5, 900, 3),      # multi-warp (three warps): the hot loop
                                         (10000, 3, 2000, 2),    # NT = 160
                                         (32768, 2, 3000, 2)])   # NT = 512, two half-row copies
def test_async_rounds_replay_bitexact(n, S, L, steps):
    """Async mode: timing decides which target each round gets, but given the
    targets a search actually used (trace), its trajectory is determined: the
    oracle replay must match every (B, E_B), the final state and the hash."""
    W = random_qubo(n, 40 + n)
    s = make(W, searches=S, local_flips=L, pool_size=16, seed=3, mode=abs_b200.MODE_ASYNC, trace=True)
    s.search(steps)
    tr = s.trace()
    assert len(tr) == S * steps          # rounds per search may differ (searches run freely)
    by = {}
    for e in tr:
        by.setdefault(e[0], []).append(e)
    lad = oracle.default_ladder(n)
    check = range(S) if S <= 16 else list(range(0, S, 997)) + [S - 1]
    for i in check:
        es = sorted(by.get(i, []), key=lambda e: e[1])
        nr = len(es)
        assert [e[1] for e in es] == list(range(nr))
        if nr == 0:
            continue
        rep = _replay_async(W, i, L, es, lad[i % len(lad)])
        assert (rep["EB"] == np.array([e[4] for e in es])).all()
        assert all((rep["B"][r] == es[r][3]).all() for r in range(nr))
        st = s.search_state(i)
        assert st["hash"] == int(rep["hash"][0]) and st["flips"] == int(rep["flips"][0])
        assert st["E"] == int(rep["E"][0]) and (st["X"] == rep["X"]).all()
        assert (st["D"].astype(np.int64) == rep["D"]).all()
    PX, PE = s.pool(16)
    assert (np.diff(PE) > 0).all()
    assert (s.energy(PX) == PE).all()
    assert PE[0] == min(e[4] for e in tr)
    st = s.stats()
    assert st["rounds"] == S * steps


def test_async_second_call_continues():
    n, S, L = 200, 5, 80
    W = random_qubo(n, 77)
    s = make(W, searches=S, local_flips=L, pool_size=8, seed=4, mode=abs_b200.MODE_ASYNC, trace=True)
    s.search(2)
    s.search(3)
    tr = s.trace()
    assert len(tr) == S * 5
    lad = oracle.default_ladder(n)
    for i in range(S):
        es = sorted([e for e in tr if e[0] == i], key=lambda e: e[1])
        assert [e[1] for e in es] == list(range(len(es)))
        if not es:
            continue
        rep = _replay_async(W, i, L, es, lad[i % len(lad)])
        assert s.search_state(i)["hash"] == int(rep["hash"][0])


@pytest.mark.parametrize("n,ladder", [(2000, [256]), (5000, [256, 200]), (10000, [256, 97]), (33, [8])])
def test_lockstep_large_windows_few_warps(n, ladder):
    # the window selection is split over min(4, warps) warps; l up to 256
    W = random_qubo(n, 50)
    s, o, gB, gEB, gT = run_both(W, 3, 300, 2, pool=8, seed=50, ladder=ladder)
    assert_same(s, o, gB, gEB, 3, n, 8)


@pytest.mark.parametrize("L", [1, 2, 3, 4, 5])
def test_lockstep_short_local_phases(L):
    # lookahead pipeline edges: rows / slices issued only for flips that happen
    n = 3000
    W = random_qubo(n, 60 + L)
    s, o, gB, gEB, gT = run_both(W, 4, L, 3, pool=8, seed=60 + L, ladder=[64, 256])
    assert_same(s, o, gB, gEB, 4, n, 8)


def _degenerate_w(kind, n):
    if kind == "zeros":        # every Delta is 0: every argmin is a full tie
        return np.zeros((n, n), np.int16)
    if kind == "minus_one":    # constant W = -1: ties in every window, E strictly falls
        return np.full((n, n), -1, np.int16)
    if kind == "diag_only":    # separable: the optimum sets exactly the negative diagonal bits
        W = np.zeros((n, n), np.int16)
        d = random_qubo(n, 71).diagonal()
        W[np.arange(n), np.arange(n)] = d
        return W
    if kind == "extreme":      # +-32767/-32768 entries: the widest Delta range (reading C12)
        rng = np.random.default_rng(72)
        U = np.where(rng.random((n, n)) < 0.5, np.int16(-32768), np.int16(32767))
        U = np.triu(U)
        return (U + np.triu(U, 1).T).astype(np.int16)
    return random_qubo(n, 73)


@pytest.mark.parametrize("n,kind", [
    (1, "random"), (2, "random"), (3, "minus_one"),   # smaller than one byte-group
    (64, "zeros"), (200, "minus_one"), (500, "diag_only"),
    (2048, "extreme"),      # one warp x 64 bits, n = n_pad exactly (no ragged tail)
    (3072, "random"),       # 32 bits x 96 threads, n = n_pad exactly
])
def test_lockstep_degenerate_and_boundary(n, kind):
    # degenerate instances (all ties, separable, extreme weights) and sizes at the
    # edges of the kernel variants; trajectories, pool and every (B, E_B) bit-exact
    W = _degenerate_w(kind, n)
    S, L = 6, max(1, min(3 * n, 700))
    s, o, gB, gEB, gT = run_both(W, S, L, 3, pool=8, seed=74)
    assert_same(s, o, gB, gEB, S, n, 8)
    if kind == "diag_only":
        assert s.best()[1] == int(np.minimum(W.diagonal().astype(np.int64), 0).sum())
    if kind == "zeros":
        assert s.best()[1] == 0


# ---------------------------------------------------------------- multi-warp kernels at the ladder extremes
@pytest.mark.parametrize("n", [3000, 10000, 32768])
def test_lockstep_multiwarp_ladder_extremes(n):
    """Multi-warp kernels (n > 2048) with window lengths at both ends of
    P:L305 (l = 1 ... l = n): l in {1, 2, 3} runs the window-first prefetch
    path with windows shorter than a byte-group, l in {300, n/2+1, n} the
    non-prefetch local branch (l > kWinMax = 256; for l > n/2 consecutive
    windows overlap, l = n is steepest forced greedy).  Full state and every
    (B, E_B) identical to oracle.run_lockstep."""
    ladder = [1, 2, 3, 300, n // 2 + 1, n]
    W = random_qubo(n, 80 + n % 97)
    S, L, R = 6, 400, 2
    s, o, gB, gEB, gT = run_both(W, S, L, R, pool=8, seed=81, ladder=ladder)
    assert_same(s, o, gB, gEB, S, n, 8)


def test_full_size_bench_three_rounds_replay():
    """bench.py's default step (random n = 32768, 592 searches, L = n, seed 1)
    for THREE lockstep steps.  (1) The host GA at full size: the targets of
    rounds 1 and 2 equal oracle GA targets drawn from a pool rebuilt with
    oracle.Pool from every result the device emitted.
    (2) Three sampled searches are replayed by the oracle from the targets the
    device used: every round's (B, E_B) and the final state identical."""
    import threading

    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import bench

    W = bench.make_W("random32k")              # host copy (oracle)
    n = W.shape[0]
    S = bench.default_searches("random32k", n, 0)
    s = make(bench.make_W_device("random32k", 0), searches=S, local_flips=n, pool_size=64, seed=1)
    Ts, Bs, EBs = [], [], []
    for _ in range(3):
        s.search(1)
        Ts.append(s.round_targets())
        B, EB = s.round_results()
        Bs.append(B)
        EBs.append(EB)
    cfg = ocfg(n, S, n, 64, 1)
    pool = oracle.Pool(n, 64, 1)
    for r in range(3):
        for sid in [0, 1, S // 3, S - 1]:
            assert (Ts[r][sid] == pool.target(cfg, r, sid)).all(), ("GA target", r, sid)
        for sid in range(S):
            pool.insert(Bs[r][sid], EBs[r][sid])
    PX, PE = s.pool(64)
    fin = pool.E != oracle.EINF
    assert (PE == pool.E[fin]).all() and (PX == pool.X[fin]).all()

    lad = oracle.default_ladder(n)
    sids = [0, S // 2 + 1, S - 1]
    reps = {}

    def replay(sid):
        reps[sid] = oracle.replay_search(W, lad[sid % len(lad)], n, np.stack([Ts[r][sid] for r in range(3)]))

    th = [threading.Thread(target=replay, args=(sid,)) for sid in sids]
    for x in th:
        x.start()
    for x in th:
        x.join()
    for sid in sids:
        rep, st = reps[sid], s.search_state(sid)
        for r in range(3):
            assert EBs[r][sid] == rep["EB"][r] and (Bs[r][sid] == rep["B"][r]).all(), ("round", r, sid)
        assert st["hash"] == int(rep["hash"][0]) and st["flips"] == int(rep["flips"][0])
        assert st["E"] == int(rep["E"][0]) and (st["X"] == rep["X"]).all()
        assert (st["D"].astype(np.int64) == rep["D"]).all()


# ---------------------------------------------------------------- synthetic instance on the device (a1)
@pytest.mark.parametrize("n", [1, 7, 8, 63, 64, 65, 1000, 4097])
def test_random_qubo_dev_equals_host_generator(n):
    from workloads import random_qubo_ctr
    Wd = torch.empty((n, n), dtype=torch.int16, device="cuda:0")
    abs_b200.random_qubo_dev(Wd, 77)
    assert (Wd.cpu().numpy() == random_qubo_ctr(n, 77)).all()


def test_random_qubo_dev_full_size_rows():
    from workloads import random_qubo_ctr_rows
    n = 32768
    Wd = torch.empty((n, n), dtype=torch.int16, device="cuda:0")
    abs_b200.random_qubo_dev(Wd, 1)
    for r0 in (0, 4093, 16000, 32765):
        assert (Wd[r0:r0 + 3].cpu().numpy() == random_qubo_ctr_rows(n, 1, r0, r0 + 3)).all(), r0
    # symmetric (columns = rows) on a sample
    for c in (0, 12345, 32767):
        assert (Wd[:, c].cpu() == Wd[c].cpu()).all()
