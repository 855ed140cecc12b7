"""GPU parity of the SA policy (Eq.(7), Alg. 1, reading
E2): lockstep trajectories of the CUDA path against oracle.run_lockstep with
the same Philox proposals and temperature ladder, bit for bit, across the
kernel variants (one warp with 32 or 64 bits per thread, three warps,
NT = 160), plus Max-Cut (constant ties) and the async mode's emitted energies."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
from workloads import maxcut_qubo, random_qubo

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icpp_yasudonitkyi20_b200 as pkg  # noqa: E402


def run_sa(W, S, L, R, tmin, tmax, K, pool=8, seed=7):
    n = W.shape[0]
    s = pkg.Solver(W, searches=S, local_flips=L, pool_size=pool, seed=seed, policy=pkg.POLICY_SA,
                   sa_tau_min=tmin, sa_tau_max=tmax, sa_levels=K)
    gB, gEB = [], []
    for _ in range(R):
        s.search(1)
        B, EB = s.round_results()
        gB.append(B)
        gEB.append(EB)
    cfg = oracle.Config(n=n, searches=S, local_flips=L, pool_size=pool, seed=seed, policy=1,
                        sa_tau_min=tmin, sa_tau_max=tmax, sa_levels=K)
    o = oracle.run_lockstep(W, cfg, R)
    return s, o, np.array(gB), np.array(gEB)


def check(s, o, gB, gEB, S, pool):
    assert (gEB == o["EB"]).all(), "E_B differs"
    assert (gB == o["B"]).all(), "B differs"
    for i in range(S):
        st = s.search_state(i)
        assert st["flips"] == o["flips"][i], ("flips", i)
        assert st["hash"] == int(o["hash"][i]), ("trajectory hash", i)
        assert st["E"] == o["E"][i], ("E", i)
        assert st["a"] == 0
        assert (st["X"] == o["X"][i]).all(), ("X", i)
        assert (st["D"].astype(np.int64) == o["D"][i]).all(), ("Delta", i)
    PX, PE = s.pool(pool)
    fin = o["poolE"] != oracle.EINF
    assert (PE == o["poolE"][fin]).all()
    assert (PX == o["poolX"][fin]).all()


@pytest.mark.parametrize("n,S,L,R,seed", [
    (100, 8, 600, 3, 1),     # one warp, 32 bits per thread
    (1100, 5, 800, 2, 2),    # one warp, 64 bits per thread
    (3000, 4, 900, 2, 3),    # three warps
    (4100, 3, 700, 2, 4),    # NT = 96 (runtime NT)
    (10000, 2, 500, 1, 6),   # NT = 160 (compile-time NT: the TSP 100-city size)
])
def test_sa_lockstep_bitexact(n, S, L, R, seed):
    W = random_qubo(n, seed)
    # a temperature ladder from nearly greedy to hot (parallel-tempering style)
    s, o, gB, gEB = run_sa(W, S, L, R, tmin=2000, tmax=400000, K=4, seed=seed)
    check(s, o, gB, gEB, S, 8)
    assert o["flips"].sum() > 0


def test_sa_n32768_bench_variant():
    """The kernel variant bench.py --policy sa times at n = 32768 (one
    512-thread CTA per search), 2 searches, reduced L: bit-exact."""
    n = 32768
    W = random_qubo(n, 1)
    s, o, gB, gEB = run_sa(W, 2, 400, 1, tmin=8000, tmax=262136, K=2, seed=1)
    check(s, o, gB, gEB, 2, 8)


def test_sa_maxcut_ties():
    n = 2000
    W = maxcut_qubo(n, 19990, seed=5)
    s, o, gB, gEB = run_sa(W, 4, 3000, 2, tmin=1, tmax=6, K=3, seed=5)
    check(s, o, gB, gEB, 4, 8)


def test_sa_cold_is_descent_and_hot_accepts_all():
    n = 300
    W = random_qubo(n, 9)
    # tau = 1: no uphill step with dE >= 33 is ever accepted (P = 0, reading E2)
    s, o, gB, gEB = run_sa(W, 3, 500, 1, tmin=1, tmax=1, K=1, seed=9)
    check(s, o, gB, gEB, 3, 8)
    # huge tau: every proposal is a flip
    s2, o2, gB2, gEB2 = run_sa(W, 3, 500, 1, tmin=2 ** 31 - 1, tmax=2 ** 31 - 1, K=1, seed=9)
    check(s2, o2, gB2, gEB2, 3, 8)


def test_sa_async_emits_true_energies():
    n = 777
    W = random_qubo(n, 10)
    s = pkg.Solver(W, searches=300, local_flips=400, pool_size=16, seed=3, policy=pkg.POLICY_SA,
                   sa_tau_min=5000, sa_tau_max=50000, sa_levels=5, mode=pkg.MODE_ASYNC)
    s.search(3)
    X, E = s.pool(16)
    assert len(E) > 0
    assert (s.energy(X) == E).all()
    s.close()


@pytest.mark.parametrize("n,kind,tmin,tmax", [
    (1, "random", 1, 1),             # a single bit; cold
    (3, "random", 50000, 400000),    # smaller than one byte-group; hot
    (64, "zeros", 1, 1),             # Delta = 0 everywhere: every proposal is accepted (d <= 0)
    (500, "extreme", 1, 1),          # +-32767/-32768 entries, tau = 1: only downhill moves
    (2048, "extreme", 2000, 2000000),  # one warp x 64 bits, n = n_pad exactly
])
def test_sa_degenerate_and_boundary(n, kind, tmin, tmax):
    rng = np.random.default_rng(90 + n)
    if kind == "zeros":
        W = np.zeros((n, n), np.int16)
    elif kind == "extreme":
        U = np.triu(np.where(rng.random((n, n)) < 0.5, np.int16(-32768), np.int16(32767)))
        W = (U + np.triu(U, 1).T).astype(np.int16)
    else:
        W = random_qubo(n, 91)
    S, L = 4, max(1, min(20 * n, 900))
    s, o, gB, gEB = run_sa(W, S, L, 3, tmin=tmin, tmax=tmax, K=2, seed=92)
    check(s, o, gB, gEB, S, 8)
    if kind == "zeros":
        # every proposal accepted: exactly L flips per search and round after the straight phase
        assert (o["flips"] >= 3 * L).all()


@pytest.mark.parametrize("n,S,L,steps", [
    (300, 6, 400, 4),      # one warp x 32 bits, CTAs own their search
    (1100, 300, 200, 2),   # one warp x 64 bits
    (3000, 4, 600, 3),     # multi-warp (three warps)
    (64, 6000, 60, 2),     # more searches than resident CTAs: the (search, round) queue
])
def test_sa_async_rounds_replay_bitexact(n, S, L, steps):
    """Async mode with the SA policy: given the targets each search actually
    used (trace), its trajectory is fixed by Eq.(7) and its Philox proposal
    stream (the counter persists across rounds).  The oracle replays it:
    every (B, E_B), the final state, flip count and trajectory hash identical."""
    W = random_qubo(n, 20 + n)
    tmin, tmax, K, seed = 3000, 300000, 3, 3
    s = pkg.Solver(W, searches=S, local_flips=L, pool_size=16, seed=seed, policy=pkg.POLICY_SA,
                   sa_tau_min=tmin, sa_tau_max=tmax, sa_levels=K, mode=pkg.MODE_ASYNC, trace=True)
    s.search(steps)
    tr = s.trace()
    assert len(tr) == S * steps
    by = {}
    for e in tr:
        by.setdefault(e[0], []).append(e)
    check = range(S) if S <= 16 else list(range(0, S, 997)) + [S - 1]
    for i in check:
        es = sorted(by.get(i, []), key=lambda e: e[1])
        assert [e[1] for e in es] == list(range(len(es)))
        if not es:
            continue
        rep = oracle.replay_search(W, 0, L, np.array([e[2] for e in es]), policy=1,
                                   tau=oracle.sa_tau_of(i, tmin, tmax, K), sid=i, seed=seed)
        assert (rep["EB"] == np.array([e[4] for e in es])).all(), ("E_B", i)
        assert all((rep["B"][r] == es[r][3]).all() for r in range(len(es))), ("B", i)
        st = s.search_state(i)
        assert st["hash"] == int(rep["hash"][0]) and st["flips"] == int(rep["flips"][0]), ("trajectory", i)
        assert st["E"] == int(rep["E"][0]) and (st["X"] == rep["X"]).all()
        assert (st["D"].astype(np.int64) == rep["D"]).all()
    s.close()
