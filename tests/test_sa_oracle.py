"""Pins of the oracle's SA policy (Eq.(7) P:L116-122,
Alg. 1, reading E2 in DESIGN.md).  None retypes the oracle's
formulas: the threshold is held against math.exp2 (within one Q32 unit),
its exact integer points, and the exact floor decided in integer arithmetic
(P^tau 2^dE <= 2^(32 tau) < (P+1)^tau 2^dE; nested isqrt for tau = 2^k);
the policy against limits whose outcome is fixed (every move
accepted / no uphill move) and against the acceptance rate a binomial
experiment must show."""
from __future__ import annotations

import math

import numpy as np
import pytest

import oracle
from workloads import random_qubo


@pytest.mark.parametrize("tau", [1, 7, 1000, 2 ** 20, 2 ** 31 - 1])
def test_threshold_integer_points_and_monotone(tau):
    # at dE = q*tau, p = 2^-q exactly: 2^(32-q); below one unit (q >= 33) it is 0
    for q in range(0, 40):
        dE = q * tau
        if dE > 2 ** 40:
            break
        want = 2 ** (32 - q) if q <= 32 else 0
        assert oracle.sa_threshold(dE, tau) == want
    # monotone non-increasing in dE
    rng = np.random.default_rng(tau % 1000)
    prev = None
    for dE in sorted(int(v) for v in rng.integers(1, min(40 * tau, 2 ** 40), 400)):
        P = oracle.sa_threshold(dE, tau)
        if prev is not None:
            assert P <= prev
        prev = P


def _cases(seed, count):
    rng = np.random.default_rng(seed)
    out = []
    for _ in range(count):
        tau = int(rng.choice([rng.integers(1, 50), rng.integers(1, 70000), rng.integers(1, 2 ** 31 - 1)]))
        dE = int(rng.integers(1, min(2 ** 31 - 1, 34 * tau) + 1))
        out.append((dE, tau))
    return out + [(1, 2 ** 31 - 1), (2 ** 31 - 1, 2 ** 31 - 1), (2 ** 31 - 2, 2 ** 31 - 1), (2 ** 31 - 1, 1),
                  (1, 1), (31, 1), (32, 1), (33, 1), (65, 2)]


def test_threshold_within_one_unit_of_exp2():
    # Eq.(7) with k_B t = tau / ln 2: P must be 2^32 * 2^(-dE/tau) to within one Q32 unit
    for dE, tau in _cases(1, 20000):
        q, r = divmod(dE, tau)
        v = math.ldexp(math.exp2(-r / tau), 32 - q)   # 2^(32-q) * 2^(-r/tau), double precision
        P = oracle.sa_threshold(dE, tau)
        assert abs(P - v) < 1.0 + 1e-6 * max(v, 1.0) * 2 ** -20, (dE, tau, P, v)
        if abs(v - round(v)) > 1e-4:                  # away from an integer, P is the floor
            assert P == math.floor(v), (dE, tau, P, v)


def test_threshold_is_exact_floor_small_tau():
    # P = floor(2^32 2^(-dE/tau))  <=>  P^tau 2^dE <= 2^(32 tau) < (P+1)^tau 2^dE,
    # decided in exact integer arithmetic (no floating point, no logarithm)
    rng = np.random.default_rng(5)
    for tau in list(range(1, 41)) + [int(v) for v in rng.integers(41, 300, 20)]:
        for dE in sorted({1, 2, tau - 1, tau, tau + 1, 32 * tau - 1, 33 * tau - 1}
                         | {int(v) for v in rng.integers(1, 33 * tau, 25)}):
            if dE < 1:
                continue
            P = oracle.sa_threshold(dE, tau)
            assert P ** tau * 2 ** dE <= 2 ** (32 * tau) < (P + 1) ** tau * 2 ** dE, (dE, tau, P)


@pytest.mark.parametrize("k", [1, 2, 5, 10, 16])
def test_threshold_is_exact_floor_power_of_two_tau(k):
    # tau = 2^k: floor(2^(32 - dE/2^k)) = floor((2^(32*2^k - dE))^(1/2^k)) = k nested
    # integer square roots (floor(sqrt(floor(sqrt(N)))) = floor(N^(1/4)), exactly)
    tau = 2 ** k
    for dE in [1, 3, tau - 1, tau + 1, 5 * tau + 7, 31 * tau + 1]:
        v = 2 ** (32 * tau - dE)
        for _ in range(k):
            v = math.isqrt(v)
        assert oracle.sa_threshold(dE, tau) == v, (dE, tau)


def test_hot_limit_accepts_every_proposal():
    n = 40
    rng = np.random.default_rng(1)
    A = rng.integers(-10, 11, (n, n)).astype(np.int16)
    W = np.triu(A) + np.triu(A, 1).T            # |dE| <= 10 (2n-1) < 800
    s = oracle.Search(W)
    s.set_sa(tau=2 ** 30, sid=5, seed=9)
    s.local_sa(3000)
    assert s.flips == 3000 and s.sa_ctr == 3000  # rejection odds per move < 4e-7


def test_cold_limit_never_goes_uphill():
    n = 60
    W = (random_qubo(n, 2).astype(np.int32) // 1024 * 64).astype(np.int16)  # every dE is a multiple of 64
    s = oracle.Search(W)
    s.set_sa(tau=1, sid=0, seed=3)                # uphill dE >= 64 -> q >= 32 -> P = 0
    E = s.E
    for _ in range(4000):
        s.local_sa(1)
        assert s.E <= E
        E = s.E
    assert s.flips > 0


def test_uphill_acceptance_rate_matches_threshold():
    # diagonal W = D: proposing an unset bit is uphill by D, a set bit downhill by D
    n, D, tau, L = 64, 1000, 700, 40000
    W = np.diag(np.full(n, D)).astype(np.int16)
    s = oracle.Search(W)
    s.set_sa(tau=tau, sid=11, seed=17)
    up = down = 0
    E = s.E
    for _ in range(L):
        s.local_sa(1)
        if s.E > E:
            up += 1
        elif s.E < E:
            down += 1
        E = s.E
    proposals_up = L - down                       # set-bit proposals are always accepted
    p = math.exp2(-D / tau)                       # Eq.(7) with k_B t = tau / ln 2
    sigma = math.sqrt(p * (1 - p) / proposals_up)
    assert abs(up / proposals_up - p) < 5 * sigma


def test_counter_persists_across_calls():
    W = random_qubo(80, 4)
    a, b = oracle.Search(W), oracle.Search(W)
    a.set_sa(tau=5000, sid=2, seed=6)
    b.set_sa(tau=5000, sid=2, seed=6)
    a.local_sa(700)
    b.local_sa(300)
    b.local_sa(400)
    assert a.sa_ctr == b.sa_ctr == 700
    assert a.E == b.E and a.hash == b.hash and (a.x == b.x).all() and (a.d == b.d).all()


def test_replay_search_sa_equals_lockstep_run():
    """oracle.replay_search with the SA policy (the async-parity reference)
    re-runs one search of oracle.run_lockstep exactly, given the targets that
    search received: same temperature (reading E2 ladder), same Philox stream
    (global search id), the proposal counter persisting across rounds."""
    n, S, L, R, seed = 120, 5, 300, 3, 21
    tmin, tmax, K = 2000, 90000, 3
    W = random_qubo(n, 22)
    cfg = oracle.Config(n=n, searches=S, local_flips=L, pool_size=8, seed=seed, policy=1,
                        sa_tau_min=tmin, sa_tau_max=tmax, sa_levels=K)
    o = oracle.run_lockstep(W, cfg, R)
    # the targets of rounds 0..R-1: rebuild the pool exactly as run_lockstep does
    pool = oracle.Pool(n, 8, seed)
    T = np.zeros((R, S, (n + 31) // 32), np.uint32)
    for r in range(R):
        for s in range(S):
            T[r, s] = pool.target(cfg, r, s)
        for s in range(S):
            pool.insert(o["B"][r, s], o["EB"][r, s])
    for s in range(S):
        rep = oracle.replay_search(W, 0, L, T[:, s], policy=1, tau=oracle.sa_tau_of(s, tmin, tmax, K),
                                   sid=s, seed=seed)
        assert (rep["EB"] == o["EB"][:, s]).all() and (rep["B"] == o["B"][:, s]).all()
        assert int(rep["hash"][0]) == int(o["hash"][s]) and int(rep["flips"][0]) == int(o["flips"][s])
        assert (rep["D"] == o["D"][s]).all() and int(rep["E"][0]) == int(o["E"][s])
