"""Pins of the oracle's SA policy (Eq.(7) P:L116-122,
Alg. 1, reading E2 in DESIGN.md).  None retypes the oracle's
formulas: the threshold is held against math.exp2 and its exact integer
points; the policy against limits whose outcome is fixed (every move
accepted / no uphill move) and against the acceptance rate a binomial
experiment must show."""
from __future__ import annotations

import math

import numpy as np
import pytest

import oracle
from workloads import random_qubo


@pytest.mark.parametrize("tau", [1, 7, 1000, 2 ** 20, 2 ** 31 - 1])
def test_threshold_integer_points_and_bounds(tau):
    # at dE = q*tau the interpolation is exact: 2^(32-q); beyond 31 halvings it is 0
    for q in range(0, 34):
        dE = q * tau
        if dE > 2 ** 40:
            break
        want = 2 ** (32 - q) if q < 32 else 0
        assert oracle.sa_threshold(dE, tau) == want
    # monotone non-increasing, and within the linear-interpolation error of 2^-x
    rng = np.random.default_rng(tau % 1000)
    prev = None
    for dE in sorted(int(v) for v in rng.integers(1, min(40 * tau, 2 ** 40), 400)):
        P = oracle.sa_threshold(dE, tau)
        if prev is not None:
            assert P <= prev
        prev = P
        exact = math.exp2(-dE / tau)
        if exact > 2.0 ** -31:
            assert abs(P / 2 ** 32 - exact) <= 0.0616 * exact + 2.0 ** -32


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
    p = oracle.sa_threshold(D, tau) / 2 ** 32
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
