"""Ising front end.

The oracle's Ising energy (definition) is pinned to physics facts that
do not retype its formula: the all-aligned ferromagnet's ground-state energy
(closed form, which also fixes the pairs-once reading E1), a single spin in a
field, spin-flip symmetry at h = 0, and the anti-aligned ground state of an
antiferromagnetic pair.  The library conversions (host-only C ABI calls, no
GPU) are then checked against the oracle by brute force over all 2^n states."""
from __future__ import annotations

import itertools

import numpy as np
import pytest

import oracle
import paper_conf_icpp_yasudonitkyi20_b200 as pkg
from paper_conf_icpp_yasudonitkyi20_b200 import AbsError


def _spins(n):
    return [np.array(c, np.int8) for c in itertools.product([-1, 1], repeat=n)]


def _bits(s):
    x = (np.asarray(s) > 0).astype(np.uint8)  # s = 2x - 1
    w = np.zeros((len(x) + 31) // 32, np.uint32)
    for i, b in enumerate(x):
        if b:
            w[i >> 5] |= np.uint32(1 << (i & 31))
    return w


# ---------------------------------------------------------------- oracle pins
@pytest.mark.parametrize("n", [2, 3, 5, 8])
def test_ferromagnet_ground_state_closed_form(n):
    # J_ij = 1 on every pair, h = 0: ground states all-up / all-down with
    # H = -n(n-1)/2 (each pair counted once, reading E1)
    J = np.ones((n, n), np.int32)
    h = np.zeros(n, np.int32)
    Hs = {tuple(s): oracle.ising_energy(J, h, s) for s in _spins(n)}
    gmin = min(Hs.values())
    assert gmin == -n * (n - 1) // 2
    assert {k for k, v in Hs.items() if v == gmin} == {tuple([1] * n), tuple([-1] * n)}


def test_single_spin_in_field():
    J = np.zeros((1, 1), np.int32)
    for hv in (-7, 0, 5):
        h = np.array([hv], np.int32)
        assert oracle.ising_energy(J, h, np.array([1], np.int8)) == -hv  # aligned with the field: -h
        assert oracle.ising_energy(J, h, np.array([-1], np.int8)) == hv


def test_spin_flip_symmetry_without_field():
    rng = np.random.default_rng(3)
    n = 7
    J = rng.integers(-50, 50, (n, n)).astype(np.int32)
    h = np.zeros(n, np.int32)
    for s in _spins(n):
        assert oracle.ising_energy(J, h, s) == oracle.ising_energy(J, h, -s)


def test_antiferromagnetic_pair():
    J = np.array([[0, -3], [0, 0]], np.int32)  # only i<j is read
    h = np.zeros(2, np.int32)
    H = {tuple(s): oracle.ising_energy(J, h, s) for s in _spins(2)}
    assert H[(1, -1)] == H[(-1, 1)] == -3
    assert H[(1, 1)] == H[(-1, -1)] == 3


# ---------------------------------------------------------------- library conversions
@pytest.mark.parametrize("n,seed", [(1, 1), (2, 2), (5, 3), (9, 4)])
def test_ising_to_qubo_brute_force(n, seed):
    rng = np.random.default_rng(seed)
    J = rng.integers(-4000, 4000, (n, n)).astype(np.int32)
    h = rng.integers(-4000, 4000, n).astype(np.int32)
    W, off = pkg.ising_to_qubo(J, h)
    assert (W == W.T).all()
    for s in _spins(n):
        assert oracle.ising_energy(J, h, s) == oracle.energy(W, _bits(s)) + off


@pytest.mark.parametrize("n,seed", [(1, 5), (4, 6), (8, 7)])
def test_qubo_to_ising_brute_force(n, seed):
    rng = np.random.default_rng(seed)
    A = rng.integers(-32768, 32768, (n, n)).astype(np.int16)
    W = np.triu(A) + np.triu(A, 1).T
    J2, h2, off2 = pkg.qubo_to_ising(W)
    assert (np.diag(J2) == 0).all() and (J2 == J2.T).all()
    for s in _spins(n):
        # H is linear in (J, h): the energy of (2J, 2h) is 2H = 2E(X) + 2*offset
        assert oracle.ising_energy(J2, h2, s) == 2 * oracle.energy(W, _bits(s)) + off2


def test_round_trip():
    rng = np.random.default_rng(8)
    n = 12
    J = np.triu(rng.integers(-1000, 1000, (n, n)), 1).astype(np.int32)
    h = rng.integers(-1000, 1000, n).astype(np.int32)
    W, off = pkg.ising_to_qubo(J, h)
    J2, h2, off2 = pkg.qubo_to_ising(W)
    assert (J2 == 2 * (J + J.T)).all()
    assert (h2 == 2 * h).all()
    assert off2 == 2 * off


def test_maxcut_is_an_ising_model():
    # Max-Cut as the antiferromagnet J = -w (Eq.(17) in Ising form):
    # H(S) = sum_{i<j} w_ij s_i s_j = (total weight) - 2 cut(S)
    from workloads import maxcut_graph
    n = 9
    ei, ej, w = maxcut_graph(n, 14, seed=2)
    J = np.zeros((n, n), np.int32)
    J[ei, ej] = -w
    h = np.zeros(n, np.int32)
    W, off = pkg.ising_to_qubo(J, h)
    for s in _spins(n):
        cut = sum(int(wt) for u, v, wt in zip(ei, ej, w) if s[u] != s[v])
        assert oracle.energy(W, _bits(s)) + off == int(np.sum(w)) - 2 * cut


def test_out_of_range_rejected():
    J = np.array([[0, 20000], [0, 0]], np.int32)  # W_01 = -40000
    with pytest.raises(AbsError):
        pkg.ising_to_qubo(J, np.zeros(2, np.int32))
    with pytest.raises(AbsError):
        pkg.qubo_to_ising(np.array([[0, 1], [2, 0]], np.int16))  # not symmetric
