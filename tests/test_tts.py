"""Time-to-solution harness (paper_conf_icpp_yasudonitkyi20_b200/tts.py;
Table 1).  CPU: the loop logic with a scripted solver and clock,
the target arithmetic, the problem decoders against oracle energies, and the
2-rank agreement over gloo.  GPU: the real solver reaches the brute-force
optimum of a config-1 sized instance."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

import oracle
from paper_conf_icpp_yasudonitkyi20_b200 import AbsError, tts
from paper_conf_icpp_yasudonitkyi20_b200.abs import ABS_EEMPTY
from workloads import maxcut_graph, maxcut_qubo, random_qubo, tsp_instance, tsp_qubo

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as tmp  # noqa: E402


class ScriptedSolver:
    """best() follows a fixed list of energies, one entry per search() call
    (None = empty pool)."""

    def __init__(self, energies):
        self.energies = list(energies)
        self.i = -1
        self.words = 1
        self.calls = []

    def search(self, steps):
        self.calls.append(steps)
        self.i += 1

    def best(self):
        E = self.energies[min(self.i, len(self.energies) - 1)]
        if E is None:
            raise AbsError(ABS_EEMPTY, "abs_best", "empty")
        return np.array([self.i], np.uint32), E

    def pool(self, k):
        X, E = self.best()
        return X[None, :], np.array([E], np.int64)

    def pool_insert(self, X, E):
        return 0


class Clock:
    def __init__(self, dt):
        self.t = 0.0
        self.dt = dt

    def __call__(self):
        v = self.t
        self.t += self.dt
        return v


def test_reaches_target_and_traces_improvements():
    s = ScriptedSolver([None, -5, -5, -9, -12, -20])
    r = tts.time_to_target(s, target_energy=-12, max_seconds=100, rounds_per_call=3, clock=Clock(0.5))
    assert r.reached and r.calls == 5 and s.calls == [3] * 5
    assert r.seconds == pytest.approx(2.5)  # clock read once at start, once per call
    assert [e for _, e in r.trace] == [-5, -9, -12]
    assert r.best_energy == -12


def test_times_out():
    s = ScriptedSolver([-1, -2, -3])
    r = tts.time_to_target(s, target_energy=-100, max_seconds=2.0, clock=Clock(0.5))
    assert not r.reached and r.seconds is None and r.calls == 4 and r.best_energy == -3


def test_accept_predicate():
    s = ScriptedSolver([-5, -6, -7])
    r = tts.time_to_target(s, accept=lambda X, E: int(X[0]) == 1, max_seconds=10, clock=Clock(1.0))
    assert r.reached and r.calls == 2


def test_targets():
    assert tts.energy_target(-1000, 0.99) == -990
    assert tts.energy_target(-1001, 0.99) == -991      # E <= -990.99
    assert tts.energy_target(-33115098990, 0.99) == -32783948001
    assert tts.cut_target(13225, 0.99) == -13093       # cut >= 13092.75
    assert tts.cut_target(100, 1) == -100


def test_cut_value_matches_qubo_energy():
    n = 60
    ei, ej, w = maxcut_graph(n, 400, seed=4)
    W = maxcut_qubo(n, 400, seed=4)
    rng = np.random.default_rng(1)
    for _ in range(20):
        X = rng.integers(0, 2 ** 32, (n + 31) // 32, dtype=np.uint64).astype(np.uint32)
        X[-1] &= np.uint32((1 << (n % 32)) - 1)
        assert oracle.energy(W, X) == -tts.cut_value(X, n, ei, ej, w)   # Eq.(17)


def test_tsp_tour_decode_and_energy():
    c = 7
    _, D = tsp_instance(c, seed=3)
    W = tsp_qubo(c, seed=3)
    A = 2 * int(D.max())
    rng = np.random.default_rng(2)
    for _ in range(10):
        tour = [int(u) for u in rng.permutation(c)]
        bits = np.zeros(c * c, np.uint8)
        for t, u in enumerate(tour):
            bits[u * c + t] = 1
        X = np.packbits(bits, bitorder="little")
        X = np.concatenate([X, np.zeros((-len(X)) % 4, np.uint8)]).view(np.uint32)
        assert tts.tsp_tour(X, c) == tour
        assert oracle.energy(W, X) == 2 * tts.tour_length(tour, D) - 2 * c * A   # reading C13
        bits[tour[0] * c + 0] = 0                    # drop a city: not a permutation
        Y = np.packbits(bits, bitorder="little")
        Y = np.concatenate([Y, np.zeros((-len(Y)) % 4, np.uint8)]).view(np.uint32)
        assert tts.tsp_tour(Y, c) is None


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank_worker(rank, world, port, out_dir):
    dist.init_process_group("gloo", init_method="tcp://127.0.0.1:%d" % port, rank=rank, world_size=world)
    # rank 1 reaches the target on its 3rd call, rank 0 never does: both stop after call 3
    s = ScriptedSolver([-1, -2, -3, -4] if rank == 0 else [-1, -2, -50, -60])
    r = tts.time_to_target(s, target_energy=-40, max_seconds=100, exchange_k=1, clock=Clock(1.0))
    np.savez(os.path.join(out_dir, "r%d.npz" % rank), reached=r.reached, calls=r.calls)
    dist.destroy_process_group()


def test_ranks_agree_on_success(tmp_path):
    tmp.spawn(_rank_worker, args=(2, _free_port(), str(tmp_path)), nprocs=2, join=True)
    for r in range(2):
        z = np.load(os.path.join(tmp_path, "r%d.npz" % r))
        assert bool(z["reached"]) and int(z["calls"]) == 3


@pytest.mark.gpu
def test_gpu_reaches_bruteforce_optimum():
    import paper_conf_icpp_yasudonitkyi20_b200 as pkg
    n = 16
    W = random_qubo(n, 21)
    e_min, _ = oracle.bruteforce(W)
    s = pkg.Solver(W, searches=64, local_flips=200, pool_size=16, seed=5)
    r = tts.time_to_target(s, target_energy=e_min, max_seconds=30)
    assert r.reached and r.best_energy == e_min
    assert oracle.energy(W, r.best_X) == e_min
    s.close()
