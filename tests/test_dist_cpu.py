"""Multi-process (world_size 2, gloo, CPU) tests of the multi-GPU host logic in
paper_conf_icpp_yasudonitkyi20_b200/dist.py: the lockstep result exchange and
the elite exchange.  The per-rank solver is an oracle-backed stand-in with the
same methods as abs.Solver (search / round_results / pool_insert / pool), so
the exchange logic is exercised without a GPU; the GPU path itself is covered
by tests/test_gpu_parity.py::test_sharded_ranks_equal_single_process."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

import oracle
from workloads import random_qubo

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as tmp  # noqa: E402


class OracleRankSolver:
    """Lockstep searches [offset, offset+S) of a run with a replicated pool."""

    def __init__(self, W, S, offset, cfg: oracle.Config):
        self.W = W
        self.n = W.shape[0]
        self.words = (self.n + 31) // 32
        self.cfg = cfg
        self.offset = offset
        lad = oracle.default_ladder(self.n)
        self.searches = [oracle.Search(W, l=lad[(offset + s) % len(lad)]) for s in range(S)]
        self.pool_ = oracle.Pool(self.n, cfg.pool_size, seed=cfg.seed)
        self.r = 0
        self._B = None
        self._E = None

    def search(self, steps):
        for _ in range(steps):
            B, E = [], []
            for i, s in enumerate(self.searches):
                T = self.pool_.target(self.cfg, self.r, self.offset + i)
                s.round(T, self.cfg.local_flips)
                B.append(s.b)
                E.append(s.EB)
            self._B, self._E = np.array(B, np.uint32), np.array(E, np.int64)
            self.r += 1

    def round_results(self):
        return self._B, self._E

    def pool_insert(self, X, E):
        return sum(self.pool_.insert(x, e) for x, e in zip(X, E))

    def pool(self, k):
        E = self.pool_.E
        X = self.pool_.X
        fin = E != oracle.EINF
        return X[fin][:k], E[fin][:k]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, S, R, L, out_dir):
    from paper_conf_icpp_yasudonitkyi20_b200 import dist as pdist
    dist.init_process_group("gloo", init_method="tcp://127.0.0.1:%d" % port, rank=rank, world_size=world)
    W = random_qubo(n, 31)
    cfg = oracle.Config(n=n, searches=S * world, local_flips=L, pool_size=8, seed=9)
    sol = OracleRankSolver(W, S, rank * S, cfg)
    for _ in range(R):
        pdist.lockstep_step(sol)
    X, E = sol.pool(8)
    # elite exchange must leave identical pools unchanged
    ins = pdist.exchange_elites(sol, 4)
    X2, E2 = sol.pool(8)
    np.savez(os.path.join(out_dir, "rank%d.npz" % rank), X=X, E=E, X2=X2, E2=E2, ins=ins)
    dist.destroy_process_group()


def test_lockstep_exchange_two_ranks_equals_single_process(tmp_path):
    n, S, R, L, world = 40, 3, 3, 30, 2
    tmp.spawn(_worker, args=(world, _free_port(), n, S, R, L, str(tmp_path)), nprocs=world, join=True)
    W = random_qubo(n, 31)
    o = oracle.run_lockstep(W, oracle.Config(n=n, searches=S * world, local_flips=L, pool_size=8, seed=9), R)
    fin = o["poolE"] != oracle.EINF
    for r in range(world):
        z = np.load(os.path.join(tmp_path, "rank%d.npz" % r))
        assert (z["E"] == o["poolE"][fin]).all()
        assert (z["X"] == o["poolX"][fin]).all()
        assert int(z["ins"]) == 0                 # identical pools: nothing new
        assert (z["E2"] == z["E"]).all()


def _elite_worker(rank, world, port, out_dir):
    from paper_conf_icpp_yasudonitkyi20_b200 import dist as pdist

    class Fake:
        words = 2

        def __init__(self, r):
            self.X = np.array([[r + 1, 0], [r + 7, 1]], np.uint32)
            self.E = np.array([-100 * (r + 1), -5 * (r + 1)], np.int64)
            self.got = []

        def pool(self, k):
            return self.X[:k], self.E[:k]

        def pool_insert(self, X, E):
            self.got.append((X.copy(), E.copy()))
            return len(E)

    dist.init_process_group("gloo", init_method="tcp://127.0.0.1:%d" % port, rank=rank, world_size=world)
    f = Fake(rank)
    pdist.exchange_elites(f, 3)   # k larger than the pool: padding must be dropped
    X, E = f.got[0]
    np.savez(os.path.join(out_dir, "e%d.npz" % rank), X=X, E=E)
    dist.destroy_process_group()


def test_elite_exchange_rank_order_and_padding(tmp_path):
    tmp.spawn(_elite_worker, args=(2, _free_port(), str(tmp_path)), nprocs=2, join=True)
    for r in range(2):
        z = np.load(os.path.join(tmp_path, "e%d.npz" % r))
        assert z["E"].tolist() == [-100, -5, -200, -10]      # rank order, +inf padding removed
        assert z["X"][:, 0].tolist() == [1, 7, 2, 8]


def test_bench_refuses_gpus_world_mismatch():
    """bench.py --gpus N under a launcher with WORLD_SIZE != N must refuse to run
    (one process per GPU), instead of silently timing a different world."""
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, WORLD_SIZE="3", RANK="0", LOCAL_RANK="0")
    p = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--steps", "1"],
                       env=env, capture_output=True, text=True, timeout=120)
    assert p.returncode == 2 and "WORLD_SIZE" in p.stderr
