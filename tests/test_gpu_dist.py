"""Multi-GPU path with REAL solvers: two processes,
each with its own libabs context on cuda:0 (the only GPU a test box has) and a
gloo process group for the exchange, driven by dist.py exactly as bench.py
drives it over NCCL on N GPUs.

  * lockstep: rank r owns global search ids [r*S, (r+1)*S); every step
    all-gathers all (B, E_B) and inserts them in global-id order.  The pools,
    every emitted result and every search's trajectory must equal
    oracle.run_lockstep with 2*S searches in one process (pin P14).
  * async: each rank runs its searches freely, then the ranks all-gather their
    elites; both pools must then be sorted, distinct, hold true energies and
    share the same best solution."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

import oracle
from workloads import random_qubo

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as tmp  # noqa: E402


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _lockstep_worker(rank, world, port, n, S, R, L, out_dir):
    import paper_conf_icpp_yasudonitkyi20_b200 as pkg
    from paper_conf_icpp_yasudonitkyi20_b200 import dist as pdist
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method="tcp://127.0.0.1:%d" % port, rank=rank, world_size=world)
    W = random_qubo(n, 31)
    s = pkg.Solver(W, searches=S, search_offset=rank * S, external_merge=True, local_flips=L, pool_size=8, seed=9)
    Bs, Es = [], []
    for _ in range(R):
        B, E = pdist.lockstep_step(s)
        Bs.append(B)
        Es.append(E)
    PX, PE = s.pool(8)
    ins = pdist.exchange_elites(s, 4)          # identical pools: nothing new
    st = [s.search_state(i) for i in range(S)]
    np.savez(os.path.join(out_dir, "rank%d.npz" % rank), B=np.array(Bs), E=np.array(Es), PX=PX, PE=PE, ins=ins,
             hash=np.array([x["hash"] for x in st], np.uint64), flips=np.array([x["flips"] for x in st]),
             Es=np.array([x["E"] for x in st]), D=np.array([x["D"] for x in st]))
    s.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("n,S,R,L", [(300, 3, 3, 200), (3000, 2, 2, 300)])
def test_two_ranks_lockstep_equal_oracle_single_process(tmp_path, n, S, R, L):
    world = 2
    tmp.spawn(_lockstep_worker, args=(world, _free_port(), n, S, R, L, str(tmp_path)), nprocs=world, join=True)
    W = random_qubo(n, 31)
    o = oracle.run_lockstep(W, oracle.Config(n=n, searches=S * world, local_flips=L, pool_size=8, seed=9), R)
    fin = o["poolE"] != oracle.EINF
    for r in range(world):
        z = np.load(os.path.join(tmp_path, "rank%d.npz" % r))
        assert (z["E"] == o["EB"]).all(), "gathered E_B differ"            # every round, all 2S searches
        assert (z["B"] == o["B"]).all(), "gathered B differ"
        assert (z["PE"] == o["poolE"][fin]).all() and (z["PX"] == o["poolX"][fin]).all()
        assert int(z["ins"]) == 0
        g = slice(r * S, (r + 1) * S)                                       # this rank's global ids
        assert (z["hash"] == o["hash"][g]).all() and (z["flips"] == o["flips"][g]).all()
        assert (z["Es"] == o["E"][g]).all()
        assert (z["D"].astype(np.int64) == o["D"][g]).all()


def _async_worker(rank, world, port, n, S, steps, out_dir):
    import paper_conf_icpp_yasudonitkyi20_b200 as pkg
    from paper_conf_icpp_yasudonitkyi20_b200 import dist as pdist
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method="tcp://127.0.0.1:%d" % port, rank=rank, world_size=world)
    W = random_qubo(n, 44)
    s = pkg.Solver(W, searches=S, search_offset=rank * S, local_flips=150, pool_size=16, seed=12 + rank,
                   mode=pkg.MODE_ASYNC)
    s.search(steps)
    X0, E0 = s.pool(16)
    pdist.exchange_elites(s, 8)
    X1, E1 = s.pool(16)
    true = s.energy(X1) if len(E1) else np.zeros(0, np.int64)
    np.savez(os.path.join(out_dir, "a%d.npz" % rank), X0=X0, E0=E0, X1=X1, E1=E1, true=true)
    s.close()
    dist.destroy_process_group()


def test_two_ranks_async_elite_exchange(tmp_path):
    world = 2
    tmp.spawn(_async_worker, args=(world, _free_port(), 500, 40, 3, str(tmp_path)), nprocs=world, join=True)
    z = [np.load(os.path.join(tmp_path, "a%d.npz" % r)) for r in range(world)]
    best = min(int(x["E0"][0]) for x in z)
    for x in z:
        E1 = x["E1"]
        assert (np.diff(E1) > 0).all()                       # sorted, distinct
        assert (x["true"] == E1).all()                       # true energies (Eq.(1), on device)
        assert int(E1[0]) == best                            # both ranks hold the global best
    W = random_qubo(500, 44)
    Xb = z[0]["X1"][0]
    assert oracle.energy(W, Xb) == best


def _nccl_worker(rank, world, port, out_dir):
    import paper_conf_icpp_yasudonitkyi20_b200 as pkg
    from paper_conf_icpp_yasudonitkyi20_b200 import dist as pdist
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", init_method="tcp://127.0.0.1:%d" % port, rank=rank, world_size=world,
                            device_id=torch.device("cuda", 0))
    n, S, R, L = 300, 4, 2, 150
    W = random_qubo(n, 32)
    s = pkg.Solver(W, searches=S, external_merge=True, local_flips=L, pool_size=8, seed=10)
    Es = []
    for _ in range(R):
        _, E = pdist.lockstep_step(s)   # all_gather_into_tensor over NCCL on cuda:0
        Es.append(E)
    PX, PE = s.pool(8)
    ins = pdist.exchange_elites(s, 4)
    np.savez(os.path.join(out_dir, "nccl%d.npz" % rank), E=np.array(Es), PX=PX, PE=PE, ins=ins,
             backend=np.array([dist.get_backend()]))
    s.close()
    dist.destroy_process_group()


def test_nccl_backend_single_rank(tmp_path):
    """The NCCL path of dist.py (device tensors, all_gather_into_tensor) with a
    one-rank communicator on cuda:0 -- NCCL refuses two ranks on one device, so
    this is the only NCCL execution a one-GPU box allows.  The run equals the
    one-process oracle."""
    tmp.spawn(_nccl_worker, args=(1, _free_port(), str(tmp_path)), nprocs=1, join=True)
    z = np.load(os.path.join(tmp_path, "nccl0.npz"))
    assert str(z["backend"][0]) == "nccl"
    W = random_qubo(300, 32)
    o = oracle.run_lockstep(W, oracle.Config(n=300, searches=4, local_flips=150, pool_size=8, seed=10), 2)
    fin = o["poolE"] != oracle.EINF
    assert (z["E"] == o["EB"]).all()
    assert (z["PE"] == o["poolE"][fin]).all() and (z["PX"] == o["poolX"][fin]).all()
    assert int(z["ins"]) == 0
