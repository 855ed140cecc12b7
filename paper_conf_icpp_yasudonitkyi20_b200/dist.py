"""Multi-GPU partitioning (one process per GPU) and the only collective of
the path: an all-gather of search results / elite solutions over
torch.distributed (NCCL on B200s, gloo in the CPU tests).

The paper runs independent searches on every GPU over ALL n bits (P:L546,
P:L389 Fig. 5) under one host; here each GPU has its own process, so the
host GA pools are joined by exchanging solutions:

  * Lockstep (deterministic) mode: rank r owns global search ids
    [r*S, (r+1)*S).  After every step each rank all-gathers the (B, E_B) of
    every search and inserts them all in global-id order, so every rank holds
    the SAME pool and the run is identical to one process with world*S
    searches (pin P14).
  * Elite exchange (async mode): every `every` steps the top-k pool entries
    of each rank are all-gathered and inserted in rank order.

The solver object only needs the methods of abs.Solver used below, which
lets the CPU tests drive this module with a stand-in."""
from __future__ import annotations

import numpy as np


def _gather(t, group=None):
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    out = torch.empty((world * t.shape[0],) + tuple(t.shape[1:]), dtype=t.dtype, device=t.device)
    dist.all_gather_into_tensor(out, t.contiguous(), group=group)  # concatenated in rank order
    return out


def _device_for_backend():
    import torch
    import torch.distributed as dist
    if dist.get_backend() == "nccl":
        return torch.device("cuda", torch.cuda.current_device())
    return torch.device("cpu")


def exchange_round_results(B: np.ndarray, EB: np.ndarray, group=None):
    """All-gather every rank's emitted (B [S, words] uint32, E_B [S] int64);
    returns the concatenation in rank order (= global search-id order)."""
    import torch
    dev = _device_for_backend()
    tb = torch.from_numpy(np.ascontiguousarray(B).view(np.int32)).to(dev)
    te = torch.from_numpy(np.ascontiguousarray(EB)).to(dev)
    gb = _gather(tb, group).cpu().numpy().view(np.uint32)
    ge = _gather(te, group).cpu().numpy()
    return gb.reshape(-1, B.shape[1]), ge.reshape(-1)


def lockstep_step(solver, group=None):
    """One deterministic multi-rank step: local round (abs_search(1) with
    external_merge), all-gather of all results, insert in global-id order."""
    solver.search(1)
    B, EB = solver.round_results()
    allB, allE = exchange_round_results(B, EB, group)
    solver.pool_insert(allB, allE)
    return allB, allE


def exchange_elites(solver, k: int, group=None):
    """All-gather the top-k finite pool entries of every rank and insert them
    (rank order).  Ranks with fewer than k finite entries pad with +inf rows
    that the pool rule rejects."""
    X, E = solver.pool(k)
    words = solver.words
    Xp = np.zeros((k, words), np.uint32)
    Ep = np.full(k, np.iinfo(np.int64).max, np.int64)
    Xp[: len(E)] = X
    Ep[: len(E)] = E
    allX, allE = exchange_round_results(Xp, Ep, group)
    keep = allE != np.iinfo(np.int64).max
    return solver.pool_insert(allX[keep], allE[keep])
