"""Time-to-solution harness: the Table 1 analogue (SURVEY §8(f)
row 1) on top of the public Solver API.  The hot path is reused unchanged.

TTS is the wall time from the first abs_search call until the solution pool
holds a solution that meets the target.  Table 1 takes as targets "the
best-known solution or those close to it": 99% / 95% of a best-known
cut (Max-Cut), best-known tour + 5% / 10% (TSP), and 99% of a best-known
energy (random instances).  For random instances the best-known value is
itself "computed by repeating searches until convergence";
tools/tts_run.py does that with a long reference run.

Multi-GPU: each rank runs its own Solver (its own search ids).  After every
abs_search call the ranks all-gather their elites (dist.exchange_elites) and
all-reduce the success flag, so every rank stops after the same call.
Time is rank 0's clock after that collective, i.e. the max over ranks."""
from __future__ import annotations

import math
import time
from dataclasses import dataclass, field
from fractions import Fraction

import numpy as np

from .abs import ABS_EEMPTY, AbsError


@dataclass
class TTSResult:
    reached: bool
    seconds: float | None          # wall time to the target (None if not reached)
    best_energy: int | None        # best pool energy at the end (this rank)
    best_X: np.ndarray | None
    calls: int                     # abs_search calls made
    elapsed: float                 # wall time of the whole run
    trace: list = field(default_factory=list)  # [(seconds, best energy)] at every improvement


def energy_target(best_known: int, fraction) -> int:
    """The largest integer energy E with E <= fraction * best_known: reaching
    `fraction` (e.g. 0.99) of a negative best-known energy (Table 1(c))."""
    f = Fraction(fraction).limit_denominator(10 ** 9)
    return math.floor(f * best_known)


def cut_target(best_cut: int, fraction) -> int:
    """Energy target for a Max-Cut QUBO (E = -cut, Eq.(17)): cut >= ceil(fraction * best_cut)."""
    f = Fraction(fraction).limit_denominator(10 ** 9)
    return -math.ceil(f * best_cut)


def _unpack(X, n):
    X = np.asarray(X, dtype=np.uint32)
    bits = np.unpackbits(X.view(np.uint8), bitorder="little")
    return bits[:n]


def cut_value(X, n: int, ei, ej, w) -> int:
    """Cut weight of the partition X (bit i = side of vertex i), edges (ei, ej, w)."""
    x = _unpack(X, n).astype(bool)
    return int(np.sum(np.asarray(w)[x[np.asarray(ei)] != x[np.asarray(ej)]]))


def tsp_tour(X, c: int):
    """Decode the one-hot TSP encoding of reading C13 (bit u*c + t = city u at
    position t): the tour as a list of cities by position, or None if X is not
    a permutation matrix."""
    x = _unpack(X, c * c).reshape(c, c)
    if not ((x.sum(axis=0) == 1).all() and (x.sum(axis=1) == 1).all()):
        return None
    return [int(u) for u in np.argmax(x, axis=0)]


def tour_length(tour, D) -> int:
    D = np.asarray(D)
    return int(sum(D[tour[t], tour[(t + 1) % len(tour)]] for t in range(len(tour))))


def _best(solver):
    try:
        X, E = solver.best()
        return X, int(E)
    except AbsError as e:
        if e.rc == ABS_EEMPTY:
            return None, None
        raise


def time_to_target(solver, target_energy: int | None = None, accept=None, max_seconds: float = 10.0,
                   rounds_per_call: int = 1, exchange_k: int = 0, group=None, clock=time.perf_counter) -> TTSResult:
    """Run `solver` until its best solution meets the target or max_seconds pass.

    target_energy: success when the best pool energy is <= target_energy.
    accept(X, E) -> bool: success predicate on the best pool entry instead
      (e.g. a valid TSP tour within a length bound).
    Under torch.distributed (group or the default group initialised) the ranks
    exchange their top `exchange_k` elites after every call and agree on success."""
    if target_energy is None and accept is None:
        raise ValueError("need target_energy or accept")
    dist = None
    try:
        import torch.distributed as _d
        if _d.is_available() and _d.is_initialized():
            dist = _d
    except ImportError:
        pass
    t0 = clock()
    best = None
    trace = []
    calls = 0
    while True:
        solver.search(rounds_per_call)
        calls += 1
        if dist is not None and exchange_k > 0:
            from .dist import exchange_elites
            exchange_elites(solver, exchange_k, group)
        X, E = _best(solver)
        ok = E is not None and (accept(X, E) if accept is not None else E <= target_energy)
        if dist is not None:
            import torch
            from .dist import _device_for_backend
            flag = torch.tensor([1 if ok else 0], dtype=torch.int32, device=_device_for_backend())
            dist.all_reduce(flag, op=dist.ReduceOp.MAX, group=group)
            ok = bool(flag.item())
        t = clock() - t0
        if E is not None and (best is None or E < best):
            best = E
            trace.append((t, E))
        if ok:
            return TTSResult(True, t, best, X, calls, t, trace)
        if t >= max_seconds:
            return TTSResult(False, None, best, X, calls, t, trace)
