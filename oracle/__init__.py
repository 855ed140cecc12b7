"""ORACLE — TEST INFRASTRUCTURE ONLY.

ctypes wrapper around the plain-C oracle (oracle/oracle.c).  Only tests/,
__graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
may import this package; the product path (paper_conf_icpp_yasudonitkyi20_b200)
never does and shares no code with it.

Every function mirrors one in oracle.h, which cites the PAPER.md passage it
follows.  Parity pins: tests/test_oracle_pins.py.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_HDR = os.path.join(_HERE, "oracle.h")
_LIB = os.path.join(_HERE, "liboracle.so")

EINF = np.iinfo(np.int64).max


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (plain -O2, no vectorisation flags)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(os.path.getmtime(_SRC), os.path.getmtime(_HDR)):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-std=c99", "-O2", "-fPIC", "-shared", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


class _Cfg(C.Structure):
    _fields_ = [
        ("n", C.c_int32),
        ("searches", C.c_int32),
        ("local_flips", C.c_int64),
        ("pool_size", C.c_int32),
        ("ladder_len", C.c_int32),
        ("ladder", C.c_int32 * 32),
        ("seed", C.c_uint64),
        ("p_cross", C.c_int32),
        ("p_mut", C.c_int32),
        ("mut_max", C.c_int32),
        ("policy", C.c_int32),
        ("sa_tau_min", C.c_int32),
        ("sa_tau_max", C.c_int32),
        ("sa_levels", C.c_int32),
    ]


def _P(t):
    return C.POINTER(t)


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        L.oracle_philox4x32_10.argtypes = [_P(C.c_uint32), _P(C.c_uint32), _P(C.c_uint32)]
        L.oracle_energy.restype = C.c_int64
        L.oracle_energy.argtypes = [C.c_int32, _P(C.c_int16), _P(C.c_uint32)]
        L.oracle_ising_energy.restype = C.c_int64
        L.oracle_ising_energy.argtypes = [C.c_int32, _P(C.c_int32), _P(C.c_int32), _P(C.c_int8)]
        L.oracle_delta_by_definition.restype = C.c_int64
        L.oracle_delta_by_definition.argtypes = [C.c_int32, _P(C.c_int16), _P(C.c_uint32), C.c_int32]
        L.oracle_init_batch.argtypes = [C.c_int32, _P(C.c_int16), C.c_int32, _P(C.c_uint32), _P(C.c_int64), _P(C.c_int64)]
        L.oracle_run_lockstep.restype = C.c_int
        L.oracle_run_lockstep.argtypes = [C.c_int32, _P(C.c_int16), _P(_Cfg), C.c_int32,
                                          _P(C.c_uint32), _P(C.c_int64), _P(C.c_int64), _P(C.c_int32),
                                          _P(C.c_uint64), _P(C.c_int64), _P(C.c_uint32), _P(C.c_int64),
                                          _P(C.c_int64), _P(C.c_uint32)]
        L.oracle_replay_search.restype = C.c_int
        L.oracle_replay_search.argtypes = [C.c_int32, _P(C.c_int16), C.c_int32, C.c_int64, C.c_int32,
                                           _P(C.c_uint32), _P(C.c_uint32), _P(C.c_int64), _P(C.c_int64),
                                           _P(C.c_int32), _P(C.c_uint64), _P(C.c_int64), _P(C.c_uint32), _P(C.c_int64)]
        L.oracle_replay_search_sa.restype = C.c_int
        L.oracle_replay_search_sa.argtypes = [C.c_int32, _P(C.c_int16), C.c_int32, C.c_uint32, C.c_uint64, C.c_int64,
                                              C.c_int32, _P(C.c_uint32), _P(C.c_uint32), _P(C.c_int64),
                                              _P(C.c_int64), _P(C.c_int32), _P(C.c_uint64), _P(C.c_int64),
                                              _P(C.c_uint32), _P(C.c_int64)]
        L.oracle_sa_threshold.restype = C.c_uint64
        L.oracle_sa_threshold.argtypes = [C.c_int64, C.c_int32]
        L.oracle_local_sa.restype = None
        L.oracle_local_sa.argtypes = [_P(_Search), C.c_int64]
        L.oracle_bruteforce.restype = C.c_int64
        L.oracle_bruteforce.argtypes = [C.c_int32, _P(C.c_int16), _P(C.c_uint32)]
        L.oracle_pool_insert.restype = C.c_int
        _lib = L
    return _lib


def _ptr(a, t):
    if a is None:
        return None
    return a.ctypes.data_as(_P(t))


def _W(W):
    W = np.ascontiguousarray(W, dtype=np.int16)
    assert W.ndim == 2 and W.shape[0] == W.shape[1]
    return W


def _X(X, n):
    X = np.ascontiguousarray(X, dtype=np.uint32)
    return X


def words(n: int) -> int:
    return (n + 31) // 32


# ---------------------------------------------------------------- primitives
def philox4x32_10(ctr, key):
    c = np.ascontiguousarray(ctr, dtype=np.uint32)
    k = np.ascontiguousarray(key, dtype=np.uint32)
    o = np.zeros(4, dtype=np.uint32)
    lib().oracle_philox4x32_10(_ptr(c, C.c_uint32), _ptr(k, C.c_uint32), _ptr(o, C.c_uint32))
    return o


def energy(W, X) -> int:
    """Eq.(1) for one packed vector."""
    W = _W(W)
    X = _X(X, W.shape[0])
    return int(lib().oracle_energy(W.shape[0], _ptr(W, C.c_int16), _ptr(X, C.c_uint32)))


def ising_energy(J, h, s) -> int:
    """P:L40 for spins s in {-1,+1} (pairs i<j, reading E1)."""
    J = np.ascontiguousarray(J, dtype=np.int32)
    h = np.ascontiguousarray(h, dtype=np.int32)
    s = np.ascontiguousarray(s, dtype=np.int8)
    return int(lib().oracle_ising_energy(J.shape[0], _ptr(J, C.c_int32), _ptr(h, C.c_int32), _ptr(s, C.c_int8)))


def delta_by_definition(W, X, k: int) -> int:
    W = _W(W)
    X = _X(X, W.shape[0])
    return int(lib().oracle_delta_by_definition(W.shape[0], _ptr(W, C.c_int16), _ptr(X, C.c_uint32), int(k)))


def init_batch(W, X):
    """Eq.(13) deltas and Eq.(1) energies for a batch X uint32[count, words]."""
    W = _W(W)
    n = W.shape[0]
    X = np.ascontiguousarray(np.atleast_2d(X), dtype=np.uint32)
    cnt = X.shape[0]
    D = np.zeros((cnt, n), dtype=np.int64)
    E = np.zeros(cnt, dtype=np.int64)
    lib().oracle_init_batch(n, _ptr(W, C.c_int16), cnt, _ptr(X, C.c_uint32), _ptr(D, C.c_int64), _ptr(E, C.c_int64))
    return D, E


def bruteforce(W):
    W = _W(W)
    x = np.zeros(1, dtype=np.uint32)
    e = lib().oracle_bruteforce(W.shape[0], _ptr(W, C.c_int16), _ptr(x, C.c_uint32))
    return int(e), x


# ---------------------------------------------------------------- runs
def sa_threshold(dE: int, tau: int) -> int:
    """Reading E2: the uint32 acceptance bound of an uphill move dE > 0."""
    return int(lib().oracle_sa_threshold(int(dE), int(tau)))


def default_ladder(n: int):
    """Reading C7: l in {4, 8, 16, ..., min(256, n/4)} (n < 16 -> {max(1, n//4)})."""
    top = min(256, max(1, n // 4))
    lad = []
    v = 4
    while v <= top:
        lad.append(v)
        v *= 2
    return lad or [max(1, top)]


@dataclass
class Config:
    n: int
    searches: int
    local_flips: int | None = None     # default n (reading C8)
    pool_size: int = 64
    ladder: list = field(default_factory=list)
    seed: int = 1
    p_cross: int = 450
    p_mut: int = 450
    mut_max: int | None = None        # default max(1, n // 32)
    policy: int = 0                   # 0 = window (Fig. 2), 1 = SA (Eq.(7), reading E2)
    sa_tau_min: int = 1
    sa_tau_max: int = 1
    sa_levels: int = 1

    def c(self) -> _Cfg:
        c = _Cfg()
        c.n = self.n
        c.searches = self.searches
        c.local_flips = self.n if self.local_flips is None else int(self.local_flips)
        c.pool_size = self.pool_size
        lad = list(self.ladder) or default_ladder(self.n)
        assert 1 <= len(lad) <= 32
        c.ladder_len = len(lad)
        for i, v in enumerate(lad):
            c.ladder[i] = int(v)
        c.seed = int(self.seed) & 0xFFFFFFFFFFFFFFFF
        c.p_cross = self.p_cross
        c.p_mut = self.p_mut
        c.mut_max = max(1, self.n // 32) if self.mut_max is None else int(self.mut_max)
        c.policy = int(self.policy)
        c.sa_tau_min = int(self.sa_tau_min)
        c.sa_tau_max = int(self.sa_tau_max)
        c.sa_levels = int(self.sa_levels)
        return c


def run_lockstep(W, cfg: Config, rounds: int, want_emitted: bool = True):
    """Deterministic lockstep run; returns a dict of numpy arrays."""
    W = _W(W)
    n = W.shape[0]
    assert cfg.n == n
    S, w, m = cfg.searches, words(n), cfg.pool_size
    out = dict(
        X=np.zeros((S, w), np.uint32), D=np.zeros((S, n), np.int64), E=np.zeros(S, np.int64),
        a=np.zeros(S, np.int32), hash=np.zeros(S, np.uint64), flips=np.zeros(S, np.int64),
        poolE=np.zeros(m, np.int64), poolX=np.zeros((m, w), np.uint32))
    if want_emitted:
        out["B"] = np.zeros((rounds, S, w), np.uint32)
        out["EB"] = np.zeros((rounds, S), np.int64)
    c = cfg.c()
    rc = lib().oracle_run_lockstep(
        n, _ptr(W, C.c_int16), C.byref(c), int(rounds),
        _ptr(out["X"], C.c_uint32), _ptr(out["D"], C.c_int64), _ptr(out["E"], C.c_int64),
        _ptr(out["a"], C.c_int32), _ptr(out["hash"], C.c_uint64), _ptr(out["flips"], C.c_int64),
        _ptr(out.get("B"), C.c_uint32), _ptr(out.get("EB"), C.c_int64),
        _ptr(out["poolE"], C.c_int64), _ptr(out["poolX"], C.c_uint32))
    if rc != 0:
        raise RuntimeError("oracle_run_lockstep rc=%d" % rc)
    return out


def replay_search(W, l: int, L: int, T, policy: int = 0, tau: int = 1, sid: int = 0, seed: int = 1):
    """Rounds of one search against a given target sequence T uint32[rounds, words].
    policy 0: window of length l (Fig. 2); policy 1: SA (reading E2) at
    temperature tau, global search id sid, Philox key seed (l unused)."""
    W = _W(W)
    n = W.shape[0]
    T = np.ascontiguousarray(np.atleast_2d(T), dtype=np.uint32)
    R, w = T.shape[0], words(n)
    out = dict(X=np.zeros(w, np.uint32), D=np.zeros(n, np.int64), E=np.zeros(1, np.int64),
               a=np.zeros(1, np.int32), hash=np.zeros(1, np.uint64), flips=np.zeros(1, np.int64),
               B=np.zeros((R, w), np.uint32), EB=np.zeros(R, np.int64))
    outs = (_ptr(out["X"], C.c_uint32), _ptr(out["D"], C.c_int64), _ptr(out["E"], C.c_int64),
            _ptr(out["a"], C.c_int32), _ptr(out["hash"], C.c_uint64), _ptr(out["flips"], C.c_int64),
            _ptr(out["B"], C.c_uint32), _ptr(out["EB"], C.c_int64))
    if policy == 1:
        rc = lib().oracle_replay_search_sa(n, _ptr(W, C.c_int16), int(tau), int(sid), int(seed) & 0xFFFFFFFFFFFFFFFF,
                                           int(L), R, _ptr(T, C.c_uint32), *outs)
    else:
        rc = lib().oracle_replay_search(n, _ptr(W, C.c_int16), int(l), int(L), R, _ptr(T, C.c_uint32), *outs)
    if rc != 0:
        raise RuntimeError("oracle_replay_search rc=%d" % rc)
    return out


def sa_tau_of(sid: int, tau_min: int, tau_max: int, levels: int) -> int:
    """Reading E2: search sid (global id) at level j = sid mod K has
    tau = tau_min + (tau_max - tau_min) j / (K - 1) (integer division)."""
    K = max(1, levels)
    j = sid % K
    return tau_min if K == 1 else tau_min + (tau_max - tau_min) * j // (K - 1)


# ---------------------------------------------------------------- stepwise access
class _Search(C.Structure):
    _fields_ = [
        ("n", C.c_int32), ("W", _P(C.c_int16)), ("x", _P(C.c_uint32)), ("d", _P(C.c_int64)),
        ("E", C.c_int64), ("a", C.c_int32), ("l", C.c_int32), ("b", _P(C.c_uint32)),
        ("EB", C.c_int64), ("hash", C.c_uint64), ("flips", C.c_int64), ("overflow", C.c_int32),
        ("policy", C.c_int32), ("tau", C.c_int32), ("sid", C.c_uint32), ("seed", C.c_uint64),
        ("sa_ctr", C.c_uint64),
    ]


class Search:
    """Step-by-step handle on one oracle search (for invariant tests)."""

    def __init__(self, W, l: int = 4):
        self.W = _W(W)
        self.n = self.W.shape[0]
        self._s = _Search()
        if lib().oracle_search_init(C.byref(self._s), self.n, _ptr(self.W, C.c_int16), int(l)) != 0:
            raise MemoryError

    def __del__(self):
        try:
            lib().oracle_search_free(C.byref(self._s))
        except Exception:
            pass

    @property
    def x(self):
        return np.ctypeslib.as_array(self._s.x, shape=(words(self.n),)).copy()

    @property
    def b(self):
        return np.ctypeslib.as_array(self._s.b, shape=(words(self.n),)).copy()

    @property
    def d(self):
        return np.ctypeslib.as_array(self._s.d, shape=(self.n,)).copy()

    E = property(lambda self: int(self._s.E))
    EB = property(lambda self: int(self._s.EB))
    a = property(lambda self: int(self._s.a))
    l = property(lambda self: int(self._s.l))
    flips = property(lambda self: int(self._s.flips))
    hash = property(lambda self: int(self._s.hash))
    overflow = property(lambda self: bool(self._s.overflow))

    def set_best(self, B=None, EB=None):
        """Step 3 reset (B = X, E_B = E) or explicit values."""
        w = words(self.n)
        src = self.x if B is None else np.ascontiguousarray(B, dtype=np.uint32)
        dst = np.ctypeslib.as_array(self._s.b, shape=(w,))
        dst[:] = src
        self._s.EB = self.E if EB is None else int(EB)

    def set_offset(self, a: int):
        self._s.a = int(a)

    def flip(self, k: int):
        lib().oracle_flip(C.byref(self._s), int(k))

    def track(self):
        lib().oracle_track(C.byref(self._s))

    def straight(self, T) -> int:
        T = np.ascontiguousarray(T, dtype=np.uint32)
        lib().oracle_straight.restype = C.c_int64
        return int(lib().oracle_straight(C.byref(self._s), _ptr(T, C.c_uint32)))

    def local(self, L: int):
        lib().oracle_local(C.byref(self._s), C.c_int64(int(L)))

    def set_sa(self, tau: int, sid: int = 0, seed: int = 1, ctr: int = 0):
        """Switch this search to the SA policy (reading E2)."""
        self._s.policy = 1
        self._s.tau = int(tau)
        self._s.sid = int(sid)
        self._s.seed = int(seed) & 0xFFFFFFFFFFFFFFFF
        self._s.sa_ctr = int(ctr)

    @property
    def sa_ctr(self) -> int:
        return int(self._s.sa_ctr)

    def local_sa(self, L: int):
        lib().oracle_local_sa(C.byref(self._s), C.c_int64(int(L)))

    def round(self, T, L: int):
        T = np.ascontiguousarray(T, dtype=np.uint32)
        lib().oracle_round(C.byref(self._s), _ptr(T, C.c_uint32), C.c_int64(int(L)))


class Pool:
    """Handle on an oracle pool (host GA)."""

    class _CPool(C.Structure):
        _fields_ = [("n", C.c_int32), ("m", C.c_int32), ("words", C.c_int32),
                    ("E", _P(C.c_int64)), ("X", _P(C.c_uint32))]

    def __init__(self, n: int, m: int, seed: int = 1):
        self.n, self.m = n, m
        self._p = Pool._CPool()
        if lib().oracle_pool_init(C.byref(self._p), int(n), int(m), C.c_uint64(int(seed))) != 0:
            raise MemoryError

    def __del__(self):
        try:
            lib().oracle_pool_free(C.byref(self._p))
        except Exception:
            pass

    @property
    def E(self):
        return np.ctypeslib.as_array(self._p.E, shape=(self.m,)).copy()

    @property
    def X(self):
        return np.ctypeslib.as_array(self._p.X, shape=(self.m, words(self.n))).copy()

    def insert(self, X, E) -> bool:
        X = np.ascontiguousarray(X, dtype=np.uint32)
        return bool(lib().oracle_pool_insert(C.byref(self._p), _ptr(X, C.c_uint32), C.c_int64(int(E))))

    def target(self, cfg: Config, r: int, sid: int):
        T = np.zeros(words(self.n), dtype=np.uint32)
        c = cfg.c()
        lib().oracle_ga_target(C.byref(self._p), C.byref(c), C.c_int64(int(r)), C.c_int64(int(sid)), _ptr(T, C.c_uint32))
        return T
