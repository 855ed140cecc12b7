"""Thin ctypes binding of libabs.so (include/abs.h).  Argument marshalling
only: every step of the search runs in the library's sm_100a kernels and its
host GA; there is no Python or CPU fallback.  Names follow the C ABI."""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

from . import build as _build

ABS_OK = 0
ABS_EINVAL = -1
ABS_ENOMEM = -2
ABS_ECUDA = -3
ABS_ESTATE = -5
ABS_EEMPTY = -6
ABS_ERANGE = -7
ABS_N_MAX = 32768
ABS_LADDER_MAX = 32
MODE_LOCKSTEP = 0
MODE_ASYNC = 1
POLICY_WINDOW = 0
POLICY_SA = 1


class AbsError(RuntimeError):
    def __init__(self, rc: int, where: str, detail: str):
        super().__init__("%s failed: %s (%d): %s" % (where, _strerror(rc), rc, detail))
        self.rc = rc


class abs_config(C.Structure):
    _fields_ = [
        ("searches", C.c_int32),
        ("search_offset", C.c_int32),
        ("local_flips", C.c_int64),
        ("pool_size", C.c_int32),
        ("ladder_len", C.c_int32),
        ("ladder", C.c_int32 * ABS_LADDER_MAX),
        ("seed", C.c_uint64),
        ("p_cross", C.c_int32),
        ("p_mut", C.c_int32),
        ("mut_max", C.c_int32),
        ("mode", C.c_int32),
        ("external_merge", C.c_int32),
        ("device", C.c_int32),
        ("trace", C.c_int32),
        ("policy", C.c_int32),
        ("sa_tau_min", C.c_int32),
        ("sa_tau_max", C.c_int32),
        ("sa_levels", C.c_int32),
        ("reserved", C.c_int32 * 3),
    ]


class abs_stats(C.Structure):
    _fields_ = [
        ("flips", C.c_int64),
        ("straight_flips", C.c_int64),
        ("evaluated", C.c_int64),
        ("rounds", C.c_int64),
        ("search_seconds", C.c_double),
        ("pool_inserted", C.c_int64),
        ("n", C.c_int32),
        ("n_pad", C.c_int32),
        ("searches", C.c_int32),
        ("threads_per_search", C.c_int32),
        ("steps", C.c_int64),
        ("h2d_bytes", C.c_int64),
        ("d2h_bytes", C.c_int64),
        ("kernel_launches", C.c_int64),
        ("step_seconds", C.c_double),
        ("round_kernel_launches", C.c_int64),
        ("init_seconds", C.c_double),
    ]


EXPORTS = [
    "abs_config_init", "abs_create", "abs_create_dev", "abs_seed_pool", "abs_search", "abs_best",
    "abs_stats_get", "abs_pool_get", "abs_pool_insert", "abs_energy", "abs_energy_dev", "abs_round_results",
    "abs_round_targets", "abs_trace_count", "abs_trace_get", "abs_search_state", "abs_debug_timing", "abs_destroy", "abs_strerror", "abs_last_error", "abs_device_searches", "abs_ising_to_qubo", "abs_qubo_to_ising", "abs_version",
    "abs_random_qubo_dev",
]

_lib = None


def library_path() -> str:
    return _build.LIB


def load(build_if_missing: bool = True):
    """Load libabs.so (building it in-tree with nvcc if it is missing or stale)."""
    global _lib
    if _lib is not None:
        return _lib
    path = os.environ.get("ABS_LIB") or _build.LIB  # ABS_LIB: diagnostics builds only
    if build_if_missing and not os.environ.get("ABS_LIB"):
        try:
            path = _build.build()
        except Exception as e:  # no nvcc: only an existing library can be used
            if not os.path.exists(path):
                raise ImportError("libabs.so is missing and cannot be built: %s" % e) from e
    if not os.path.exists(path):
        raise ImportError("libabs.so not found at %s (run paper_conf_icpp_yasudonitkyi20_b200/build.py)" % path)
    L = C.CDLL(path)
    P = C.POINTER
    vp = C.c_void_p
    L.abs_config_init.argtypes = [P(abs_config)]
    L.abs_config_init.restype = None
    L.abs_create.argtypes = [P(vp), C.c_int32, vp, P(abs_config)]
    L.abs_create_dev.argtypes = [P(vp), C.c_int32, vp, P(abs_config)]
    L.abs_seed_pool.argtypes = [vp, vp, C.c_int32]
    L.abs_search.argtypes = [vp, C.c_int64]
    L.abs_best.argtypes = [vp, vp, P(C.c_int64)]
    L.abs_stats_get.argtypes = [vp, P(abs_stats)]
    L.abs_pool_get.argtypes = [vp, C.c_int32, vp, vp, P(C.c_int32)]
    L.abs_pool_insert.argtypes = [vp, vp, vp, C.c_int32, P(C.c_int32)]
    L.abs_energy.argtypes = [vp, vp, C.c_int32, vp, vp]
    if hasattr(L, "abs_energy_dev") or not os.environ.get("ABS_LIB"):
        L.abs_energy_dev.argtypes = [vp, vp, C.c_int32, vp, vp, C.c_int32]
    L.abs_round_results.argtypes = [vp, vp, vp]
    L.abs_round_targets.argtypes = [vp, vp]
    L.abs_trace_count.argtypes = [vp, P(C.c_int64)]
    L.abs_debug_timing.argtypes = [vp, vp]
    L.abs_trace_get.argtypes = [vp, C.c_int64, P(C.c_int32), P(C.c_int32), vp, vp, P(C.c_int64)]
    L.abs_search_state.argtypes = [vp, C.c_int32, vp, vp, P(C.c_int64), P(C.c_int32), P(C.c_int32),
                                   P(C.c_uint64), P(C.c_int64)]
    L.abs_destroy.argtypes = [vp]
    L.abs_destroy.restype = None
    L.abs_strerror.argtypes = [C.c_int]
    L.abs_strerror.restype = C.c_char_p
    L.abs_last_error.argtypes = []
    L.abs_last_error.restype = C.c_char_p
    if hasattr(L, "abs_device_searches") or not os.environ.get("ABS_LIB"):  # older diagnostics builds lack it
        L.abs_device_searches.argtypes = [C.c_int32, C.c_int32, P(C.c_int32)]
    if hasattr(L, "abs_ising_to_qubo") or not os.environ.get("ABS_LIB"):
        L.abs_ising_to_qubo.argtypes = [C.c_int32, vp, vp, vp, P(C.c_int64)]
        L.abs_qubo_to_ising.argtypes = [C.c_int32, vp, vp, vp, P(C.c_int64)]
    if hasattr(L, "abs_random_qubo_dev") or not os.environ.get("ABS_LIB"):
        L.abs_random_qubo_dev.argtypes = [C.c_int32, C.c_uint64, vp, C.c_int32]
    L.abs_version.argtypes = []
    L.abs_version.restype = C.c_char_p
    for name in EXPORTS:
        if os.environ.get("ABS_LIB") and not hasattr(L, name):
            continue
        fn = getattr(L, name)
        if fn.restype is C.c_int:  # default restype
            fn.restype = C.c_int
    _lib = L
    return L


def _strerror(rc: int) -> str:
    try:
        return load(False).abs_strerror(rc).decode()
    except Exception:
        return "error"


def _check(rc: int, where: str):
    if rc != ABS_OK:
        raise AbsError(rc, where, load().abs_last_error().decode())


def _ptr(a):
    return None if a is None else C.c_void_p(a.ctypes.data)


INIT_AUTO, INIT_ALU, INIT_MMA = 0, 1, 2  # batched-init engines (include/abs.h)


def words(n: int) -> int:
    return (int(n) + 31) // 32


def make_config(n: int, searches: int = 148, search_offset: int = 0, local_flips: int | None = None,
                pool_size: int = 64, ladder=None, seed: int = 1, p_cross: int = -1, p_mut: int = -1,
                mut_max: int = 0, mode: int = MODE_LOCKSTEP, external_merge: bool = False,
                device: int = -1, trace: bool = False, policy: int = POLICY_WINDOW, sa_tau_min: int = 0,
                sa_tau_max: int = 0, sa_levels: int = 0) -> abs_config:
    cfg = abs_config()
    load().abs_config_init(C.byref(cfg))
    cfg.searches = int(searches)
    cfg.search_offset = int(search_offset)
    cfg.local_flips = 0 if local_flips is None else int(local_flips)
    cfg.pool_size = int(pool_size)
    lad = list(ladder or [])
    if len(lad) > ABS_LADDER_MAX:
        raise ValueError("ladder too long")
    cfg.ladder_len = len(lad)
    for i, v in enumerate(lad):
        cfg.ladder[i] = int(v)
    cfg.seed = int(seed) & 0xFFFFFFFFFFFFFFFF
    cfg.p_cross = int(p_cross)
    cfg.p_mut = int(p_mut)
    cfg.mut_max = int(mut_max)
    cfg.mode = int(mode)
    cfg.external_merge = 1 if external_merge else 0
    cfg.device = int(device)
    cfg.trace = 1 if trace else 0
    cfg.policy = int(policy)
    cfg.sa_tau_min = int(sa_tau_min)
    cfg.sa_tau_max = int(sa_tau_max)
    cfg.sa_levels = int(sa_levels)
    return cfg


class Solver:
    """One abs_ctx (one GPU / rank).  W: numpy int16 [n, n] (host) or a CUDA
    torch.int16 tensor (device; abs_create_dev)."""

    def __init__(self, W, **cfg_kwargs):
        L = load()
        self._c = C.c_void_p()
        if hasattr(W, "is_cuda") and W.is_cuda:
            import torch
            assert W.dtype == torch.int16 and W.dim() == 2 and W.shape[0] == W.shape[1]
            W = W.contiguous()
            n = int(W.shape[0])
            cfg_kwargs.setdefault("device", W.device.index if W.device.index is not None else torch.cuda.current_device())
            self.cfg = make_config(n, **cfg_kwargs)
            torch.cuda.synchronize(W.device)
            _check(L.abs_create_dev(C.byref(self._c), n, C.c_void_p(W.data_ptr()), C.byref(self.cfg)), "abs_create_dev")
        else:
            W = np.ascontiguousarray(W, dtype=np.int16)
            if W.ndim != 2 or W.shape[0] != W.shape[1]:
                raise ValueError("W must be square")
            n = int(W.shape[0])
            self.cfg = make_config(n, **cfg_kwargs)
            _check(L.abs_create(C.byref(self._c), n, _ptr(W), C.byref(self.cfg)), "abs_create")
        self.n = n
        self.words = words(n)
        st = self.stats()
        self.searches = st["searches"]

    # -- lifecycle
    def close(self):
        if self._c:
            load().abs_destroy(self._c)
            self._c = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # -- calls
    def seed_pool(self, X=None):
        if X is None:
            _check(load().abs_seed_pool(self._c, None, 0), "abs_seed_pool")
        else:
            X = np.ascontiguousarray(np.atleast_2d(X), dtype=np.uint32)
            assert X.shape[1] == self.words
            _check(load().abs_seed_pool(self._c, _ptr(X), X.shape[0]), "abs_seed_pool")

    def search(self, steps: int):
        _check(load().abs_search(self._c, int(steps)), "abs_search")

    def best(self):
        X = np.zeros(self.words, np.uint32)
        E = C.c_int64()
        _check(load().abs_best(self._c, _ptr(X), C.byref(E)), "abs_best")
        return X, int(E.value)

    def stats(self) -> dict:
        s = abs_stats()
        _check(load().abs_stats_get(self._c, C.byref(s)), "abs_stats_get")
        return {k: getattr(s, k) for k, _ in abs_stats._fields_}

    def pool(self, k: int):
        X = np.zeros((k, self.words), np.uint32)
        E = np.zeros(k, np.int64)
        cnt = C.c_int32()
        _check(load().abs_pool_get(self._c, int(k), _ptr(X), _ptr(E), C.byref(cnt)), "abs_pool_get")
        return X[:cnt.value], E[:cnt.value]

    def pool_insert(self, X, E) -> int:
        X = np.ascontiguousarray(np.atleast_2d(X), dtype=np.uint32)
        E = np.ascontiguousarray(np.atleast_1d(E), dtype=np.int64)
        assert X.shape[0] == E.shape[0] and X.shape[1] == self.words
        ins = C.c_int32()
        _check(load().abs_pool_insert(self._c, _ptr(X), _ptr(E), X.shape[0], C.byref(ins)), "abs_pool_insert")
        return int(ins.value)

    def energy(self, X, want_delta: bool = False):
        X = np.ascontiguousarray(np.atleast_2d(X), dtype=np.uint32)
        assert X.shape[1] == self.words
        cnt = X.shape[0]
        E = np.zeros(cnt, np.int64)
        D = np.zeros((cnt, self.n), np.int32) if want_delta else None
        _check(load().abs_energy(self._c, _ptr(X), cnt, _ptr(E), _ptr(D)), "abs_energy")
        return (E, D) if want_delta else E

    def energy_dev(self, X, E, D=None, engine: int = INIT_AUTO) -> float:
        """abs_energy_dev on CUDA torch tensors: X int32/uint32-bit words
        [count, words], E int64 [count] (written), D int32 [count, n] or None.
        Returns the device time of the launch (seconds, CUDA events)."""
        import torch
        assert X.is_cuda and X.dtype == torch.int32 and X.shape[1] == self.words and X.is_contiguous()
        cnt = int(X.shape[0])
        assert E.is_cuda and E.dtype == torch.int64 and E.numel() >= cnt
        if D is not None:
            assert D.is_cuda and D.dtype == torch.int32 and D.is_contiguous() and D.numel() >= cnt * self.n
        torch.cuda.synchronize(X.device)
        _check(load().abs_energy_dev(self._c, C.c_void_p(X.data_ptr()), cnt, C.c_void_p(E.data_ptr()),
                                     None if D is None else C.c_void_p(D.data_ptr()), int(engine)), "abs_energy_dev")
        return float(self.stats()["init_seconds"])

    def round_results(self):
        B = np.zeros((self.searches, self.words), np.uint32)
        EB = np.zeros(self.searches, np.int64)
        _check(load().abs_round_results(self._c, _ptr(B), _ptr(EB)), "abs_round_results")
        return B, EB

    def round_targets(self):
        T = np.zeros((self.searches, self.words), np.uint32)
        _check(load().abs_round_targets(self._c, _ptr(T)), "abs_round_targets")
        return T

    def debug_timing(self):
        """Diagnostics build only: int64 [searches, 32, 8] cycle accumulators."""
        out = np.zeros((self.searches, 32, 24), np.int64)
        _check(load().abs_debug_timing(self._c, _ptr(out)), "abs_debug_timing")
        return out

    def trace(self):
        """Async trace: list of (search, round, T, B, E_B) in arrival order."""
        cnt = C.c_int64()
        _check(load().abs_trace_count(self._c, C.byref(cnt)), "abs_trace_count")
        out = []
        for i in range(cnt.value):
            s, r, EB = C.c_int32(), C.c_int32(), C.c_int64()
            T = np.zeros(self.words, np.uint32)
            B = np.zeros(self.words, np.uint32)
            _check(load().abs_trace_get(self._c, i, C.byref(s), C.byref(r), _ptr(T), _ptr(B), C.byref(EB)),
                   "abs_trace_get")
            out.append((s.value, r.value, T, B, int(EB.value)))
        return out

    def search_state(self, s: int) -> dict:
        X = np.zeros(self.words, np.uint32)
        D = np.zeros(self.n, np.int32)
        E, a, l, h, f = C.c_int64(), C.c_int32(), C.c_int32(), C.c_uint64(), C.c_int64()
        _check(load().abs_search_state(self._c, int(s), _ptr(X), _ptr(D), C.byref(E), C.byref(a), C.byref(l),
                                       C.byref(h), C.byref(f)), "abs_search_state")
        return dict(X=X, D=D, E=int(E.value), a=int(a.value), l=int(l.value), hash=int(h.value), flips=int(f.value))


def ising_to_qubo(J, h):
    """Ising (J, h) of P:L40 -> (W int16 [n, n], offset) with H(S) = E(X) + offset,
    s_i = 2 x_i - 1.  Only the upper triangle of J is read."""
    J = np.ascontiguousarray(J, dtype=np.int32)
    h = np.ascontiguousarray(h, dtype=np.int32)
    n = h.shape[0]
    if J.shape != (n, n):
        raise ValueError("J must be n x n")
    W = np.zeros((n, n), np.int16)
    off = C.c_int64()
    _check(load().abs_ising_to_qubo(n, _ptr(J), _ptr(h), _ptr(W), C.byref(off)), "abs_ising_to_qubo")
    return W, int(off.value)


def qubo_to_ising(W):
    """W -> (2J, 2h, 2*offset) exactly (integers): the Ising form of Eq.(1)
    with H(S) = E(X) + offset."""
    W = np.ascontiguousarray(W, dtype=np.int16)
    n = W.shape[0]
    J2 = np.zeros((n, n), np.int32)
    h2 = np.zeros(n, np.int32)
    off2 = C.c_int64()
    _check(load().abs_qubo_to_ising(n, _ptr(W), _ptr(J2), _ptr(h2), C.byref(off2)), "abs_qubo_to_ising")
    return J2, h2, int(off2.value)


def device_searches(n: int, device: int = 0) -> int:
    """Searches that fill `device` in one wave for an n-bit instance."""
    out = C.c_int32()
    _check(load().abs_device_searches(int(n), int(device), C.byref(out)), "abs_device_searches")
    return int(out.value)


def random_qubo_dev(W, seed: int = 1):
    """Fill the CUDA int16 tensor W [n, n] with the synthetic random QUBO of
    abs_random_qubo_dev, generated on W's device."""
    assert W.is_cuda and str(W.dtype) == "torch.int16" and W.dim() == 2 and W.shape[0] == W.shape[1]
    assert W.is_contiguous()
    _check(load().abs_random_qubo_dev(int(W.shape[0]), C.c_uint64(int(seed) & 0xFFFFFFFFFFFFFFFF),
                                      C.c_void_p(W.data_ptr()), int(W.device.index)), "abs_random_qubo_dev")
    return W


def version() -> str:
    return load().abs_version().decode()
