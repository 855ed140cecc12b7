"""Parity of the batched initialisation engines (SURVEY §8(a) row a2, §8(f)
row 3) through the C ABI (abs_energy_dev): the tensor-core engine
(tcgen05.mma kind::i8, W split exactly into int8 planes) and the ALU engine
against the oracle's Eq.(13) / Eq.(1) (oracle.init_batch), element by
element.  Sizes span several 128 x 128 output tiles with ragged tails in
both the solution (M) and field (N) directions; the int8 split is checked
on the values where hi / lo carry (W = -1, -256, 255, 256, +-32767,
-32768) and on the largest |Delta| (reading C12)."""
from __future__ import annotations

import time

import numpy as np
import pytest

import oracle
from workloads import pack_bits, random_qubo, random_solutions

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icpp_yasudonitkyi20_b200 as abs_b200  # noqa: E402

ENGINES = [abs_b200.INIT_MMA, abs_b200.INIT_ALU]


def run_dev(s, X, engine, want_delta=True):
    Xd = torch.from_numpy(np.ascontiguousarray(X).view(np.int32)).cuda()
    E = torch.zeros(X.shape[0], dtype=torch.int64, device="cuda")
    D = torch.zeros((X.shape[0], s.n), dtype=torch.int32, device="cuda") if want_delta else None
    s.energy_dev(Xd, E, D, engine)
    return E.cpu().numpy(), (D.cpu().numpy() if want_delta else None)


@pytest.mark.parametrize("engine", ENGINES)
@pytest.mark.parametrize("n,count", [(1, 3), (16, 256), (100, 129), (1000, 300), (1024, 128),
                                     (1500, 257), (2050, 130), (5000, 200)])
def test_init_engines_match_oracle(engine, n, count):
    W = random_qubo(n, 100 + n)
    X = random_solutions(count, n, 7 + n)
    X[0] = 0
    X[min(1, count - 1)] = pack_bits(np.ones((1, n), bool))[0]
    s = abs_b200.Solver(W, searches=1)
    Xdirty = X.copy()
    if n % 32:  # bits >= n must be ignored
        Xdirty[:, -1] |= np.uint32(~((1 << (n % 32)) - 1) & 0xFFFFFFFF)
    E, D = run_dev(s, Xdirty, engine)
    oD, oE = oracle.init_batch(W, X)
    assert (E == oE).all()
    assert (D.astype(np.int64) == oD).all()
    s.close()


@pytest.mark.parametrize("engine", ENGINES)
def test_init_int8_split_carry_values(engine):
    """Entries where the exact split W = 256 hi + lo carries or saturates."""
    n = 640
    rng = np.random.default_rng(3)
    vals = np.array([-32768, -32767, -257, -256, -255, -129, -128, -1, 0, 1, 127, 128, 255, 256, 257, 32511,
                     32512, 32767], np.int16)
    U = rng.choice(vals, size=(n, n))
    W = np.triu(U) + np.triu(U, 1).T
    X = random_solutions(200, n, 11)
    s = abs_b200.Solver(W, searches=1)
    E, D = run_dev(s, X, engine)
    oD, oE = oracle.init_batch(W, X)
    assert (E == oE).all() and (D.astype(np.int64) == oD).all()


@pytest.mark.parametrize("engine", ENGINES)
@pytest.mark.parametrize("v", [-32768, 32767])
def test_init_extreme_magnitudes(engine, v):
    # reading C12: W == -32768, X = 1^n -> Delta_i = 32768 (2n - 1), the largest |Delta|
    n = 4096
    W = np.full((n, n), v, np.int16)
    s = abs_b200.Solver(W, searches=1)
    X = np.full((130, n // 32), 0xFFFFFFFF, np.uint32)
    X[129] = 0
    E, D = run_dev(s, X, engine)
    assert (D[:129] == -v * (2 * n - 1)).all() and (E[:129] == v * n * n).all()
    assert (D[129] == v).all() and E[129] == 0


def test_init_full_size_n32768_sampled():
    """n = 32768 (config 5), 300 solutions (3 M tiles, ragged): sampled rows
    against the oracle; every row identical between the two engines."""
    n, count = 32768, 300
    W = random_qubo(n, 1)
    X = random_solutions(count, n, 9)
    s = abs_b200.Solver(W, searches=1)
    t0 = time.time()
    E, D = run_dev(s, X, abs_b200.INIT_MMA)
    E2, D2 = run_dev(s, X, abs_b200.INIT_ALU)
    assert (E == E2).all() and (D == D2).all()
    for b in (0, 173, 299):
        oD, oE = oracle.init_batch(W, X[b:b + 1])
        assert E[b] == oE[0] and (D[b].astype(np.int64) == oD[0]).all()
    assert time.time() - t0 < 600


def test_init_energy_only_and_host_api():
    """abs_energy (host buffers) runs the tensor-core engine; E without Delta."""
    n = 3000
    W = random_qubo(n, 4)
    X = random_solutions(77, n, 4)
    s = abs_b200.Solver(W, searches=1)
    E = s.energy(X)
    E2, _ = run_dev(s, X, abs_b200.INIT_MMA, want_delta=False)
    _, oE = oracle.init_batch(W, X)
    assert (E == oE).all() and (E2 == oE).all()
