"""Small lockstep / async runs for compute-sanitizer (memcheck, racecheck,
synccheck): every kernel variant the size selects, both policies.

  compute-sanitizer --tool racecheck python tools/sanitize_run.py --n 1100 --mode async
"""
from __future__ import annotations

import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

import paper_conf_icpp_yasudonitkyi20_b200 as pkg  # noqa: E402
from workloads import random_qubo, random_solutions  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=100)
    ap.add_argument("--mode", default="lockstep", choices=["lockstep", "async"])
    ap.add_argument("--policy", default="window", choices=["window", "sa"])
    ap.add_argument("--searches", type=int, default=3)
    ap.add_argument("--steps", type=int, default=2)
    ap.add_argument("--local-flips", type=int, default=60)
    a = ap.parse_args()
    W = random_qubo(a.n, 11)
    kw = dict(searches=a.searches, local_flips=a.local_flips, pool_size=8, seed=3,
              mode=pkg.MODE_ASYNC if a.mode == "async" else pkg.MODE_LOCKSTEP)
    if a.policy == "sa":
        kw.update(policy=pkg.POLICY_SA, sa_tau_min=2000, sa_tau_max=40000, sa_levels=3)
    s = pkg.Solver(W, **kw)
    s.search(a.steps)
    X, E = s.best()
    Xs = random_solutions(5, a.n, 2)
    Eb = s.energy(Xs)          # batched init (tensor-core engine)
    s.close()
    print("ok n=%d mode=%s policy=%s best=%d batchE0=%d" % (a.n, a.mode, a.policy, E, int(Eb[0])))


if __name__ == "__main__":
    main()
