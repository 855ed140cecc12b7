"""Small driver for ncu: a few lockstep steps of the round kernel."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_yasudonitkyi20_b200 as pkg  # noqa: E402
from workloads import random_qubo, maxcut_qubo  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=32768)
ap.add_argument("--searches", type=int, default=148)
ap.add_argument("--L", type=int, default=2048)
ap.add_argument("--steps", type=int, default=2)
ap.add_argument("--maxcut", action="store_true")
a = ap.parse_args()
torch.cuda.set_device(0)
W = maxcut_qubo(a.n, 10 * a.n, seed=1) if a.maxcut else random_qubo(a.n, 1)
Wd = torch.from_numpy(W).cuda()
s = pkg.Solver(Wd, searches=a.searches, local_flips=a.L, pool_size=64, seed=1)
s.search(a.steps)
st = s.stats()
print({k: st[k] for k in ("flips", "straight_flips", "search_seconds", "round_kernel_launches")})
print("flips/s per GPU %.3e  solutions/s %.3e" % (st["flips"] / st["search_seconds"], st["flips"] * a.n / st["search_seconds"]))
