"""Small driver for ncu / quick timing: a few lockstep steps of the round kernel.
Prints per-step flip counts (one round-kernel launch per step) as JSON lines so
that an ncu capture of launch #i can be normalised per flip."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_yasudonitkyi20_b200 as pkg  # noqa: E402
from workloads import maxcut_qubo, random_qubo, tsp_qubo  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n", type=int, default=32768)
ap.add_argument("--searches", type=int, default=148)
ap.add_argument("--L", type=int, default=0)
ap.add_argument("--steps", type=int, default=2)
ap.add_argument("--workload", default="random", choices=["random", "maxcut", "tsp"])
a = ap.parse_args()
torch.cuda.set_device(0)
if a.workload == "maxcut":
    W = maxcut_qubo(a.n, 10 * a.n, seed=1)
elif a.workload == "tsp":
    W = tsp_qubo(int(round(a.n ** 0.5)), seed=1)
else:
    W = random_qubo(a.n, 1)
n = W.shape[0]
Wd = torch.from_numpy(W).cuda()
s = pkg.Solver(Wd, searches=a.searches, local_flips=a.L or n, pool_size=64, seed=1)
prev = s.stats()
for i in range(a.steps):
    s.search(1)
    st = s.stats()
    d = {k: st[k] - prev[k] for k in ("flips", "straight_flips", "search_seconds")}
    d["launch"] = i
    d["solutions_per_s"] = d["flips"] * n / d["search_seconds"]
    print(json.dumps(d))
    prev = st
st = s.stats()
print(json.dumps({"total_flips": st["flips"], "straight": st["straight_flips"], "kernel_s": st["search_seconds"],
                  "solutions_per_s": st["flips"] * n / st["search_seconds"]}))
