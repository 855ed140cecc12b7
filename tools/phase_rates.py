"""Throughput vs local-search length L at fixed n (lockstep), to separate the
cost of straight-search flips from local flips (diagnostic)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_yasudonitkyi20_b200 as pkg
from workloads import random_qubo
n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
W = torch.from_numpy(random_qubo(n, 1)).cuda()
for mult in (1, 4, 8):
    s = pkg.Solver(W, searches=148, local_flips=mult * n, pool_size=64, seed=1)
    s.search(2)
    st0 = s.stats()
    s.search(2)
    st1 = s.stats()
    fl = st1["flips"] - st0["flips"]; sf = st1["straight_flips"] - st0["straight_flips"]
    t = st1["search_seconds"] - st0["search_seconds"]
    print(json.dumps({"L": mult * n, "sol_per_s": fl * n / t, "straight_frac": sf / fl, "s": t}))
    s.close()
