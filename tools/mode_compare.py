"""Lockstep vs async on one instance: flips per round, straight share, device seconds (diagnostic)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_yasudonitkyi20_b200 as pkg
from workloads import random_qubo
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
S = int(sys.argv[2]) if len(sys.argv) > 2 else 10000
Lm = int(sys.argv[3]) if len(sys.argv) > 3 else 1
W = torch.from_numpy(random_qubo(n, 1)).cuda()
for mode in (pkg.MODE_LOCKSTEP, pkg.MODE_ASYNC):
    s = pkg.Solver(W, searches=S, local_flips=Lm * n, pool_size=64, seed=1, mode=mode)
    s.search(3)
    a = s.stats()
    s.search(5)
    b = s.stats()
    d = {k: b[k] - a[k] for k in ("flips", "straight_flips", "rounds", "search_seconds", "step_seconds")}
    d["mode"] = "async" if mode == pkg.MODE_ASYNC else "lockstep"
    d["flips_per_round"] = d["flips"] / d["rounds"]
    d["straight_frac"] = d["straight_flips"] / d["flips"]
    d["sol_per_s"] = d["flips"] * n / d["search_seconds"]
    d["us_per_round_slot"] = d["search_seconds"] * 1e6 / d["rounds"]
    print(json.dumps(d))
    s.close()
