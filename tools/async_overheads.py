"""Async-mode per-item overheads (needs ABS_LIB=.../libabs_timing.so): cycles
thread 0 spends per round waiting for the previous round (queue mode), for the
host's acknowledgement (rack backpressure), reading the target version, and
publishing the result; plus the round's flip-loop cycles for scale."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_icpp_yasudonitkyi20_b200 as pkg
from workloads import random_qubo
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1024
S = int(sys.argv[2]) if len(sys.argv) > 2 else 4736
Lm = int(sys.argv[3]) if len(sys.argv) > 3 else 1
W = torch.from_numpy(random_qubo(n, 1)).cuda()
s = pkg.Solver(W, searches=S, local_flips=Lm * n, pool_size=64, seed=1, mode=pkg.MODE_ASYNC)
s.search(5)
T = s.debug_timing().astype(np.float64)
items = T[:, 0, 20].sum()
st = s.stats()
out = {"n": n, "S": S, "L": Lm * n, "items": items,
       "cyc_per_item": {k: round(T[:, 0, i].sum() / items, 1) for k, i in
                        (("wait_prev", 16), ("wait_rack", 17), ("read_tver", 18), ("publish", 19))},
       "round_cycles_per_item": round(T[:, 0, 0:6].sum() / items + T[:, 0, 8:14].sum() / items, 1),
       "sol_per_s": st["flips"] * n / st["search_seconds"]}
print(json.dumps(out))
