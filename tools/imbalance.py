"""Lockstep imbalance at the bench configuration: per-search busy cycles of one
step (control warp, diagnostics build) against the step's kernel time.  Needs
ABS_LIB=.../libabs_timing.so (python paper_conf_icpp_yasudonitkyi20_b200/build.py --timing)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_icpp_yasudonitkyi20_b200 as pkg
from workloads import random_qubo

n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
S = pkg.device_searches(n)
W = torch.from_numpy(random_qubo(n, 1)).cuda()
s = pkg.Solver(W, searches=S, local_flips=n, pool_size=64, seed=1)
s.search(1)
nw = s.stats()["threads_per_search"] // 32
rows = []
for _ in range(steps):
    t0 = s.debug_timing().astype(np.float64)
    f0 = np.array([s.search_state(i)["flips"] for i in range(S)])
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); e0.record()
    s.search(1)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    T = s.debug_timing().astype(np.float64) - t0
    f1 = np.array([s.search_state(i)["flips"] for i in range(S)])
    busy = T[:, nw - 1, 0:6].sum(1) + T[:, nw - 1, 8:14].sum(1)  # cycles per search (control warp)
    st = T[:, nw - 1, 14]
    rows.append(dict(step_ms=ms, busy_ms_max=float(busy.max() / 1965e3), busy_ms_mean=float(busy.mean() / 1965e3),
                     busy_ms_min=float(busy.min() / 1965e3), flips_mean=float((f1 - f0).mean()),
                     flips_max=int((f1 - f0).max()), straight_mean=float(st.mean()), straight_max=int(st.max()),
                     straight_min=int(st.min())))
print(json.dumps(rows, indent=1))
