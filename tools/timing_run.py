"""Per-phase cycle accounting of the round kernel (needs libabs_timing.so:
python paper_conf_icpp_yasudonitkyi20_b200/build.py --timing; run with
ABS_LIB=paper_conf_icpp_yasudonitkyi20_b200/libabs_timing.so)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_icpp_yasudonitkyi20_b200 as pkg
from workloads import random_qubo
n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
lad = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else None
W = torch.from_numpy(random_qubo(n, 1)).cuda()
s = pkg.Solver(W, searches=148, local_flips=n, pool_size=64, seed=1, ladder=lad)
s.search(3)
T = s.debug_timing().astype(np.float64)   # [S][32][8]
nw = s.stats()["threads_per_search"] // 32
T = T[:, :nw, :]
flips = T[:, :, 6]
names = ["window", "row_wait", "row_update", "publish_book", "reduce_barrier", "tail"]
per = {nm: float((T[:, :, i].sum() / flips.sum())) for i, nm in enumerate(names)}
last = {nm: float((T[:, -1, i].sum() / flips[:, -1].sum())) for i, nm in enumerate(names)}
first = {nm: float((T[:, 0, i].sum() / flips[:, 0].sum())) for i, nm in enumerate(names)}
print(json.dumps({"n": n, "ladder": lad, "cycles_per_flip_all_warps": per, "warp0": first, "control_warp": last,
                  "straight_frac": float(T[:, 0, 7].sum() / flips[:, 0].sum())}, indent=1))
