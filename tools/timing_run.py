"""Per-phase cycle accounting of the round kernel (needs libabs_timing.so:
python paper_conf_icpp_yasudonitkyi20_b200/build.py --timing; run with
ABS_LIB=paper_conf_icpp_yasudonitkyi20_b200/libabs_timing.so)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_icpp_yasudonitkyi20_b200 as pkg
from workloads import maxcut_qubo, random_qubo, tsp_qubo
n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
kind = sys.argv[5] if len(sys.argv) > 5 else "random"
lad = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 and sys.argv[2] else None
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 4
S = int(sys.argv[4]) if len(sys.argv) > 4 else pkg.device_searches(n)
Wh = {"random": lambda: random_qubo(n, 1), "maxcut": lambda: maxcut_qubo(n, int(round(9.995 * n)), seed=1),
      "tsp": lambda: tsp_qubo(int(round(n ** 0.5)), seed=1)}[kind]()
n = Wh.shape[0]
W = torch.from_numpy(Wh).cuda()
s = pkg.Solver(W, searches=S, local_flips=n, pool_size=64, seed=1, ladder=lad)
s.search(1)
t0 = s.debug_timing().astype(np.float64)
s.search(steps)
T = s.debug_timing().astype(np.float64) - t0   # steady-state rounds only
nw = s.stats()["threads_per_search"] // 32
T = T[:, :nw, :]
names = ["window", "row_wait", "row_update", "publish_book", "reduce_barrier", "tail"]
out = {"n": n, "kind": kind, "ladder": lad, "searches": S}
for kind, o in (("local", 0), ("straight", 8)):
    fl = T[:, :, o + 6]
    if fl.sum() == 0:
        continue
    out[kind] = {
        "flips_per_search": float(fl[:, 0].sum() / T.shape[0]),
        "row_warps": {nm: round(float(T[:, :-1, o + i].sum() / fl[:, :-1].sum()), 1) for i, nm in enumerate(names)}
        if nw > 1 else None,
        "control_warp": {nm: round(float(T[:, -1, o + i].sum() / fl[:, -1].sum()), 1) for i, nm in enumerate(names)},
    }
if T[:, :, 14].sum() > 0:  # straight flips that improved E_B (control warp's count)
    fl = T[:, -1, 14].sum()
    out["straight_improve"] = {"fraction": float(T[:, -1, 7].sum() / fl),
                               "fraction_neighbour": float(T[:, -1, 15].sum() / fl)}
if T[:, -1, 20].sum() > 0 and T[:, -1, 21].sum() > 0:  # certain window selections (prefetch path)
    out["certain_selection_fraction"] = float(T[:, -1, 21].sum() / T[:, -1, 20].sum())
sub = T[:, -1, 16:21]
if sub[:, 4].sum() > 0:
    out["selection_subphases"] = {nm: round(float(sub[:, i].sum() / sub[:, 4].sum()), 1) for i, nm in
                                  enumerate(["wait_row_half", "arith", "reduce", "issue"])}
print(json.dumps(out, indent=1))
