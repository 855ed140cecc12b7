"""Time of the FIRST lockstep step of a fresh solver at n = 32768 (592 searches, L = n):
round 0 walks from X = 0 to a random target, so it is dominated by the straight
search (Alg. 5).  A/B helper for straight-phase changes: ABS_LIB selects the library."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_yasudonitkyi20_b200 as pkg
n = 32768
torch.cuda.set_device(0)
Wd = torch.empty((n, n), dtype=torch.int16, device="cuda:0")
pkg.random_qubo_dev(Wd, 1)
for rep in range(2):
    s = pkg.Solver(Wd, searches=592, local_flips=n, pool_size=64, seed=1 + rep)
    st0 = s.stats()
    torch.cuda.synchronize()
    t = time.perf_counter()
    s.search(1)
    torch.cuda.synchronize()
    dt = time.perf_counter() - t
    st = s.stats()
    print(json.dumps({"lib": os.environ.get("ABS_LIB", "libabs.so").split("/")[-1], "rep": rep, "ms": 1e3 * dt,
                      "flips": st["flips"], "straight": st["straight_flips"],
                      "kernel_ms": 1e3 * (st["search_seconds"] - st0["search_seconds"])}))
    s.close()
