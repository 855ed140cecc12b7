"""Where the end-to-end time of the bench goes besides the steps: abs_create from a
pinned host W (H2D inside) vs from a device W, at n = 32768, with CUDA events."""
import os, sys, time, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_yasudonitkyi20_b200 as pkg

n = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
torch.cuda.set_device(0)
Wd = torch.empty((n, n), dtype=torch.int16, device="cuda:0")
pkg.random_qubo_dev(Wd, 1)
Wh = torch.empty((n, n), dtype=torch.int16, pin_memory=True)
Wh.copy_(Wd)
torch.cuda.synchronize()
for rep in range(3):
    for src in ("host", "device"):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        e0.record()
        s = pkg.Solver(Wh.numpy() if src == "host" else Wd, searches=592, local_flips=n, pool_size=64, seed=1)
        e1.record()
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        s.search(1)
        torch.cuda.synchronize()
        t2 = time.perf_counter()
        X, E = s.best()
        t3 = time.perf_counter()
        s.close()
        torch.cuda.synchronize()
        t4 = time.perf_counter()
        print(json.dumps({"rep": rep, "src": src, "create_ms": 1e3 * (t1 - t0), "create_ev_ms": e0.elapsed_time(e1),
                          "step_ms": 1e3 * (t2 - t1), "best_ms": 1e3 * (t3 - t2), "close_ms": 1e3 * (t4 - t3)}))
