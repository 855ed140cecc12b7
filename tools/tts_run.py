"""Time-to-solution runs (Table 1 analogue) on synthetic
instances: Max-Cut G(n, m) graphs (G-set-like sizes), TSP with c random
cities (c^2 bits, reading C13) and random int16 QUBO.

For each instance: a reference run of --ref-seconds gives the "best-known"
value ("we compute good solutions by repeating searches until
convergence and regard them as best-known"); then --repeats fresh runs
(other seeds) measure the wall time until the pool reaches --fraction of it
(cut >= f * best cut; energy <= f * best energy; a valid tour no longer than
best / f).  One JSON line per run.  Multi-GPU: launch with torchrun; ranks
exchange elites after every call and agree on success (tts.py).

  python tools/tts_run.py --workload maxcut --n 2000 --edges 19990 --fraction 0.99
  python tools/tts_run.py --workload tsp --cities 29 --fraction 0.95
  python tools/tts_run.py --workload random --n 32768 --fraction 0.99
"""
from __future__ import annotations

import argparse
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_icpp_yasudonitkyi20_b200 as pkg  # noqa: E402
from paper_conf_icpp_yasudonitkyi20_b200 import tts  # noqa: E402
from workloads import maxcut_graph, maxcut_qubo, random_qubo, tsp_instance, tsp_qubo  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", choices=["maxcut", "tsp", "random"], default="maxcut")
    ap.add_argument("--n", type=int, default=2000)
    ap.add_argument("--edges", type=int, default=19990)
    ap.add_argument("--weights", choices=["pm1", "one"], default="pm1")
    ap.add_argument("--cities", type=int, default=16)
    ap.add_argument("--instance-seed", type=int, default=1)
    ap.add_argument("--fraction", type=float, default=0.99)
    ap.add_argument("--also", default="", help="comma list of looser fractions reported from the same runs "
                    "(energy workloads: the first time on the improvement trace each target was met)")
    ap.add_argument("--ref-seconds", type=float, default=20.0)
    ap.add_argument("--max-seconds", type=float, default=20.0)
    ap.add_argument("--repeats", type=int, default=3)
    ap.add_argument("--searches", type=int, default=0)
    ap.add_argument("--local-flips", type=int, default=0)
    ap.add_argument("--mode", choices=["async", "lockstep"], default="async")
    ap.add_argument("--rounds-per-call", type=int, default=1)
    a = ap.parse_args()

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    if a.workload == "maxcut":
        ei, ej, w = maxcut_graph(a.n, a.edges, seed=a.instance_seed, weights=a.weights)
        W = maxcut_qubo(a.n, a.edges, seed=a.instance_seed, weights=a.weights)
        desc = {"workload": "maxcut", "n": a.n, "edges": a.edges, "weights": a.weights}
    elif a.workload == "tsp":
        c = a.cities
        _, D = tsp_instance(c, seed=a.instance_seed)
        W = tsp_qubo(c, seed=a.instance_seed)
        desc = {"workload": "tsp", "cities": c, "n": c * c}
    else:
        W = random_qubo(a.n, a.instance_seed)
        desc = {"workload": "random", "n": a.n}
    n = W.shape[0]
    S = a.searches or pkg.device_searches(n, local)
    mode = pkg.MODE_ASYNC if a.mode == "async" else pkg.MODE_LOCKSTEP
    Wd = torch.from_numpy(W).cuda()

    def solver(seed):
        return pkg.Solver(Wd, searches=S, search_offset=rank * S, local_flips=a.local_flips or n,
                          pool_size=64, seed=seed, mode=mode)

    # ---- reference ("best-known") run
    ref = solver(10_000 + a.instance_seed)
    if a.workload == "tsp":
        best_len = [None]

        def note(X, E):
            tour = tts.tsp_tour(X, c)
            if tour is not None:
                L = tts.tour_length(tour, D)
                best_len[0] = L if best_len[0] is None else min(best_len[0], L)
            return False
        r = tts.time_to_target(ref, accept=note, max_seconds=a.ref_seconds, exchange_k=16)
        best_known = best_len[0]
        limit = None if best_known is None else math.floor(best_known / a.fraction)

        def accept(X, E):
            tour = tts.tsp_tour(X, c)
            return tour is not None and tts.tour_length(tour, D) <= limit
        target = {"tour_length_le": limit}
    else:
        r = tts.time_to_target(ref, target_energy=-(2 ** 62), max_seconds=a.ref_seconds, exchange_k=16)
        best_E = r.best_energy
        if world > 1:
            import torch.distributed as dist
            t = torch.tensor([best_E], dtype=torch.int64, device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MIN)
            best_E = int(t.item())
        if a.workload == "maxcut":
            best_known = -best_E
            e_target = tts.cut_target(best_known, a.fraction)
            target = {"cut_ge": -e_target}
        else:
            best_known = best_E
            e_target = tts.energy_target(best_known, a.fraction)
            target = {"energy_le": e_target}
        accept = None
    st = ref.stats()
    ref.close()
    if rank == 0:
        print(json.dumps({**desc, "phase": "reference", "seconds": a.ref_seconds, "best_known": best_known,
                          "searches_per_gpu": S, "gpus": world, "mode": a.mode,
                          "ref_solutions_per_s": st["flips"] * n / max(st["search_seconds"], 1e-9)}), flush=True)
    if best_known is None:
        return

    for rep in range(a.repeats):
        s = solver(1 + rep)
        if accept is not None:
            r = tts.time_to_target(s, accept=accept, max_seconds=a.max_seconds, exchange_k=16,
                                   rounds_per_call=a.rounds_per_call)
        else:
            r = tts.time_to_target(s, target_energy=e_target, max_seconds=a.max_seconds, exchange_k=16,
                                   rounds_per_call=a.rounds_per_call)
        s.close()
        if rank == 0:
            line = {**desc, "phase": "tts", "repeat": rep, "fraction": a.fraction, "target": target,
                    "reached": r.reached, "seconds": r.seconds, "best_energy": r.best_energy,
                    "calls": r.calls, "gpus": world}
            if a.also and a.workload != "tsp":
                also = {}
                for f in sorted(float(v) for v in a.also.split(",")):
                    et = tts.cut_target(best_known, f) if a.workload == "maxcut" else tts.energy_target(best_known, f)
                    hit = [t for t, E in r.trace if E <= et]
                    also[str(f)] = hit[0] if hit else None
                line["seconds_at_fraction"] = also
            print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
