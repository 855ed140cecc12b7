#!/usr/bin/env python
"""Benchmark of the ABS hot path (BASELINE.json metric: searched solutions/s,
n evaluations per flip, at n = 32k on 1/2/4/8 B200).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl abs|reference] [--workload ...]

One step = one pass of the whole hot path over the batch of searches: the
host GA makes one target per search, every search runs one round (straight
search to its target + L window-policy local flips, each flip one W-row
update evaluating n neighbours), the results are inserted into the pool
(multi-GPU: all-gathered over NCCL first).  Inputs are synthetic (Philox
random int16 QUBO); W (2 GiB at n = 32768) exceeds L2, so no flush
is needed between steps.

N > 1: launched by torchrun, one process per GPU; each GPU runs its own
searches (global ids rank*S ... ) on a replicated W (weak scaling) and the
ranks all-gather every step's results so all pools stay identical.

--impl reference: the repository's oracle (oracle/, plain C, the checker of
the parity tests) timed on this host's cores over a bounded sample of the
same workload (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import multiprocessing as mp
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

WORKLOADS = {
    # name: (description, n, generator kwargs)
    "random32k": "random int16 QUBO n=32768 (config 5)",
    "random1k": "random int16 QUBO n=1024, 10k searches (config 2)",
    "maxcut2k": "Max-Cut G(2000, 19990) +-1 weights (config 3)",
    "tsp100": "TSP 100 cities, n=10000 one-hot (config 4)",
}

METRIC = "searched solutions/sec (n evals per flip)"


def make_W(workload: str):
    from workloads import maxcut_qubo, random_qubo, tsp_qubo
    if workload == "random32k":
        return random_qubo(32768, 1)
    if workload == "random1k":
        return random_qubo(1024, 1)
    if workload == "maxcut2k":
        return maxcut_qubo(2000, 19990, seed=1)
    if workload == "tsp100":
        return tsp_qubo(100, seed=1)
    raise ValueError(workload)


# Waves of co-resident searches per step.  A lockstep step ends with its
# slowest search (straight-search lengths differ per target); with several
# waves an SM whose search finishes early starts another.  Measured on one
# B200: random32k 1/2/4/8 waves 2.49/2.52/2.59/2.61e12,
# tsp100 1/4 waves 1.93/2.01e12; maxcut2k already runs 16 searches per SM.
WAVES = {"random32k": 4, "tsp100": 4}


def default_searches(workload: str, n: int, device: int) -> int:
    """Config 2 fixes 10k searches at n=1024; elsewhere WAVES x the searches
    whose CTAs are co-resident on the GPU (148 at n=32k: one 512-thread CTA
    per SM)."""
    if workload == "random1k":
        return 10000
    import paper_conf_icpp_yasudonitkyi20_b200 as pkg
    return WAVES.get(workload, 1) * pkg.device_searches(n, device)


# ------------------------------------------------------------------ clocks
class ClockSampler:
    FIELDS = ["clocks.sm", "clocks.max.sm", "clocks_event_reasons.sw_power_cap",
              "clocks_event_reasons.hw_slowdown", "clocks_event_reasons.hw_thermal_slowdown",
              "clocks_event_reasons.sw_thermal_slowdown", "power.draw"]

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self._stop = threading.Event()
        self._p = None

    def __enter__(self):
        try:
            self._p = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=" + ",".join(self.FIELDS),
                 "--format=csv,noheader,nounits", "-lms", "200"], stdout=subprocess.PIPE,
                stderr=subprocess.DEVNULL, text=True)
            self._t = threading.Thread(target=self._read, daemon=True)
            self._t.start()
        except Exception:
            self._p = None
        return self

    def _read(self):
        for line in self._p.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) == len(self.FIELDS):
                self.rows.append(parts)

    def __exit__(self, *a):
        if self._p:
            self._p.terminate()
            try:
                self._p.wait(timeout=5)
            except Exception:
                self._p.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["sw_power_cap", "hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[2 + i].lower().startswith("active")})
        pw = [float(r[6]) for r in self.rows if r[6].replace(".", "").isdigit()]
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows),
                "power_w_max": max(pw) if pw else None}


# ------------------------------------------------------------------ oracle (cpu baseline / reference arm)
_W_SHARED = None


def _oracle_job(args):
    l, flips, seed = args
    import oracle
    n = _W_SHARED.shape[0]
    T = np.zeros((1, (n + 31) // 32), np.uint32)  # target = start: local flips only
    t = time.perf_counter()
    out = oracle.replay_search(_W_SHARED, l, flips, T)
    return int(out["flips"][0]), time.perf_counter() - t


def oracle_sample(W, procs: int, flips_per_proc: int):
    """Run `procs` oracle searches in parallel (fork; W shared copy-on-write),
    each from the zero vector with `flips_per_proc` window-policy flips.
    Returns (flips, seconds)."""
    global _W_SHARED
    _W_SHARED = W
    import oracle
    oracle.build()
    ctx = mp.get_context("fork")
    t = time.perf_counter()
    with ctx.Pool(procs) as pool:
        res = pool.map(_oracle_job, [(16, flips_per_proc, s) for s in range(procs)])
    dt = time.perf_counter() - t
    return sum(r[0] for r in res), dt


def cpu_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def oracle_flips_for(n: int, seconds: float) -> int:
    # measured oracle cost per flip ~ 35 ns * n (column walk of W) on one core
    return max(50, int(seconds / (35e-9 * n)))


# ------------------------------------------------------------------ arms
def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    W = make_W(args.workload)
    n = W.shape[0]
    procs = min(cpu_cores(), 32)
    flips = oracle_flips_for(n, args.ref_step_seconds)
    for _ in range(args.warmup):
        oracle_sample(W, procs, max(50, flips // 10))
    tot_f, tot_t = 0, 0.0
    for _ in range(args.steps):
        f, dt = oracle_sample(W, procs, flips)
        tot_f += f
        tot_t += dt
    value = tot_f * n / tot_t
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "solutions/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * tot_t / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "int64", "data": "synthetic",
        "config": {"workload": args.workload, "n": n, "desc": WORKLOADS[args.workload],
                   "parallelism": "host processes"},
        "cpu_baseline": {"value": value, "unit": "solutions/s", "cores": procs, "kind": "oracle",
                         "sample": "%d oracle searches in parallel, each %d window-policy flips from X=0 per step"
                                   % (procs, flips)},
        "e2e": {"value": value, "unit": "solutions/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def run_abs(args):
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_yasudonitkyi20_b200 as pkg
    from paper_conf_icpp_yasudonitkyi20_b200 import dist as pdist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # test hooks for exercising the multi-rank flow on a single GPU (both ranks on
    # one device, gloo for the exchange); the driver's runs use the defaults
    local = int(os.environ.get("ABS_BENCH_DEVICE", local))
    backend = os.environ.get("ABS_BENCH_BACKEND", "nccl")
    assert torch.cuda.is_available(), "bench.py needs B200 GPUs"
    torch.cuda.set_device(local)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)

    rdev = "cuda" if backend == "nccl" else "cpu"  # device of the timing reductions

    def barrier():
        if world > 1:
            dist.barrier()

    W = make_W(args.workload)
    n = W.shape[0]
    S = args.searches or default_searches(args.workload, n, local)
    L = args.local_flips or n
    Wp = torch.from_numpy(W).pin_memory()
    Wd = Wp.to(f"cuda:{local}", non_blocking=False)
    mode = pkg.MODE_ASYNC if args.mode == "async" else pkg.MODE_LOCKSTEP
    common = dict(searches=S, local_flips=L, pool_size=64, seed=1, device=local, mode=mode)
    if args.policy == "sa":
        # SA policy (reading E2): a 4-level temperature ladder from the weight scale up
        wmax = int(np.abs(W[:256].astype(np.int32)).max()) or 1  # weight scale from a row sample
        common.update(policy=pkg.POLICY_SA, sa_tau_min=max(1, wmax // 4), sa_tau_max=8 * wmax, sa_levels=4)
    solver = pkg.Solver(Wd, search_offset=rank * S, external_merge=(world > 1 and mode == pkg.MODE_LOCKSTEP),
                        **common)
    del Wd

    def step(s):
        if world > 1:
            pdist.lockstep_step(s)
        else:
            s.search(1)

    def run_steps(s, k):
        if mode == pkg.MODE_ASYNC:
            # one persistent launch for all k rounds of every search (the
            # blocks run asynchronously); ranks then all-gather their elites
            s.search(k)
            if world > 1:
                pdist.exchange_elites(s, 64)
        else:
            for _ in range(k):
                step(s)

    run_steps(solver, args.warmup)
    barrier()
    torch.cuda.synchronize()
    st0 = solver.stats()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        barrier()
        torch.cuda.synchronize()
        ev0.record()
        run_steps(solver, args.steps)
        ev1.record()
        torch.cuda.synchronize()
        barrier()
    st1 = solver.stats()
    ms = ev0.elapsed_time(ev1)
    flips = st1["flips"] - st0["flips"]
    kern_s = st1["search_seconds"] - st0["search_seconds"]
    launches = st1["round_kernel_launches"] - st0["round_kernel_launches"]
    all_launches = st1["kernel_launches"] - st0["kernel_launches"]
    t_ms = torch.tensor([ms], dtype=torch.float64, device=rdev)
    t_fl = torch.tensor([flips], dtype=torch.float64, device=rdev)
    if world > 1:
        dist.all_reduce(t_ms, op=dist.ReduceOp.MAX)
        dist.all_reduce(t_fl, op=dist.ReduceOp.SUM)
    ms_max = float(t_ms.item())
    flips_all = float(t_fl.item())
    value = flips_all * n / (ms_max * 1e-3)

    # roofline of the dominant kernel (the round kernel): algorithmic bytes =
    # one W row (2n bytes) per flip; time = its CUDA-event duration.
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    hbm = float(peaks.get("hbm_gbs", 6650.0))
    peak_src = "measured" if "hbm_gbs" in peaks else "fallback"
    achieved = flips * 2.0 * n / kern_s / 1e9 if kern_s > 0 else None
    # traffic: DRAM bytes per flip of the round kernel from the committed ncu
    # --set full capture (profiles/round_kernel_ncu.json), times this run's flips
    # per launch; only for the workload it was captured on.
    traffic = None
    try:
        prof = json.load(open(os.path.join(ROOT, "profiles", "round_kernel_ncu.json")))
        if args.workload == "random32k" and launches > 0:
            traffic = prof["dram_bytes_per_flip"] * flips / launches / 1e9
    except Exception:
        pass
    roof = {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
            "frac": (achieved / hbm) if achieved else None, "traffic": traffic, "traffic_unit": "GB per launch",
            "peak_source": peak_src, "kernel": "round_kernel",
            "algorithmic_bytes_per_launch": flips * 2.0 * n / max(1, launches),
            "avg_launch_ms": 1e3 * kern_s / max(1, launches),
            "kernel_share_of_step": kern_s / (ms * 1e-3) if ms > 0 else None}
    n_pad = int(st1["n_pad"])
    if 2 * n_pad * n_pad <= 126 * 2 ** 20:
        # W is L2-resident (n <= ~8k): the second roof of SURVEY §8(d) binds, n int32
        # adds per flip against the INT32 pipe: 64 lanes/clk/SM (IMAD/IADD3 issue
        # every 2 cycles per SMSP, B300_MICROARCH "pipe rates") x SMs x max SM clock
        sms = torch.cuda.get_device_properties(local).multi_processor_count
        mhz = float(peaks.get("sm_max_mhz", 1965.0))
        int_peak = sms * 64 * mhz * 1e6 / 1e12
        ach = flips * float(n) / kern_s / 1e12 if kern_s > 0 else None
        roof.update({"bound": "alu", "achieved": ach, "peak": int_peak, "unit": "T int32 adds/s",
                     "frac": (ach / int_peak) if ach else None,
                     "peak_source": "derived: %d SMs x 64 int32 lanes/clk x %.0f MHz" % (sms, mhz),
                     "row_bytes_GBps": achieved})
    solver.close()
    del solver
    torch.cuda.synchronize()

    # ---------------- end to end through the public API with host buffers
    e2e = None
    if not args.no_e2e:
        barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        s2 = pkg.Solver(Wp.numpy(), search_offset=rank * S,
                        external_merge=(world > 1 and mode == pkg.MODE_LOCKSTEP), **common)
        run_steps(s2, args.steps)
        Xb, Eb = s2.best() if world == 1 else (None, None)
        e1.record()
        torch.cuda.synchronize()
        st2 = s2.stats()
        s2.close()
        ems = e0.elapsed_time(e1)
        t2 = torch.tensor([ems], dtype=torch.float64, device=rdev)
        f2 = torch.tensor([st2["flips"]], dtype=torch.float64, device=rdev)
        if world > 1:
            dist.all_reduce(t2, op=dist.ReduceOp.MAX)
            dist.all_reduce(f2, op=dist.ReduceOp.SUM)
        e2e = {"value": float(f2.item()) * n / (float(t2.item()) * 1e-3), "unit": "solutions/s",
               "h2d_bytes_per_step": st2["h2d_bytes"] / args.steps,
               "d2h_bytes_per_step": (st2["d2h_bytes"] + 8 * ((n + 31) // 32)) / args.steps,
               "includes": "abs_create from pinned host W (H2D 2n^2 bytes) + steps + abs_best"}

    # ---------------- cpu baseline (oracle), rank 0 at N = 1 only
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        procs = min(cpu_cores(), 32)
        fl = oracle_flips_for(n, args.cpu_seconds)
        f, dt = oracle_sample(W, procs, fl)
        cpu = {"value": f * n / dt, "unit": "solutions/s", "cores": procs, "kind": "oracle",
               "sample": "%d oracle searches in parallel, %d window-policy flips each from X=0 (%.1f s)"
                         % (procs, fl, dt)}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "solutions/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_max / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic (Philox random int16 QUBO, P:L468)" if args.workload.startswith("random")
            else "synthetic",
            "config": {"workload": args.workload, "desc": WORKLOADS[args.workload], "n": n,
                       "searches_per_gpu": S, "local_flips": L, "pool": 64, "mode": args.mode, "policy": args.policy,
                       "parallelism": "dp%d (replicated W, independent searches)" % world,
                       "l2": "inputs larger than L2 (W = %d MiB)" % (2 * n * n >> 20)
                       if 2 * n * n > 126 * 2 ** 20 else "W fits in L2 (resident by design)"},
            "flips_per_step": flips_all / args.steps,
            "roofline": roof,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": int(all_launches),
            "clocks": clk.summary(),
            "paper_context": "1.24e12 solutions/s on 4x RTX 2080 Ti at n=1024; 4.39e11 at n=32768 (P:L529, P:L544)",
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="abs", choices=["abs", "reference"])
    ap.add_argument("--workload", default="random32k", choices=sorted(WORKLOADS))
    ap.add_argument("--searches", type=int, default=0)
    ap.add_argument("--mode", default="lockstep", choices=["lockstep", "async"])
    ap.add_argument("--policy", default="window", choices=["window", "sa"])
    ap.add_argument("--local-flips", type=int, default=0)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--ref-step-seconds", type=float, default=8.0)
    args = ap.parse_args()
    if args.warmup < 3:
        print("warning: --warmup < 3 violates the timing rules", file=sys.stderr)
    if args.impl == "reference":
        return run_reference(args)
    return run_abs(args)


if __name__ == "__main__":
    sys.exit(main())
