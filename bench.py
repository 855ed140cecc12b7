#!/usr/bin/env python
"""Benchmark of the ABS hot path (BASELINE.json metric: searched solutions/s,
n evaluations per flip, at n = 32k on 1/2/4/8 B200).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl abs|reference] [--workload ...]

One step = one pass of the whole hot path over the batch of searches: the
host GA makes one target per search, every search runs one round (straight
search to its target + L window-policy local flips, each flip one W-row
update evaluating n neighbours), the results are inserted into the pool
(multi-GPU: all-gathered over NCCL first).  Inputs are synthetic: the random
QUBO is generated on each GPU by the library's counter-based rule
(abs_random_qubo_dev; workloads.random_qubo_ctr is its host copy, used by the
oracle); W (2 GiB at n = 32768) exceeds L2, so no flush is needed between
steps.

--gpus N > 1: one process per GPU.  Launched by the driver under torchrun;
run directly, bench.py re-executes itself under torch.distributed.run.  Each
GPU runs its own searches (global ids rank*S ...) on its own replica of W
(weak scaling) and the ranks all-gather every step's results (lockstep) or
their elites (async), so all pools stay identical.

The default line (random n = 32768, config 5) also carries `sub_results`:
configs 2-4 (random n = 1024 with 10,000 searches, Max-Cut n = 2000, TSP
n = 10,000), each timed for >= 2 s with its own clock record, and config 2
in async mode for ~10 s.

--impl reference: the repository's oracle (oracle/, plain C, the checker of
the parity tests) timed on this host's cores over a bounded sample of the
same workload (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import math
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
    "random32k": "random int16 QUBO n=32768 (config 5)",
    "random1k": "random int16 QUBO n=1024, 10k searches (config 2)",
    "maxcut2k": "Max-Cut G(2000, 19990) +-1 weights (config 3)",
    "tsp100": "TSP 100 cities, n=10000 one-hot (config 4)",
}
SIZES = {"random32k": 32768, "random1k": 1024, "maxcut2k": 2000, "tsp100": 10000}
SEED = 1
METRIC = "searched solutions/sec (n evals per flip)"


def make_W(workload: str):
    """Host copy of the workload's W (oracle, e2e input for the non-random
    workloads, parity tests)."""
    from workloads import maxcut_qubo, random_qubo_ctr, tsp_qubo
    if workload in ("random32k", "random1k"):
        return random_qubo_ctr(SIZES[workload], SEED)
    if workload == "maxcut2k":
        return maxcut_qubo(2000, 19990, seed=SEED)
    if workload == "tsp100":
        return tsp_qubo(100, seed=SEED)
    raise ValueError(workload)


def make_W_device(workload: str, device: int):
    """W in HBM: the random workloads are generated on the device (no host
    copy per rank); the others are small and copied from the host copy."""
    import torch

    import paper_conf_icpp_yasudonitkyi20_b200 as pkg
    if workload in ("random32k", "random1k"):
        n = SIZES[workload]
        Wd = torch.empty((n, n), dtype=torch.int16, device=f"cuda:{device}")
        return pkg.random_qubo_dev(Wd, SEED)
    return torch.from_numpy(make_W(workload)).to(f"cuda:{device}")


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

    def __init__(self, index: int, period_ms: int = 100):
        self.index = index
        self.period_ms = period_ms
        self.rows = []
        self._p = None

    def __enter__(self):
        try:
            self._p = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=" + ",".join(self.FIELDS),
                 "--format=csv,noheader,nounits", "-lms", str(self.period_ms)], stdout=subprocess.PIPE,
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
    """One search of the bench workload's first step, run by the oracle: the
    GA target of round 0 (host Step 4), the round with its window
    l and L = n (straight search + local search, Alg. 5 + Fig. 2)."""
    sid, L = args
    import oracle
    W = _W_SHARED
    n = W.shape[0]
    cfg = oracle.Config(n=n, searches=sid + 1, local_flips=L, pool_size=64, seed=SEED)
    T = oracle.Pool(n, 64, SEED).target(cfg, 0, sid)
    lad = oracle.default_ladder(n)
    t = time.perf_counter()
    out = oracle.replay_search(W, lad[sid % len(lad)], L, T)
    return int(out["flips"][0]), time.perf_counter() - t


def oracle_sample(W, procs: int, budget_s: float):
    """Run searches 0, 1, 2, ... of the bench workload's first step with the
    oracle, `procs` at a time (fork; W shared copy-on-write), until about
    `budget_s` seconds of wall time are spent.  Returns (flips, seconds,
    searches)."""
    global _W_SHARED
    _W_SHARED = W
    import oracle
    oracle.build()
    n = W.shape[0]
    ctx = mp.get_context("fork")
    flips, secs, done = 0, 0.0, 0
    with ctx.Pool(procs) as pool:
        batch = procs
        while secs < budget_s:
            t = time.perf_counter()
            res = pool.map(_oracle_job, [(done + i, n) for i in range(batch)])
            dt = time.perf_counter() - t
            flips += sum(r[0] for r in res)
            secs += dt
            done += batch
            # size the next batch to the remaining budget (whole multiples of procs)
            left = budget_s - secs
            if left <= 0.25 * dt:
                break
            batch = procs * max(1, int(left / dt))
    return flips, secs, done


def cpu_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    W = make_W(args.workload)
    n = W.shape[0]
    procs = min(cpu_cores(), 32)
    for _ in range(args.warmup):
        oracle_sample(W, procs, 0.5)
    tot_f, tot_t, tot_s = 0, 0.0, 0
    for _ in range(args.steps):
        f, dt, s = oracle_sample(W, procs, args.ref_step_seconds)
        tot_f += f
        tot_t += dt
        tot_s += s
    value = tot_f * n / tot_t
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "solutions/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * tot_t / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "int64", "data": "synthetic",
        "config": {"workload": args.workload, "n": n, "desc": WORKLOADS[args.workload],
                   "parallelism": "host processes"},
        "cpu_baseline": {"value": value, "unit": "solutions/s", "cores": procs, "kind": "oracle",
                         "sample": "per step: searches 0..k of the workload's first step (round-0 GA target, "
                                   "straight search + L=n local flips each), %d at a time, ~%.0f s; %d searches "
                                   "over %d steps" % (procs, args.ref_step_seconds, tot_s, args.steps)},
        "e2e": {"value": value, "unit": "solutions/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ rooflines
def _load_json(path, default=None):
    try:
        with open(path) as f:
            return json.load(f)
    except FileNotFoundError:
        return default


def _load_jsonl(path):
    try:
        with open(path) as f:
            return [json.loads(l) for l in f if l.strip().startswith("{")]
    except FileNotFoundError:
        return []


def probe_numbers():
    """Measured denominators (bench_probe/): the random-row read bandwidth of
    HBM (row_probe, 64 KiB rows) and of L2 (small_probe), and the int32 issue
    rate in lanes/clk/SM (small_probe)."""
    out = {}
    rows = _load_jsonl(os.path.join(ROOT, "profiles", "r01_row_probe.jsonl"))
    if rows:
        out["hbm_row_GBps"] = max(r["GBps"] for r in rows)
    small = _load_jsonl(os.path.join(ROOT, "profiles", "r02_small_probe.jsonl"))
    l2 = [r for r in small if r.get("probe") == "l2_rows"]
    for n in (1024, 2048, 10240):
        v = [r["GBps"] for r in l2 if r["n"] == n]
        if v:
            out["l2_row_GBps_n%d" % n] = max(v)
    ints = {r["op"]: r["lanes_per_clk_per_sm"] for r in small if r.get("probe") == "int32"}
    if ints:
        out["int32_lanes_per_clk_per_sm"] = max(ints.values())
        out["int32_probe"] = ints
    return out


def roofline(workload, n, n_pad, flips, launches, kern_s, ms, local):
    import torch
    peaks = _load_json(os.path.join(ROOT, "MEASURED_PEAKS.json"), {}) or {}
    hbm = float(peaks.get("hbm_gbs", 6650.0))
    peak_src = "MEASURED_PEAKS.json hbm_gbs (copy bandwidth)" if "hbm_gbs" in peaks else \
        "fallback 6650 GB/s (B200_PROFILING.md)"
    probes = probe_numbers()
    achieved = flips * 2.0 * n / kern_s / 1e9 if kern_s > 0 else None
    roof = {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
            "frac": (achieved / hbm) if achieved else None, "traffic": None, "traffic_unit": "GB per launch",
            "peak_source": peak_src, "kernel": "round_kernel",
            "algorithmic_bytes_per_launch": flips * 2.0 * n / max(1, launches),
            "algorithmic_unit": "2n bytes (one W row) per flip",
            "avg_launch_ms": 1e3 * kern_s / max(1, launches),
            "kernel_share_of_step": kern_s / (ms * 1e-3) if ms > 0 else None}
    if "hbm_row_GBps" in probes and achieved:
        roof["row_probe_GBps"] = probes["hbm_row_GBps"]
        roof["frac_vs_row_probe"] = achieved / probes["hbm_row_GBps"]
    # traffic: DRAM bytes per flip of the round kernel from the committed ncu --set
    # full capture of this workload, times this run's flips per launch
    prof = _load_json(os.path.join(ROOT, "profiles", "round_kernel_ncu_%s.json" % workload))
    if prof is None and workload == "random32k":
        prof = _load_json(os.path.join(ROOT, "profiles", "round_kernel_ncu.json"))
    if prof is not None and launches > 0:
        if prof.get("unit") != "flips":
            raise ValueError("ncu summary unit %r, expected 'flips'" % prof.get("unit"))
        roof["traffic"] = prof["dram_bytes_per_unit"] * flips / launches / 1e9
        roof["traffic_source"] = prof.get("source", "profiles/round_kernel_ncu*.json")
        roof["traffic_over_algorithmic"] = prof["dram_bytes_per_unit"] / (2.0 * n)
    if 2 * n_pad * n_pad <= 126 * 2 ** 20:
        # W is L2-resident (n <= ~8k): the second roof of SURVEY 8(d) binds, n int32
        # adds per flip against the integer pipes (measured lanes/clk/SM x SMs x max clock)
        sms = torch.cuda.get_device_properties(local).multi_processor_count
        mhz = float(peaks.get("sm_max_mhz", 1965.0))
        lanes = probes.get("int32_lanes_per_clk_per_sm")
        src = "measured (bench_probe/small_probe.cu, profiles/r02_small_probe.jsonl): %s lanes/clk/SM" % lanes
        if lanes is None:
            lanes = 128.0
            src = "derived: ALU + FMA pipes, 2 x 64 int32 lanes/clk/SM (B300_MICROARCH pipe rates)"
        int_peak = sms * lanes * mhz * 1e6 / 1e12
        ach = flips * float(n) / kern_s / 1e12 if kern_s > 0 else None
        l2key = "l2_row_GBps_n%d" % (1024 if n_pad <= 1024 else 2048 if n_pad <= 2048 else 10240)
        roof.update({"bound": "alu", "achieved": ach, "peak": int_peak, "unit": "T int32 adds/s",
                     "frac": (ach / int_peak) if ach else None,
                     "peak_source": "%s x %d SMs x %.0f MHz (max SM clock)" % (src, sms, mhz),
                     "row_bytes_GBps": achieved})
        if l2key in probes and achieved:
            roof["l2_row_probe_GBps"] = probes[l2key]
            roof["frac_vs_l2_row_probe"] = achieved / probes[l2key]
    return roof


# ------------------------------------------------------------------ the GPU arm
class Ctx:
    def __init__(self):
        import torch
        import torch.distributed as dist
        self.torch, self.dist = torch, dist
        self.world = int(os.environ.get("WORLD_SIZE", "1"))
        self.rank = int(os.environ.get("RANK", "0"))
        local = int(os.environ.get("LOCAL_RANK", "0"))
        # test hooks for exercising the multi-rank flow on a single GPU (both ranks on
        # one device, gloo for the exchange); the driver's runs use the defaults
        self.local = int(os.environ.get("ABS_BENCH_DEVICE", local))
        self.backend = os.environ.get("ABS_BENCH_BACKEND", "nccl")
        assert torch.cuda.is_available(), "bench.py needs B200 GPUs"
        torch.cuda.set_device(self.local)
        if self.world > 1:
            if self.backend == "nccl":
                dist.init_process_group("nccl", device_id=torch.device("cuda", self.local))
            else:
                dist.init_process_group(self.backend)
        self.rdev = "cuda" if self.backend == "nccl" else "cpu"

    def barrier(self):
        if self.world > 1:
            self.dist.barrier()

    def allreduce(self, v, op):
        t = self.torch.tensor([float(v)], dtype=self.torch.float64, device=self.rdev)
        if self.world > 1:
            self.dist.all_reduce(t, op=op)
        return float(t.item())

    def max(self, v):
        return self.allreduce(v, self.dist.ReduceOp.MAX)

    def sum(self, v):
        return self.allreduce(v, self.dist.ReduceOp.SUM)


def run_workload(X: Ctx, workload, steps, warmup, mode="lockstep", policy="window", searches=0, local_flips=0,
                 min_seconds=0.0, e2e=True, W_host=None):
    """Time `steps` steps (or, with min_seconds, enough steps to fill that
    much time, decided after the warm-up) of one workload on every rank.
    Returns a result dict (rank 0 fields meaningful)."""
    torch = X.torch
    import paper_conf_icpp_yasudonitkyi20_b200 as pkg
    from paper_conf_icpp_yasudonitkyi20_b200 import dist as pdist

    n = SIZES[workload]
    Wd = make_W_device(workload, X.local)
    S = searches or default_searches(workload, n, X.local)
    L = local_flips or n
    amode = pkg.MODE_ASYNC if mode == "async" else pkg.MODE_LOCKSTEP
    common = dict(searches=S, local_flips=L, pool_size=64, seed=SEED, device=X.local, mode=amode)
    if policy == "sa":
        # SA policy (reading E2): a 4-level temperature ladder from the weight scale up
        wmax = int(Wd[:256].abs().max().item()) or 1  # weight scale from a row sample
        common.update(policy=pkg.POLICY_SA, sa_tau_min=max(1, wmax // 4), sa_tau_max=8 * wmax, sa_levels=4)
    ext = X.world > 1 and amode == pkg.MODE_LOCKSTEP
    solver = pkg.Solver(Wd, search_offset=X.rank * S, external_merge=ext, **common)

    def step(s):
        if X.world > 1:
            pdist.lockstep_step(s)
        else:
            s.search(1)

    def run_steps(s, k):
        if amode == pkg.MODE_ASYNC:
            # one persistent launch for all k rounds of every search (the
            # blocks run asynchronously); ranks then all-gather their elites
            s.search(k)
            if X.world > 1:
                pdist.exchange_elites(s, 64)
        else:
            for _ in range(k):
                step(s)

    X.barrier()
    torch.cuda.synchronize()
    tw = time.perf_counter()
    run_steps(solver, warmup)
    torch.cuda.synchronize()
    warm_s = time.perf_counter() - tw
    if min_seconds > 0:
        per = warm_s / max(1, warmup)
        if amode == pkg.MODE_ASYNC:
            # one launch per call: calibrate on a longer (untimed) call than the warm-up
            k = max(1, int(0.15 * min_seconds / max(per, 1e-6)))
            torch.cuda.synchronize()
            tw = time.perf_counter()
            run_steps(solver, k)
            torch.cuda.synchronize()
            per = (time.perf_counter() - tw) / k
        steps = int(X.max(max(steps, math.ceil(min_seconds / max(per, 1e-6)))))
    st0 = solver.stats()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(X.local) as clk:
        X.barrier()
        torch.cuda.synchronize()
        ev0.record()
        run_steps(solver, steps)
        ev1.record()
        torch.cuda.synchronize()
        X.barrier()
    st1 = solver.stats()
    ms = ev0.elapsed_time(ev1)
    flips = st1["flips"] - st0["flips"]
    kern_s = st1["search_seconds"] - st0["search_seconds"]
    launches = st1["round_kernel_launches"] - st0["round_kernel_launches"]
    all_launches = st1["kernel_launches"] - st0["kernel_launches"]
    ms_max = X.max(ms)
    flips_all = X.sum(flips)
    res = {
        "value": flips_all * n / (ms_max * 1e-3), "unit": "solutions/s", "steps": steps, "warmup": warmup,
        "ms_per_step": ms_max / steps, "seconds": ms_max * 1e-3, "flips_per_step": flips_all / steps,
        "gpu_launches": int(all_launches),
        "config": {"workload": workload, "desc": WORKLOADS[workload], "n": n, "searches_per_gpu": S,
                   "local_flips": L, "pool": 64, "mode": mode, "policy": policy,
                   "w_source": "generated on device (abs_random_qubo_dev)" if workload.startswith("random")
                   else "host generator, copied once"},
        "roofline": roofline(workload, n, int(st1["n_pad"]), flips, launches, kern_s, ms, X.local),
        "clocks": clk.summary(),
    }
    solver.close()
    del solver
    torch.cuda.synchronize()

    if e2e:
        # end to end through the public API with HOST buffers: abs_create from pinned host
        # W (H2D inside the timed region), the steps, abs_best (D2H of the result)
        if W_host is None:
            W_host = torch.empty(Wd.shape, dtype=torch.int16, pin_memory=True)
            W_host.copy_(Wd)  # staging of the input, outside the timed region
        Wh = W_host.numpy()
        del Wd
        torch.cuda.synchronize()
        X.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        s2 = pkg.Solver(Wh, search_offset=X.rank * S, external_merge=ext, **common)
        run_steps(s2, steps)
        Xb, Eb = s2.best() if X.world == 1 else (None, None)
        e1.record()
        torch.cuda.synchronize()
        st2 = s2.stats()
        s2.close()
        ems = X.max(e0.elapsed_time(e1))
        f2 = X.sum(st2["flips"])
        res["e2e"] = {"value": f2 * n / (ems * 1e-3), "unit": "solutions/s",
                      "h2d_bytes_per_step": st2["h2d_bytes"] / steps,
                      "d2h_bytes_per_step": (st2["d2h_bytes"] + 8 * ((n + 31) // 32)) / steps,
                      "includes": "abs_create from pinned host W (H2D 2n^2 bytes) + steps + abs_best"}
    return res


def run_abs(args):
    X = Ctx()
    main = run_workload(X, args.workload, args.steps, args.warmup, mode=args.mode, policy=args.policy,
                        searches=args.searches, local_flips=args.local_flips, e2e=not args.no_e2e)
    n = SIZES[args.workload]

    subs = {}
    if not args.no_sub and args.workload == "random32k" and args.mode == "lockstep" and args.policy == "window":
        # configs 2-4 of BASELINE.json, each >= 2 s, and config 2 async for ~10 s
        for w in ("random1k", "maxcut2k", "tsp100"):
            r = run_workload(X, w, 3, 3, min_seconds=args.sub_seconds, e2e=False)
            subs[w] = {k: r[k] for k in ("value", "unit", "steps", "ms_per_step", "seconds", "roofline", "clocks",
                                         "config", "gpu_launches")}
        r = run_workload(X, "random1k", 3, 3, mode="async", min_seconds=args.async_seconds, e2e=False)
        subs["random1k_async"] = {k: r[k] for k in ("value", "unit", "steps", "seconds", "roofline", "clocks",
                                                    "config", "gpu_launches")}
        subs["random1k_async"]["note"] = "config 2: throughput of one asynchronous abs_search call of ~%.0f s " \
                                         "(persistent kernel + host GA thread, Fig. 5)" % args.async_seconds

    # ---------------- cpu baseline (oracle), rank 0 at N = 1 only
    cpu = None
    if X.rank == 0 and X.world == 1 and not args.no_cpu_baseline:
        W = make_W(args.workload)
        procs = min(cpu_cores(), 32)
        f, dt, s = oracle_sample(W, procs, args.cpu_seconds)
        cpu = {"value": f * n / dt, "unit": "solutions/s", "cores": procs, "kind": "oracle",
               "sample": "searches 0..%d of the bench step (round-0 GA targets, straight search + L=n local "
                         "flips each), %d at a time on %d cores, %.1f s" % (s - 1, procs, procs, dt)}

    if X.rank == 0:
        line = {
            "metric": METRIC, "value": main["value"], "unit": "solutions/s", "n_gpus": X.world,
            "steps": main["steps"], "warmup": args.warmup, "ms_per_step": main["ms_per_step"],
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic (Philox random int16 QUBO generated on device, P:L468)"
            if args.workload.startswith("random") else "synthetic",
            "config": dict(main["config"], parallelism="dp%d (replicated W, independent searches)" % X.world,
                           l2="inputs larger than L2 (W = %d MiB)" % (2 * n * n >> 20)
                           if 2 * n * n > 126 * 2 ** 20 else "W fits in L2 (resident by design)"),
            "flips_per_step": main["flips_per_step"],
            "roofline": main["roofline"],
            "cpu_baseline": cpu,
            "e2e": main.get("e2e"),
            "gpu_launches": main["gpu_launches"],
            "clocks": main["clocks"],
            "sub_results": subs or None,
            "paper_context": "1.24e12 solutions/s on 4x RTX 2080 Ti at n=1024; 4.39e11 at n=32768 (P:L529, P:L544)",
        }
        print(json.dumps(line), flush=True)
    if X.world > 1:
        X.dist.destroy_process_group()
    return 0


def relaunch_distributed(n: int) -> int:
    """bench.py --gpus N run directly: re-execute under torch.distributed.run,
    one process per GPU (the driver's own launch form)."""
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(n),
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


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
    ap.add_argument("--no-sub", action="store_true", help="skip the configs 2-4 sub-results")
    ap.add_argument("--sub-seconds", type=float, default=3.0)
    ap.add_argument("--async-seconds", type=float, default=10.0)
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--ref-step-seconds", type=float, default=8.0)
    args = ap.parse_args()
    if args.warmup < 3:
        print("warning: --warmup < 3 violates the timing rules", file=sys.stderr)
    world = os.environ.get("WORLD_SIZE")
    if world is None and args.gpus > 1:
        return relaunch_distributed(args.gpus)
    if world is not None and int(world) != args.gpus:
        print("bench.py: --gpus %d but WORLD_SIZE=%s (one process per GPU)" % (args.gpus, world), file=sys.stderr)
        return 2
    if args.impl == "reference":
        return run_reference(args)
    return run_abs(args)


if __name__ == "__main__":
    sys.exit(main())
