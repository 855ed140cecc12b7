#!/usr/bin/env python
"""Batched initialisation throughput: the tensor-core engine
(tcgen05.mma kind::i8) against the ALU engine, through abs_energy_dev on
device-resident inputs.  Kernel time = CUDA events around the launch on the
library stream (abs_stats.init_seconds), median of --reps after --warmup.

Roofline (tensor engine): the contraction S = X Wz^T is count * n * n
multiply-adds; it runs as TWO int8 GEMMs (hi and lo planes), so the int8
pipe executes 2 * 2 * count * n^2 ops.  Peak = the measured dense bf16
figure x 2 (the guide's int8 : bf16 ratio), else 4500 TOP/s nominal.

  python tools/init_bench.py [--n 1024 --count 10000] [--engine mma|alu|both]
One JSON line per (n, count, engine)."""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def int8_peak_tops():
    try:
        mp = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
        for k in ("bf16_dense_tflops", "bf16_tflops", "dense_bf16_tflops"):
            if k in mp:
                return 2.0 * float(mp[k]), "measured bf16 x 2"
    except Exception:
        pass
    return 4500.0, "nominal int8 dense (B200_PROFILING fallback)"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, nargs="*", default=[1024, 32768])
    ap.add_argument("--count", type=int, nargs="*", default=[10000, 1024])
    ap.add_argument("--engine", default="both")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--delta", type=int, default=1, help="also write the n Delta per solution")
    a = ap.parse_args()
    import torch

    import paper_conf_icpp_yasudonitkyi20_b200 as pkg
    from workloads import random_qubo, random_solutions
    peak, peak_src = int8_peak_tops()
    engines = {"mma": pkg.INIT_MMA, "alu": pkg.INIT_ALU}
    sel = list(engines) if a.engine == "both" else [a.engine]
    for n, count in zip(a.n, a.count):
        W = random_qubo(n, 1)
        s = pkg.Solver(W, searches=1)
        X = torch.from_numpy(random_solutions(count, n, 3).view(np.int32)).cuda()
        E = torch.zeros(count, dtype=torch.int64, device="cuda")
        D = torch.zeros((count, n), dtype=torch.int32, device="cuda") if a.delta else None
        ref = None
        for name in sel:
            ts = []
            for r in range(a.warmup + a.reps):
                t = s.energy_dev(X, E, D, engines[name])
                if r >= a.warmup:
                    ts.append(t)
            Ec = E.cpu().numpy().copy()
            if ref is None:
                ref = Ec
            agree = bool((Ec == ref).all())
            t = statistics.median(ts)
            macs = float(count) * n * n
            line = {"kernel": "init_" + name, "n": n, "count": count, "delta": bool(a.delta),
                    "ms": t * 1e3, "solutions_per_s": count / t, "contraction_tmacs": macs / t / 1e12,
                    "energies_agree_with_first_engine": agree}
            if name == "mma":
                ops = 4.0 * macs
                line["roofline"] = {"bound": "tensor", "achieved": ops / t / 1e12, "peak": peak,
                                    "unit": "TOP/s (int8)", "frac": ops / t / 1e12 / peak, "peak_source": peak_src,
                                    "algorithmic_ops_per_launch": ops}
            print(json.dumps(line), flush=True)
        s.close()


if __name__ == "__main__":
    main()
