#!/usr/bin/env python
"""Summarise an ncu --set full capture (.ncu-rep) of one kernel launch into the
JSON kept under profiles/: duration, DRAM bytes, L2 hit rate, pipe/issue
utilisation, stall mix, instructions per unit of work.

  python tools/ncu_summary.py REP --units U --unit-name flips --algorithmic-bytes B --source "..." > out.json"""
import argparse
import csv
import io
import json
import subprocess

ap = argparse.ArgumentParser()
ap.add_argument("rep")
ap.add_argument("--units", type=float, default=0.0)
ap.add_argument("--unit-name", default="flips")
ap.add_argument("--algorithmic-bytes", type=float, default=0.0)
ap.add_argument("--algorithmic-ops", type=float, default=0.0)
ap.add_argument("--source", default="")
a = ap.parse_args()
raw = subprocess.check_output(["ncu", "-i", a.rep, "--page", "raw", "--csv"], stderr=subprocess.DEVNULL).decode()
rows = list(csv.reader(io.StringIO(raw)))
h, units_row, v = rows[0], rows[1], rows[2]
d = dict(zip(h, v))
u = dict(zip(h, units_row))


def num(k):
    try:
        x = float(d[k].replace(",", ""))
    except (KeyError, ValueError):
        return None
    unit = u.get(k, "")
    scale = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0, "Tbyte": 1e12, "ms": 1e-3, "us": 1e-6,
             "ns": 1e-9, "s": 1.0, "msecond": 1e-3, "usecond": 1e-6, "nsecond": 1e-9, "second": 1.0,
             "Ghz": 1e9, "Mhz": 1e6, "hz": 1.0}.get(unit, 1.0)
    return x * scale


dur = num("gpu__time_duration.sum")
rd, wr = num("dram__bytes_read.sum"), num("dram__bytes_write.sum")
out = {
    "source": a.source,
    "kernel": d.get("Kernel Name"),
    "duration_s": dur,
    "dram_read_bytes": rd,
    "dram_write_bytes": wr,
    "dram_bytes_per_s": (rd + wr) / dur if dur else None,
    "l2_hit_rate_pct": num("lts__t_sector_hit_rate.pct"),
    "issue_active_pct": num("sm__issue_active.avg.pct_of_peak_sustained_elapsed"),
    "alu_pipe_active_pct": num("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active"),
    "fma_pipe_active_pct": num("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active"),
    "tensor_pipe_active_pct": num("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active")
    or num("sm__inst_executed_pipe_tc.avg.pct_of_peak_sustained_active"),
    "warps_active_pct": num("sm__warps_active.avg.pct_of_peak_sustained_active"),
    "registers_per_thread": num("launch__registers_per_thread"),
    "sm_clock_hz": num("sm__cycles_elapsed.avg.per_second"),
    "warp_instructions": num("smsp__inst_executed.sum"),
    "local_load_instructions": num("sass__inst_executed_local_loads"),
}
st = [k for k in h if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued")]
tot = sum(num(k) or 0 for k in st)
if tot:
    out["stall_mix"] = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): round((num(k) or 0) / tot, 3)
                        for k in sorted(st, key=lambda k: -(num(k) or 0))[:8]}
if a.units:
    out["units"] = a.units
    out["unit"] = a.unit_name
    out["dram_bytes_per_unit"] = (rd + wr) / a.units
    out["warp_instructions_per_unit"] = (out["warp_instructions"] or 0) / a.units
if a.algorithmic_bytes:
    out["algorithmic_bytes"] = a.algorithmic_bytes
    out["traffic_over_algorithmic"] = (rd + wr) / a.algorithmic_bytes
    out["algorithmic_GBps"] = a.algorithmic_bytes / dur / 1e9
if a.algorithmic_ops:
    out["algorithmic_ops"] = a.algorithmic_ops
    out["algorithmic_TOPs"] = a.algorithmic_ops / dur / 1e12
print(json.dumps(out, indent=1))
