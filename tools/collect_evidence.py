"""Copy one gpu_artifacts.sh session from gpurun_out/ into profiles/r02/ under a tag
(bench lines, reference arm, launch list, pytest log, smoke, init bench, SA lines) and
summarise its ncu captures with tools/ncu_summary.py.  Prints the headline numbers.
  python tools/collect_evidence.py r02m"""
import json, shutil, subprocess, sys

tag = sys.argv[1]
G, P = "gpurun_out", "profiles/r02"
for src, dst in [("bench.json", "bench.json"), ("bench_ref.json", "bench_ref.json"), ("launches.csv", "launches_ncu.csv"),
                 ("pytest_gpu.log", "pytest_gpu.log"), ("smoke.log", "smoke.log"), ("init_bench.jsonl", "init_bench.jsonl")]:
    shutil.copy(f"{G}/{src}", f"{P}/{tag}_{dst}")
with open(f"{P}/{tag}_sa_bench.jsonl", "w") as f:
    for w in ["random32k", "random1k", "maxcut2k", "tsp100"]:
        f.write(open(f"{G}/sa_{w}.json").read().strip().splitlines()[-1] + "\n")
cases = [("prof_round", 32768, "n32k", "--n 32768 --searches 592 --steps 3 (launch 2; config 5)"),
         ("prof_round1k", 1024, "n1k", "--n 1024 --searches 4736 --steps 3 (launch 2; config 2 at one launch per step: 32 x 148 resident searches; WarpRound<32>)"),
         ("prof_round2k", 2000, "maxcut2k", "--n 2000 --searches 2368 --steps 3 --workload maxcut (launch 2; config 3; WarpRound<64>)")]
for rep, n, name, src in cases:
    fl = [json.loads(l) for l in open(f"{G}/{rep}.log") if l.startswith('{"flips"')]
    f = [x for x in fl if x["launch"] == 2][0]["flips"]
    out = subprocess.check_output(["python", "tools/ncu_summary.py", f"{G}/{rep}.ncu-rep", "--units", str(f), "--unit-name", "flips",
                                   "--algorithmic-bytes", str(2 * n * f), "--algorithmic-ops", str(n * f), "--source",
                                   "ncu --set full --clock-control none -k regex:round_kernel -s 2 -c 1 python tools/prof_round.py "
                                   + src + f"; {tag} code"]).decode()
    open(f"{P}/{tag}_round_kernel_{name}_ncu.json", "w").write(out)
    d = json.loads(out)
    print(name, "ms %.3f" % (1e3 * d["duration_s"]), "instr/flip %.1f" % d["warp_instructions_per_unit"],
          "issue %.1f%%" % d["issue_active_pct"], "dram B/flip %.0f" % d["dram_bytes_per_unit"])
out = subprocess.check_output(["python", "tools/ncu_summary.py", f"{G}/prof_init.ncu-rep", "--source",
                               f"ncu --set full -k regex:init_mma -s 2 -c 1 python tools/init_bench.py --n 32768 --count 1024 --engine mma ({tag} code)"]).decode()
open(f"{P}/{tag}_init_mma_ncu.json", "w").write(out)
d = json.loads(open(f"{G}/bench.json").read().strip().splitlines()[-1])
print("bench", "%.4g" % d["value"], "frac %.3f" % d["roofline"]["frac"], d["clocks"], "e2e %.4g" % d["e2e"]["value"])
for k, v in d.get("sub_results", {}).items():
    print(" ", k, "%.4g" % v["value"], "frac %.3f" % (v.get("roofline", {}).get("frac") or 0), v.get("clocks", {}).get("sm_mhz"))
for l in open(f"{P}/{tag}_sa_bench.jsonl"):
    x = json.loads(l)
    print("SA", x["config"]["workload"], "%.4g" % x["value"])
print(open(f"{G}/pytest_gpu.log").read().strip().splitlines()[-1])
