"""Per-flip execution counts of the SASS of one ncu --set full capture (source page):
  python tools/sass_hot.py REP.ncu-rep FLIPS [MIN_PER_FLIP] > listing
prints 'index  executions/flip  samples  instruction' for every instruction above the threshold
and the total warp instructions per flip."""
import csv, io, subprocess, sys
rep, flips = sys.argv[1], float(sys.argv[2])
thr = float(sys.argv[3]) if len(sys.argv) > 3 else 0.05
raw = subprocess.check_output(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                              stderr=subprocess.DEVNULL).decode()
rows = list(csv.reader(io.StringIO(raw)))
h = rows[1]
ia, isamp = h.index("Instructions Executed"), h.index("# Samples")
tot = 0
for i, r in enumerate(rows[2:]):
    ex = int(r[ia])
    tot += ex
    if ex / flips > thr:
        print(f"{i:5d} {ex / flips:7.3f} {int(r[isamp]):6d}  {r[1].strip()}")
print(f"# total warp instructions per flip: {tot / flips:.1f}")
