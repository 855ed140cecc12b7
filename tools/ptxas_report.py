"""Registers / spills / stack of every kernel in abs_round.cu (nvcc -Xptxas -v),
one line per kernel: the check before spending GPU time on a flip-loop change."""
import os, re, subprocess, sys
HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "..", "paper_conf_icpp_yasudonitkyi20_b200", "csrc")
src = sys.argv[1] if len(sys.argv) > 1 else "abs_round.cu"
extra = sys.argv[2:]
out = subprocess.run(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-std=c++17", "-Xptxas", "-v",
                      "-I", os.path.join(HERE, "..", "include"), "-I", CSRC, *extra, "-c", os.path.join(CSRC, src),
                      "-o", "/dev/null"], capture_output=True, text=True).stderr
cur = None
rows = {}
for line in out.splitlines():
    m = re.search(r"Compiling entry function '([^']+)'|Function properties for (\S+)", line)
    if m:
        cur = m.group(1) or m.group(2)
        rows.setdefault(cur, {})
        continue
    if cur is None:
        continue
    m = re.search(r"(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads", line)
    if m:
        rows[cur].update(stack=int(m.group(1)), st=int(m.group(2)), ld=int(m.group(3)))
    m = re.search(r"Used (\d+) registers", line)
    if m:
        rows[cur]["reg"] = int(m.group(1))
def short(name):
    m = re.search(r"(round_kernel(?:_async)?)I.*?5RoundILi(\d+)ELi(\d+)ELi(\d+)ELb(\d)", name)
    if m:
        return "%s<%s,%s,%s,%s>" % (m.group(1), m.group(2), m.group(3), m.group(4), "SA" if m.group(5) == "1" else "win")
    m = re.search(r"(round_kernel(?:_async)?)I.*?9WarpRoundILi(\d+)ELb(\d)", name)
    if m:
        return "%s<warp %s,%s>" % (m.group(1), m.group(2), "SA" if m.group(3) == "1" else "win")
    m = re.search(r"(round_kernel(?:_async)?)ILi(\d+)ELi(\d+)ELi(\d+)ELb(\d)", name)
    if m:
        return "%s<%s,%s,%s,%s>" % (m.group(1), m.group(2), m.group(3), m.group(4), "SA" if m.group(5) == "1" else "win")
    return name[:60]
for k, v in sorted(rows.items(), key=lambda kv: short(kv[0])):
    if "reg" in v or v.get("st"):
        print("%-44s reg %3s  stack %4s  spill st %4s ld %4s" % (short(k), v.get("reg", "-"), v.get("stack", "-"),
                                                                v.get("st", "-"), v.get("ld", "-")))
