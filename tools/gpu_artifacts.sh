#!/bin/bash
# One GPU session producing the round's evidence: GPU tests, smoke, the default bench
# line (with the configs 2-4 sub-results), SA lines, the reference arm, the ncu launch
# list of the default bench command, full ncu captures of the round kernels (n = 32k
# multi-warp, n = 1k and MaxCut n = 2000 one-warp) and of the tensor-core init kernel,
#.  Run under gpurun; outputs in gpurun_out/.
set -u
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi > $OUT/nvsmi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
# SA lines: 3 steps at n >= 10,000 (~0.2-0.5 s each), 30 at n <= 2048 (a step is ~2-7 ms there)
for w in random32k random1k maxcut2k tsp100; do
  case $w in random1k|maxcut2k) st=30;; *) st=3;; esac
  timeout 600 python bench.py --workload $w --policy sa --steps $st --no-e2e --no-cpu-baseline > $OUT/sa_$w.json 2>> $OUT/bench.err; echo "sa $w rc=$?"
done
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > $OUT/bench_ref.json 2> $OUT/bench_ref.err; echo "ref rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-sub > $OUT/bench_under_ncu.log 2>&1; echo "ncu-launches rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:round_kernel -s 2 -c 1 \
    -o $OUT/prof_round python tools/prof_round.py --n 32768 --searches 592 --steps 3 > $OUT/prof_round.log 2>&1; echo "ncu-full rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:round_kernel -s 2 -c 1 \
    -o $OUT/prof_round1k python tools/prof_round.py --n 1024 --searches 4736 --steps 3 > $OUT/prof_round1k.log 2>&1; echo "ncu-full-1k rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:round_kernel -s 2 -c 1 \
    -o $OUT/prof_round2k python tools/prof_round.py --n 2000 --searches 2368 --steps 3 --workload maxcut > $OUT/prof_round2k.log 2>&1; echo "ncu-full-2k rc=$?"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:init_mma -s 2 -c 1 \
    -o $OUT/prof_init python tools/init_bench.py --n 32768 --count 1024 --engine mma --reps 2 --warmup 1 > $OUT/prof_init.log 2>&1; echo "ncu-init rc=$?"
timeout 300 python tools/init_bench.py > $OUT/init_bench.jsonl 2>&1; echo "init-bench rc=$?"
# compute-sanitizer is closed on the GPU pool (runs under it left GPUs needing a reset); the
# sanitizer logs of round 2 are under profiles/r02/sanitizer_r02*.
tail -2 $OUT/pytest_gpu.log; cut -c1-300 $OUT/bench.json
