#!/bin/bash
# One GPU session producing the round's evidence: parity tests, bench lines,
# ncu launch list and a full ncu capture of the round kernel.  Run under gpurun.
set -u
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi > $OUT/nvsmi.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q --timeout 400 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
timeout 600 python bench.py --impl reference > $OUT/bench_ref.json 2> $OUT/bench_ref.err; echo "ref rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/bench_under_ncu.log 2>&1; echo "ncu-launches rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:round_kernel -s 2 -c 1 \
    -o $OUT/prof_round python tools/prof_round.py --n 32768 --steps 3 > $OUT/prof_round.log 2>&1; echo "ncu-full rc=$?"
# time-to-solution (Table 1 analogue)
{ timeout 200 python tools/tts_run.py --workload maxcut --n 800 --edges 19176 --weights one --fraction 1.0 --ref-seconds 10 --max-seconds 10 --repeats 3
  timeout 200 python tools/tts_run.py --workload maxcut --n 2000 --edges 19990 --fraction 0.99 --ref-seconds 15 --max-seconds 10 --repeats 3
  timeout 200 python tools/tts_run.py --workload tsp --cities 16 --fraction 1.0 --ref-seconds 10 --max-seconds 10 --repeats 3
  timeout 300 python tools/tts_run.py --workload random --n 32768 --fraction 0.99 --ref-seconds 20 --max-seconds 20 --repeats 2
} > $OUT/tts.jsonl 2> $OUT/tts.err; echo "tts rc=$?"
