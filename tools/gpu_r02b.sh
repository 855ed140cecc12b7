set -u
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sa.py -q --timeout 600 > gpurun_out/pytest_sa.log 2>&1; echo "sa tests rc=$?"
tail -3 gpurun_out/pytest_sa.log
for n in 100 1100 3000; do for mode in lockstep async; do
  timeout 240 /usr/local/cuda/bin/compute-sanitizer --tool racecheck --error-exitcode 9 --print-limit 20 \
    python tools/sanitize_run.py --n $n --mode $mode --policy sa > gpurun_out/race_sa_${n}_${mode}.log 2>&1
  echo "racecheck sa n=$n $mode rc=$?"
done; done
WORKLOADS="random32k random1k maxcut2k tsp100" VARIANTS="new old new old" BENCH_ARGS="--policy sa --steps 3" bash tools/ab_bench.sh
