set -u
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sa.py -x -q --timeout 600 -k "not n32768 and not full_size and not 32768 and not bench_configuration and not multiwarp" > gpurun_out/pytest_f.log 2>&1; echo "parity rc=$?"
tail -5 gpurun_out/pytest_f.log
WORKLOADS="random1k maxcut2k" VARIANTS="new old new old" BENCH_ARGS="--steps 20" bash tools/ab_bench.sh
