set -u
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sa.py tests/test_tts.py -x -q --timeout 600 > gpurun_out/pytest_d.log 2>&1; echo "parity rc=$?"
tail -15 gpurun_out/pytest_d.log
WORKLOADS="random1k maxcut2k" VARIANTS="new old new old" BENCH_ARGS="--steps 20" bash tools/ab_bench.sh
WORKLOADS="random1k maxcut2k" VARIANTS="new old" BENCH_ARGS="--steps 10 --policy sa" bash tools/ab_bench.sh
