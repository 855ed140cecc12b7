set -u
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o bench_probe/small_probe bench_probe/small_probe.cu && \
  timeout 300 ./bench_probe/small_probe > gpurun_out/small_probe.jsonl 2>&1; echo "probe rc=$?"
timeout 1500 python -m pytest tests/test_gpu_dist.py tests/test_gpu_parity.py -q --timeout 900 \
  -k "dist or random_qubo_dev or bench_configuration or three_rounds" > gpurun_out/pytest_c.log 2>&1; echo "tests rc=$?"
tail -3 gpurun_out/pytest_c.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
ABS_BENCH_BACKEND=gloo ABS_BENCH_DEVICE=0 timeout 600 python bench.py --gpus 2 --workload maxcut2k --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_gpus2_relaunch.json 2> gpurun_out/bench_gpus2.err; echo "gpus2 relaunch rc=$?"
bash tools/multirank_check.sh
cut -c1-600 gpurun_out/bench.json; tail -5 gpurun_out/bench.err
