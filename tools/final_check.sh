mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q --timeout 600 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
for w in random32k random1k maxcut2k; do
  timeout 600 python bench.py --workload $w --policy sa --steps 3 --no-e2e --no-cpu-baseline > gpurun_out/sa_$w.json 2>> gpurun_out/bench.err; echo "sa $w rc=$?"
done
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
tail -1 gpurun_out/pytest_gpu.log; cat gpurun_out/smoke.log; cut -c1-200 gpurun_out/bench.json
