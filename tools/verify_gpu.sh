set -u
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi > $OUT/nvsmi.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q --timeout 400 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?"
tail -3 $OUT/pytest_gpu.log; cat $OUT/bench.json
