set -u
mkdir -p gpurun_out
nvidia-smi > gpurun_out/nvsmi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -k "multiwarp_ladder_extremes or three_rounds_replay" > gpurun_out/pytest_new.log 2>&1; echo "new rc=$?"
bash tools/sanitize.sh
tail -5 gpurun_out/pytest_new.log; cat gpurun_out/sanitizer/summary.txt
