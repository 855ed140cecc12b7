#!/bin/bash
# GPU-side A/B session: parity tests, A/B bench of libabs.so vs libabs_old.so, timing breakdown at n=32k.
mkdir -p gpurun_out
timeout 500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sa.py -x -q --timeout 300 2>&1 | tail -2
WORKLOADS="${WORKLOADS:-random32k tsp100 maxcut2k random1k}" VARIANTS="${VARIANTS:-new old}" bash tools/ab_bench.sh
if [ -f paper_conf_icpp_yasudonitkyi20_b200/libabs_timing.so ]; then
  ABS_LIB=$PWD/paper_conf_icpp_yasudonitkyi20_b200/libabs_timing.so timeout 300 python tools/timing_run.py 32768 "" 3 > gpurun_out/timing.txt 2>&1
fi
