#!/bin/bash
# GPU-side A/B with phase timing: parity tests, bench of libabs.so vs libabs_old.so, and the
# per-phase cycle accounting of both diagnostics builds (libabs_timing.so / libabs_timing_old.so).
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_sa.py -x -q --timeout 300 2>&1 | tail -2
WORKLOADS="${WORKLOADS:-random32k}" VARIANTS="${VARIANTS:-new old new old}" bash tools/ab_bench.sh
ABS_LIB=$PWD/paper_conf_icpp_yasudonitkyi20_b200/libabs_timing.so timeout 300 python tools/timing_run.py 32768 "" 3 > gpurun_out/timing_new.txt 2>&1
ABS_LIB=$PWD/paper_conf_icpp_yasudonitkyi20_b200/libabs_timing_old.so timeout 300 python tools/timing_run.py 32768 "" 3 > gpurun_out/timing_old.txt 2>&1
python - <<'PY'
import json
a=json.load(open('gpurun_out/timing_new.txt')); b=json.load(open('gpurun_out/timing_old.txt'))
for ph in ('local','straight'):
    for w in ('row_warps','control_warp'):
        print(ph, w, 'new', a[ph][w]); print(ph, w, 'old', b[ph][w])
print(a.get('straight_improve'), a.get('certain_selection_fraction'), a.get('selection_subphases'), b.get('selection_subphases'))
PY
