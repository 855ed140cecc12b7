# GPU iteration for the SA kernels: SA/parity GPU tests, then SA bench lines of the working
# tree's library against libabs_old.so (SA_WORKLOADS) and the window A/B (WORKLOADS, may be empty).
export TESTS="${TESTS:-tests/test_gpu_parity.py tests/test_gpu_sa.py}"
export WORKLOADS="${WORKLOADS-random1k maxcut2k}" VARIANTS="${VARIANTS:-new old new old}" BENCH_ARGS="${BENCH_ARGS:---steps 100 --no-sub}" NCU=0
bash tools/gpu_iter.sh
for w in ${SA_WORKLOADS:-random1k maxcut2k}; do for v in new old new old; do
  if [ $v = old ]; then export ABS_LIB=$PWD/paper_conf_icpp_yasudonitkyi20_b200/libabs_old.so; else unset ABS_LIB; fi
  timeout 300 python bench.py --workload $w --policy sa --steps ${SA_STEPS:-20} --no-e2e --no-cpu-baseline --no-sub > gpurun_out/sa.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/sa.json')); print('SA $w $v %.4e' % d['value'])"
done; done
