mkdir -p gpurun_out
OLD=$PWD/paper_conf_icpp_yasudonitkyi20_b200/libabs_old.so
for w in ${WORKLOADS:-random32k}; do for v in ${VARIANTS:-new old new old}; do
  if [ $v = old ]; then export ABS_LIB=$OLD; elif [ $v = new ]; then unset ABS_LIB; else export ABS_LIB=$PWD/paper_conf_icpp_yasudonitkyi20_b200/libabs_$v.so; fi
  timeout ${AB_TIMEOUT:-90} python bench.py --workload $w --no-e2e --no-cpu-baseline $BENCH_ARGS > gpurun_out/ab.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/ab.json')); print('$w $v %.4e frac=%.3f ms=%.2f' % (d['value'], d['roofline']['frac'] or 0, d['ms_per_step']))" 2>/dev/null || echo "$w $v FAILED"
done; done
