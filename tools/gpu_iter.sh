# One iteration of a kernel change on the GPU box: GPU tests (or a subset: TESTS), A/B bench of
# the working tree's library against libabs_old.so (WORKLOADS, VARIANTS), and an ncu --set full
# capture of the one-warp round kernel at n = 1024 (NCU=0 skips it).  Outputs in gpurun_out/.
set -u
OUT=gpurun_out
mkdir -p $OUT
timeout 1200 python -m pytest ${TESTS:-tests} -m gpu -x -q --timeout 600 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu.log
WORKLOADS="${WORKLOADS:-random1k maxcut2k}" VARIANTS="${VARIANTS:-new old new old}" BENCH_ARGS="${BENCH_ARGS:---steps 200 --no-sub}" bash tools/ab_bench.sh
if [ "${NCU:-1}" = 1 ]; then
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:round_kernel -s 2 -c 1 \
    -o $OUT/prof_round1k python tools/prof_round.py --n 1024 --searches 10000 --steps 3 > $OUT/prof_round1k.log 2>&1; echo "ncu-full-1k rc=$?"
fi
