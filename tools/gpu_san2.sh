set -u
OUT=gpurun_out/sanitizer2
mkdir -p $OUT
for tool in memcheck racecheck synccheck; do for n in 3000 10000; do for mode in lockstep async; do for pol in window sa; do
  timeout 300 /usr/local/cuda/bin/compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 \
    python tools/sanitize_run.py --n $n --mode $mode --policy $pol --searches 2 --local-flips 400 > $OUT/${tool}_n${n}_${mode}_${pol}.log 2>&1
  echo "$tool n=$n $mode $pol rc=$?" >> $OUT/summary.txt
done; done; done; done
cat $OUT/summary.txt
