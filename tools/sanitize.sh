#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over small runs of every
# round-kernel family (one warp: n=100, 1100; multi-warp: n=3000) in lockstep
# and async mode, window and SA policies.  Run under gpurun; logs in gpurun_out/.
set -u
OUT=gpurun_out/sanitizer
mkdir -p $OUT
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck; do
  for n in 100 1100 3000; do
    for mode in lockstep async; do
      for pol in window sa; do
        f=$OUT/${tool}_n${n}_${mode}_${pol}.log
        timeout 240 $CS --tool $tool --error-exitcode 9 --print-limit 20 \
          python tools/sanitize_run.py --n $n --mode $mode --policy $pol > $f 2>&1
        echo "$tool n=$n $mode $pol rc=$?" | tee -a $OUT/summary.txt
      done
    done
  done
done
