set -u
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:round_kernel -s 2 -c 1 \
    -o gpurun_out/prof_w1k python tools/prof_round.py --n 1024 --searches 10000 --steps 3 > gpurun_out/prof_w1k.log 2>&1; echo "ncu-1k rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:round_kernel -s 2 -c 1 \
    -o gpurun_out/prof_w2k python tools/prof_round.py --n 2000 --searches 2368 --steps 3 --workload maxcut > gpurun_out/prof_w2k.log 2>&1; echo "ncu-2k rc=$?"
