#!/bin/bash
# Multi-rank flow of bench.py on ONE GPU (both ranks on cuda:0, gloo for the
# exchange): barriers, max-over-ranks timing, summed flips, rank-0 JSON line,
# lockstep and async exchange, and the reference arm under torchrun.
export ABS_BENCH_BACKEND=gloo ABS_BENCH_DEVICE=0
R="python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1"
mkdir -p gpurun_out
timeout 600 $R --master-port 29611 bench.py --gpus 2 --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/mr_random32k.json 2> gpurun_out/mr.err; echo "random32k rc=$?"
timeout 300 $R --master-port 29612 bench.py --gpus 2 --workload maxcut2k --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/mr_maxcut2k.json 2>> gpurun_out/mr.err; echo "maxcut2k rc=$?"
timeout 300 $R --master-port 29613 bench.py --gpus 2 --workload maxcut2k --mode async --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/mr_maxcut2k_async.json 2>> gpurun_out/mr.err; echo "maxcut2k async rc=$?"
timeout 300 $R --master-port 29614 bench.py --gpus 2 --impl reference --steps 1 --warmup 0 --ref-step-seconds 2 > gpurun_out/mr_ref.json 2>> gpurun_out/mr.err; echo "reference rc=$?"
for f in mr_random32k mr_maxcut2k mr_maxcut2k_async mr_ref; do echo "$f: $(wc -l < gpurun_out/$f.json) line(s)"; cut -c1-400 gpurun_out/$f.json; done
tail -5 gpurun_out/mr.err
