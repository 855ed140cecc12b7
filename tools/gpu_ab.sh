# A/B of library variants: WORKLOADS, VARIANTS, BENCH_ARGS from the environment
set -u
mkdir -p gpurun_out
WORKLOADS="${WORKLOADS:-random1k maxcut2k}" VARIANTS="${VARIANTS:-new old}" BENCH_ARGS="${BENCH_ARGS:---steps 20 --no-sub}" bash tools/ab_bench.sh
