#!/bin/bash
# Build the working tree's library with extra nvcc flags as libabs_$1.so (A/B runs: tools/ab_bench.sh VARIANTS=...)
set -e
NAME=$1; shift
C=paper_conf_icpp_yasudonitkyi20_b200/csrc
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -shared -Xcompiler -fPIC \
  -Xcompiler -fvisibility=hidden -Xcompiler -fopenmp -I include -I $C "$@" -o paper_conf_icpp_yasudonitkyi20_b200/libabs_$NAME.so \
  $C/abs_round.cu $C/abs_round_warp.cu $C/abs_setup.cu $C/abs_init_mma.cu $C/abs_host.cpp -lpthread -lgomp
