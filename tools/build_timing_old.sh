#!/bin/bash
# Build the diagnostics (-DABS_TIMING) library of git revision $1 (default HEAD) as libabs_timing_old.so.
set -e
REV=${1:-HEAD}
D=$(mktemp -d)
git archive $REV paper_conf_icpp_yasudonitkyi20_b200/csrc include | tar -x -C $D
C=$D/paper_conf_icpp_yasudonitkyi20_b200/csrc
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -DABS_TIMING -O3 -lineinfo -std=c++17 -shared -Xcompiler -fPIC \
  -Xcompiler -fvisibility=hidden -I $D/include -I $C -o paper_conf_icpp_yasudonitkyi20_b200/libabs_timing_old.so \
  $(ls $C/*.cu $C/*.cpp) -lpthread
rm -rf $D
