#!/bin/bash
# Build the library of git revision $1 (default HEAD) as libabs_old.so (A/B runs: tools/ab_bench.sh).
set -e
REV=${1:-HEAD}
D=$(mktemp -d)
git archive $REV paper_conf_icpp_yasudonitkyi20_b200/csrc include | tar -x -C $D
C=$D/paper_conf_icpp_yasudonitkyi20_b200/csrc
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -shared -Xcompiler -fPIC \
  -Xcompiler -fvisibility=hidden -Xcompiler -fopenmp -I $D/include -I $C -o paper_conf_icpp_yasudonitkyi20_b200/libabs_old.so \
  $(ls $C/*.cu $C/*.cpp) -lpthread -lgomp
rm -rf $D
