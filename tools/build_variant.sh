#!/bin/bash
# Builds paper_conf_dsn_zhaoxcqzj24_b200/libowl_<name>.so with extra nvcc flags for the fold kernel (experiments;
# select at run time with OWL_LIBOWL_PATH).  usage: tools/build_variant.sh name "-DNWARP=12 -DPF=6"
set -e
cd "$(dirname "$0")/.."
NAME=$1; FLAGS=$2
C=paper_conf_dsn_zhaoxcqzj24_b200/csrc
T=$(mktemp -d)
for s in $C/*.cu; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -fmad=false $FLAGS -Xcompiler -fPIC,-fvisibility=hidden -I include -I $C -c $s -o $T/$(basename $s).o
done
for s in $C/*.cpp; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Xcompiler -fPIC,-fvisibility=hidden -I include -I $C -c $s -o $T/$(basename $s).o
done
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o paper_conf_dsn_zhaoxcqzj24_b200/libowl_$NAME.so $T/*.o -lcudart
rm -rf $T
