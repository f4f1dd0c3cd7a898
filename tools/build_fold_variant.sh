#!/bin/bash
# Builds paper_conf_dsn_zhaoxcqzj24_b200/libowl_<name>.so with <fold.cu> in place of csrc/owl_fold.cu (fold
# experiments; select at run time with OWL_LIBOWL_PATH).  usage: tools/build_fold_variant.sh name fold.cu [flags]
set -e
cd "$(dirname "$0")/.."
NAME=$1; SRC=$2; FLAGS=$3
C=paper_conf_dsn_zhaoxcqzj24_b200/csrc
T=$(mktemp -d)
cp "$SRC" $T/owl_fold.cu
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -fmad=false $FLAGS -Xptxas -v -Xcompiler -fPIC,-fvisibility=hidden -I include -I $C -c $T/owl_fold.cu -o $T/owl_fold.o 2> $T/ptxas.txt
grep -A2 fold_kernel $T/ptxas.txt | grep -E "spill|registers" | sed "s/^/$NAME: /"
for s in $C/*.cu; do
  [ "$(basename $s)" = owl_fold.cu ] && continue
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -fmad=false -Xcompiler -fPIC,-fvisibility=hidden -I include -I $C -c $s -o $T/$(basename $s).o
done
for s in $C/*.cpp; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Xcompiler -fPIC,-fvisibility=hidden -I include -I $C -c $s -o $T/$(basename $s).o
done
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o paper_conf_dsn_zhaoxcqzj24_b200/libowl_$NAME.so $T/*.o -lcudart
rm -rf $T
