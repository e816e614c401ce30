#!/bin/bash
# usage: build_variant.sh NAME "NVCC FLAGS" -> variants/NAME/libtsg.so (select with TSG_LIBRARY=...)
set -e
set -o pipefail
NAME=$1; FLAGS=$2
D=variants/$NAME; mkdir -p $D/obj
pids=()
for f in paper_conf_ppopp_niuljs0022_b200/csrc/*.cu; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-fvisibility=hidden -Iinclude --expt-relaxed-constexpr $FLAGS -c $f -o $D/obj/$(basename $f .cu).o &
  pids+=($!)
done
for p in "${pids[@]}"; do wait $p; done
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $D/libtsg.so $D/obj/*.o -lcudart
rm -rf $D/obj
echo built $D/libtsg.so
