#!/bin/bash
# Build an A/B variant of libdgcl.so with extra compile definitions:
#   tools/build_variant.sh NAME "-DDGCL_TMA_STAGES=2 -DDGCL_TMA_STAGE_KB=47 ..."  -> build/ab/NAME.so
# (load it with DGCL_LIBRARY=$PWD/build/ab/NAME.so; see tools/ab.sh)
set -e
cd "$(dirname "$0")/.."
NAME=$1; FLAGS=$2
PKG=paper_conf_eurosys_cai0wmcy21_b200
O=build/ab/$NAME; mkdir -p $O
NV="nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC -Iinclude $FLAGS"
for f in planner lowering api hostsim; do
  g++ -O3 -std=c++17 -fPIC -Iinclude -I/usr/local/cuda/include $FLAGS -c $PKG/csrc/$f.cpp -o $O/$f.o &
done
$NV -c $PKG/csrc/executor.cu -o $O/executor.o &
$NV -Xptxas -v -c $PKG/csrc/executor_tma.cu -o $O/executor_tma.o 2> $O/ptxas.log &
wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -Xcompiler -fPIC -cudart static $O/*.o -o build/ab/$NAME.so
echo built build/ab/$NAME.so
