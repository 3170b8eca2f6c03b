#!/bin/bash
# one bulk store per row for scattered destinations (relay stages) vs consumer STG
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2so_ab.txt; : > $O
for rep in 1 2; do
for cfg in google8_ring google8_dgx1 reddit_dgx1; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/rb512.so build/ab/rb1024.so; do
    DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py $cfg "" 2>>gpurun_out/r2so_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$(basename $L)'.ljust(12), '$cfg'.ljust(13), d['sets'][0]['ms'])" >> $O
  done
done
done
cat $O
