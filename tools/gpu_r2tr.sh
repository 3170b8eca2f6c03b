#!/bin/bash
# DUAL geometry with dual producers: 2 x 47 KB (default) vs 3 x 31 KB stages per CTA
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2tr_ab.txt; : > $O
for rep in 1 2; do
for cfg in orkut reddit google8 google2; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/d3x31.so; do
    DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py $cfg "" 2>>gpurun_out/r2tr_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$(basename $L)'.ljust(12), '$cfg'.ljust(8), d['sets'][0]['ms'])" >> $O
  done
done
done
cat $O
