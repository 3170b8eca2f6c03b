#!/bin/bash
# store split / fixed vs rotating store warps, with dual producers (the gather side no longer bounds)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2sw_ab.txt; : > $O
for rep in 1 2; do
for cfg in reddit orkut google8; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/s1r.so build/ab/s2r.so build/ab/s3r.so build/ab/s1f.so build/ab/s2f.so build/ab/s6f.so; do
    DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py $cfg "" 2>>gpurun_out/r2sw_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$(basename $L)'.ljust(12), '$cfg'.ljust(8), d['sets'][0]['ms'])" >> $O
  done
done
done
cat $O
