#!/bin/bash
# share of each bulk-store COPY stage stored with LDS + STG by the non-store consumer warps
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2sj_ab.txt; : > $O
for rep in 1 2; do
for cfg in reddit orkut google8 google8_ring; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/stg20.so build/ab/stg35.so build/ab/stg50.so; do
    DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py $cfg "" 2>>gpurun_out/r2sj_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$(basename $L)'.ljust(12), '$cfg'.ljust(13), d['sets'][0]['ms'])" >> $O
  done
done
done
cat $O
O2=gpurun_out/r2sj_geo.txt; : > $O2
for cfg in reddit orkut google8; do
  for b in geometry=0 geometry=1 geometry=2; do
    timeout 300 python tools/ab_rt.py $cfg "" --build $b 2>>gpurun_out/r2sj_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$cfg'.ljust(13), '$b', d['sets'][0]['ms'])" >> $O2
  done
done
cat $O2
