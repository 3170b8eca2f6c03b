#!/bin/bash
# bulk-store split / fixed store warps (serialised stores per CTA) A/B
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
O=gpurun_out/r2sg_ab.txt; : > $O
for rep in 1 2; do
for cfg in reddit orkut google8 google2; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/s1f.so build/ab/s2f.so build/ab/s4f.so build/ab/s1r.so build/ab/s4r.so; do
    DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py $cfg "" 2>>gpurun_out/r2sg_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$(basename $L)'.ljust(12), '$cfg'.ljust(8), d['sets'][0]['ms'])" >> $O
  done
done
done
cat $O
