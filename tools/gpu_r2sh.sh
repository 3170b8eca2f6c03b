#!/bin/bash
# owner-major item order (fused loopback forwards) x store split (default 15 rotating / s4f)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
O=gpurun_out/r2sh_ab.txt; : > $O
for rep in 1 2; do
for cfg in reddit orkut google8 google4 google2 google8_dgx1; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/s4f.so; do
    for b in owner_major=0 owner_major=1; do
    DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py $cfg "" --build $b 2>>gpurun_out/r2sh_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$(basename $L)'.ljust(12), '$cfg'.ljust(13), '$b', d['sets'][0]['ms'])" >> $O
    done
  done
done
done
cat $O
