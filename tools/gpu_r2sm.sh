#!/bin/bash
# item order of fused loopback forwards: chunk-major (0) / owner-major (1) / group-major (2)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2sm_ab.txt; : > $O
for rep in 1 2; do
for cfg in reddit orkut google8 google4; do
  for b in owner_major=0 owner_major=1 owner_major=2; do
    timeout 300 python tools/ab_rt.py $cfg "" --build $b 2>>gpurun_out/r2sm_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$cfg'.ljust(13), '$b', d['sets'][0]['ms'])" >> $O
  done
done
done
cat $O
