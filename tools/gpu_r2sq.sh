#!/bin/bash
# blocked owner-major order (owner_major 3, order_block chunks) vs owner-major (1)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2sq_ab.txt; : > $O
for rep in 1 2; do
for cfg in reddit orkut google8 google8_dgx1; do
  for b in owner_major=1 owner_major=3 owner_major=3,order_block=74 owner_major=3,order_block=592 owner_major=3,order_block=32; do
    timeout 300 python tools/ab_rt.py $cfg "" --build $b 2>>gpurun_out/r2sq_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$cfg'.ljust(13), '$b'.ljust(34), d['sets'][0]['ms'])" >> $O
  done
done
done
cat $O
