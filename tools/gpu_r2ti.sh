#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2ti_ab.txt; : > $O
for rep in 1 2; do
for cfg in google2 google4 google8 orkut reddit reddit_dgx1 google8_dgx1; do
  timeout 300 python tools/ab_rt.py $cfg "" 2>>gpurun_out/r2ti_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
for s in d['sets']: print('$cfg'.ljust(13), s['ms'])" >> $O
done
done
cat $O
