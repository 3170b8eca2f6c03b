#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2e_ab.jsonl; : > $O
for C in google2 orkut google8 reddit google4 google8_ring google8_dgx1 reddit_dgx1; do
  timeout 600 python tools/ab_rt.py $C "dynamic_items=0,l2_policy=0" "dynamic_items=1,l2_policy=0" "dynamic_items=1,l2_policy=1" "dynamic_items=0,l2_policy=1" >> $O 2>>gpurun_out/r2e_ab.err
done
cat $O | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    print(d['config'], d['build'])
    for s in d['sets']: print('   ', s['opts'], s['ms'])
"
TAG=r2e PYT=2400 bash tools/gpu_tests.sh
