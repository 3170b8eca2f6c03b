#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2h_ab.jsonl; : > $O
for C in google8_ring google8_dgx1 reddit_dgx1; do
  for B in 1 2 4 8; do
    timeout 600 python tools/ab_rt.py $C --build pipeline_blocks=$B "item_order=0" "item_order=3" >> $O 2>>gpurun_out/r2h_ab.err
  done
done
for C in google2 google4 reddit orkut; do
  timeout 600 python tools/ab_rt.py $C "item_order=4" >> $O 2>>gpurun_out/r2h_ab.err
done
cat $O | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    print(d['config'], d['build'])
    for s in d['sets']: print('   ', s['opts'], s['ms'])
"
TAG=r2h PYT=2400 bash tools/gpu_tests.sh
