#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
: > gpurun_out/r2x_relay_trace.log
for C in google8_ring google8_dgx1 reddit_dgx1; do
  timeout 300 python tools/relay_trace.py $C >> gpurun_out/r2x_relay_trace.log 2>&1
done
grep -E "launch|stage [0-9] ops" gpurun_out/r2x_relay_trace.log
O=gpurun_out/r2x_ab.jsonl; : > $O
for C in google8_ring reddit_dgx1; do
  for B in 1 2 4; do
    timeout 600 python tools/ab_rt.py $C --build pipeline_blocks=$B "" "claim_batch=8" >> $O 2>>gpurun_out/r2x_ab.err
  done
done
cat $O | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    print(d['config'], d['build'])
    for s in d['sets']: print('   ', s['opts'], s['ms'])
"
