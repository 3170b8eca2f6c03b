#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 600 python examples/gcn_overlap.py > gpurun_out/r2j_overlap.json 2> gpurun_out/r2j_overlap.err; cat gpurun_out/r2j_overlap.json; tail -2 gpurun_out/r2j_overlap.err
O=gpurun_out/r2j_ab.jsonl; : > $O
for C in orkut google2 google8 google8_ring reddit_dgx1; do
  for G in 0 1 2; do
    timeout 600 python tools/ab_rt.py $C --build geometry=$G "" "l2_policy=0" >> $O 2>>gpurun_out/r2j_ab.err
  done
done
cat $O | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    print(d['config'], d['build'])
    for s in d['sets']: print('   ', s['opts'], s['ms'])
"
