#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 120 python tools/mc_probe.py > gpurun_out/r2g_mc_probe.txt 2>&1; cat gpurun_out/r2g_mc_probe.txt
nvidia-smi -q | grep -i -A3 "fabric\|multicast" | head -20
O=gpurun_out/r2g_ab.jsonl; : > $O
for C in google2 google4 orkut google8 reddit; do
  timeout 600 python tools/ab_rt.py $C "item_order=0" "item_order=3" "item_order=1" >> $O 2>>gpurun_out/r2g_ab.err
done
cat $O | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    print(d['config'], d['build'])
    for s in d['sets']: print('   ', s['opts'], s['ms'])
"
