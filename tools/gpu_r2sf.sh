#!/bin/bash
# store path: L2 hints / TMA bulk stores vs STG, full pipeline and stores only (nogather)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
O=gpurun_out/r2sf_ab.txt; : > $O
for cfg in reddit orkut; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/nogather.so; do
    for b in l2_policy=1 l2_policy=0 bulk_store=0,l2_policy=1 bulk_store=0,l2_policy=0; do
    DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py $cfg "" --build $b 2>>gpurun_out/r2sf_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$(basename $L) $cfg $b', d['sets'][0]['ms'])" >> $O
    done
  done
done
cat $O
