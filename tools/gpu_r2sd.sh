#!/bin/bash
# fence after acquires only (libdgcl.so) vs every waiting item (fencealways.so); relay lead sizes
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
O=gpurun_out/r2sd_ab.txt; : > $O
for rep in 1 2; do
for cfg in google8_ring google8_dgx1 reddit_dgx1; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/fencealways.so; do
    for b in relay_lead_kb=65536 relay_lead_kb=196608 relay_lead_kb=393216; do
      DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py $cfg "" --build $b 2>>gpurun_out/r2sd_ab.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$(basename $L) $cfg $b', d['sets'][0]['ms'])" >> $O
    done
  done
done
done
cat $O
