#!/bin/bash
# diagnostic builds: gathers only (nostore) / stores only (nogather) vs the full pipeline
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
O=gpurun_out/r2se_ab.txt; : > $O
for cfg in reddit orkut google8; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/nogather.so build/ab/nostore.so; do
    for geo in 0 1 2; do
      DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py $cfg "" --build geometry=$geo 2>>gpurun_out/r2se_ab.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$(basename $L) $cfg geometry=$geo', d['sets'][0]['ms'])" >> $O
    done
  done
done
cat $O
