#!/bin/bash
# with dual producers: geometry of Reddit fwd256, diagnostic builds (stores only / gathers only)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2sv_ab.txt; : > $O
for rep in 1 2; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/nogather.so build/ab/nostore.so; do
    for b in geometry=0 geometry=1; do
      DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py reddit "" --build $b 2>>gpurun_out/r2sv_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$(basename $L)'.ljust(14), '$b', d['sets'][0]['ms'])" >> $O
    done
  done
done
cat $O
