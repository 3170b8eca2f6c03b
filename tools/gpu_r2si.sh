#!/bin/bash
# fixed store warps: split sweep at the new defaults; then the full GPU suite + smoke
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2si_ab.txt; : > $O
for rep in 1 2; do
for cfg in reddit orkut google8 google8_ring; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/f2.so build/ab/f3.so build/ab/f6.so build/ab/f8.so; do
    DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py $cfg "" 2>>gpurun_out/r2si_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$(basename $L)'.ljust(12), '$cfg'.ljust(13), d['sets'][0]['ms'])" >> $O
  done
done
done
cat $O
TAG=r2si PYT=2400 bash tools/gpu_tests.sh > gpurun_out/r2si_tests_summary.log 2>&1
grep -E "passed|failed" gpurun_out/r2si_pytest_gpu.log | tail -2; tail -1 gpurun_out/r2si_smoke.log
