#!/bin/bash
# WIDE geometry with dual producers: 3 x 64 KB (default) vs 4 x 48 / 4 x 47 KB stages
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2tf_ab.txt; : > $O
for rep in 1 2 3; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/w4x48.so build/ab/w4x47.so; do
    DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py reddit "" 2>>gpurun_out/r2tf_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$(basename $L)'.ljust(12), d['sets'][0]['ms'])" >> $O
  done
done
DGCL_LIBRARY=$PWD/build/ab/w4x48.so timeout 600 python -m pytest tests/test_gpu_exec.py -q -x -k "uniform and (602 or geometry)" > gpurun_out/r2tf_pytest.log 2>&1; tail -1 gpurun_out/r2tf_pytest.log
cat $O
