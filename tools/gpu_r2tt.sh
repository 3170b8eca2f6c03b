#!/bin/bash
# WIDE with dual producers: 4 x 48 KB (default) vs 5 x 38 / 5 x 37 KB stages
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2tt_ab.txt; : > $O
for rep in 1 2 3; do
for cfg in reddit google8; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/w5x38.so build/ab/w5x37.so; do
    DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py $cfg "" 2>>gpurun_out/r2tt_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$(basename $L)'.ljust(12), '$cfg'.ljust(8), d['sets'][0]['ms'])" >> $O
  done
done
done
DGCL_LIBRARY=$PWD/build/ab/w5x38.so timeout 900 python -m pytest tests/test_gpu_exec.py -q -x -k "uniform or tiny or full_size_every_row and reddit" > gpurun_out/r2tt_pytest.log 2>&1; tail -1 gpurun_out/r2tt_pytest.log
cat $O
