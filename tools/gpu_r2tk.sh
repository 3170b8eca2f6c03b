#!/bin/bash
# dual producers with dynamic claims: parity (library built with dual_claims on), then A/B
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
DGCL_LIBRARY=$PWD/build/ab/dualclaims.so timeout 1500 python -m pytest tests/test_gpu_exec.py tests/test_gpu_multiproc.py -q -x -k "not full_size or google2 or google4" > gpurun_out/r2tk_pytest.log 2>&1; tail -1 gpurun_out/r2tk_pytest.log
O=gpurun_out/r2tk_ab.txt; : > $O
for rep in 1 2; do
for cfg in google2 google4; do
  for b in geometry=0 geometry=1; do
    timeout 300 python tools/ab_rt.py $cfg "dual_claims=0" "dual_claims=1" --build $b 2>>gpurun_out/r2tk_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
for s in d['sets']: print('$cfg'.ljust(8), '$b', s['opts'], s['ms'])" >> $O
  done
done
done
cat $O
