#!/bin/bash
# dual producer warps for simple copy launches: parity tests, then A/B
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
true || timeout 600 python -m pytest tests/test_gpu_exec.py -q -x -k "tiny or uniform or full_size_every_row and (reddit or google2)" > gpurun_out/r2su_pytest.log 2>&1; tail -2 gpurun_out/r2su_pytest.log
O=gpurun_out/r2su_ab.txt; : > $O
for rep in 1 2; do
for cfg in reddit google2 google4 google8 orkut; do
  timeout 300 python tools/ab_rt.py $cfg "dual_producer=0" "dual_producer=1" 2>>gpurun_out/r2su_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
for s in d['sets']: print('$cfg'.ljust(9), s['opts'], s['ms'])" >> $O
done
done
cat $O
