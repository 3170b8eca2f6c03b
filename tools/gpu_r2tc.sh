#!/bin/bash
# dual producers for staged-fold (backward) launches: parity, then A/B
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_exec.py -q -x -k "uniform or tiny or relay or random_option or full_size_every_row and (reddit or orkut or ring)" > gpurun_out/r2tc_pytest.log 2>&1; tail -2 gpurun_out/r2tc_pytest.log
O=gpurun_out/r2tc_ab.txt; : > $O
for rep in 1 2; do
for cfg in reddit orkut google8 google2 google8_ring reddit_dgx1; do
  timeout 300 python tools/ab_rt.py $cfg "dual_producer=0" "dual_producer=1" 2>>gpurun_out/r2tc_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
for s in d['sets']: print('$cfg'.ljust(13), s['opts'], s['ms'])" >> $O
done
done
cat $O
