#!/bin/bash
# with 4 x 48 KB WIDE + dual producers: geometry auto vs WIDE forced; GPU test subset
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests/test_gpu_exec.py tests/test_gpu_multiproc.py -q -x -k "not full_size" > gpurun_out/r2tg_pytest.log 2>&1; tail -1 gpurun_out/r2tg_pytest.log
O=gpurun_out/r2tg_ab.txt; : > $O
for rep in 1 2; do
for cfg in reddit google8 orkut google2; do
  for b in geometry=0 geometry=1; do
    timeout 300 python tools/ab_rt.py $cfg "" --build $b 2>>gpurun_out/r2tg_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$cfg'.ljust(8), '$b', d['sets'][0]['ms'])" >> $O
  done
done
done
cat $O
