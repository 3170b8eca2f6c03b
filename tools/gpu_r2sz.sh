#!/bin/bash
# dual producers for gather4 launches (Com-Orkut, Web-Google-8): parity, then A/B
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_exec.py -q -x -k "uniform or tiny or random_option or full_size_every_row and (orkut or google8)" > gpurun_out/r2sz_pytest.log 2>&1; tail -2 gpurun_out/r2sz_pytest.log
O=gpurun_out/r2sz_ab.txt; : > $O
for rep in 1 2; do
for cfg in orkut google8 reddit; do
  timeout 300 python tools/ab_rt.py $cfg "dual_producer=0" "dual_producer=1" 2>>gpurun_out/r2sz_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
for s in d['sets']: print('$cfg'.ljust(8), s['opts'], s['ms'])" >> $O
done
done
cat $O
