#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_exec.py -q -x -k "uniform_loopback_fused or relay" > gpurun_out/r2p_pytest.log 2>&1; tail -2 gpurun_out/r2p_pytest.log
O=gpurun_out/r2p_ab.jsonl; : > $O
for C in orkut google8 google2 google4 reddit google8_ring; do
  timeout 600 python tools/ab_rt.py $C --build lsu_gather=0 "" >> $O 2>>gpurun_out/r2p_ab.err
  timeout 600 python tools/ab_rt.py $C --build lsu_gather=1 "" >> $O 2>>gpurun_out/r2p_ab.err
done
cat $O | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    print(d['config'], d['build'], d['sets'][0]['ms'])
"
