#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2n_ab.jsonl; : > $O
for C in google8_ring google8_dgx1 reddit_dgx1 google2 google4 orkut reddit google8; do
  timeout 600 python tools/ab_rt.py $C "claim_batch=0" "claim_batch=1" "claim_batch=2" "claim_batch=4" "claim_batch=8" >> $O 2>>gpurun_out/r2n_ab.err
done
cat $O | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    print(d['config'], d['build'])
    for s in d['sets']: print('   ', s['opts'], s['ms'])
"
timeout 900 python -m pytest tests/test_gpu_exec.py -q -x -k "relay or wait_arrival or per_rank or sixteen or trace" > gpurun_out/r2n_pytest.log 2>&1; tail -3 gpurun_out/r2n_pytest.log
