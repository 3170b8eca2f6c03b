#!/bin/bash
# leaf split A/B (relay forwards) + relay / trace GPU tests
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_exec.py -q -k "relay or trace or random_option" > gpurun_out/r2ab_pytest.log 2>&1; tail -3 gpurun_out/r2ab_pytest.log
for rep in 1 2; do
for cfg in google8_ring google8_dgx1 reddit_dgx1; do
  for ls in 0 1 2; do
    timeout 300 python tools/ab_rt.py $cfg "" --build leaf_split=$ls 2>>gpurun_out/r2ab_ab.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg leaf_split=$ls', d['sets'][0]['ms'])"
  done
  timeout 300 python tools/ab_rt.py $cfg "" --build leaf_split=2,fanout=1 2>>gpurun_out/r2ab_ab.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg leaf_split=2,fanout=1', d['sets'][0]['ms'])"
done
done | tee gpurun_out/r2ab_ab.txt
