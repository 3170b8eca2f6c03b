#!/bin/bash
# every consumer thread waits for its bulk groups at FLUSH (libdgcl) vs lane 0 only (lane0)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2ss_ab.txt; : > $O
for rep in 1 2; do
for cfg in google8_ring google8_dgx1 reddit_dgx1 reddit; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/lane0.so; do
    DGCL_LIBRARY=$PWD/$L timeout 300 python tools/ab_rt.py $cfg "" 2>>gpurun_out/r2ss_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$(basename $L)'.ljust(12), '$cfg'.ljust(13), d['sets'][0]['ms'])" >> $O
  done
done
done
cat $O
timeout 1200 python -m pytest tests/test_gpu_exec.py -q -x -k "relay or trace or random_option or fanout or atomic" > gpurun_out/r2ss_pytest.log 2>&1; tail -2 gpurun_out/r2ss_pytest.log
