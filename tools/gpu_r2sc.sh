#!/bin/bash
# relay item order (relay_lead_kb) + flush-before-non-signalling A/B, relay GPU tests, timelines
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_exec.py -q -x -k "relay or trace or random_option" > gpurun_out/r2sc_pytest.log 2>&1; tail -2 gpurun_out/r2sc_pytest.log
for rep in 1 2; do
for cfg in google8_ring google8_dgx1 reddit_dgx1; do
  for b in relay_lead_kb=-1 relay_lead_kb=0 relay_lead_kb=16384 relay_lead_kb=65536 relay_lead_kb=196608 leaf_split=2,relay_lead_kb=65536 leaf_split=2,relay_lead_kb=196608; do
    timeout 300 python tools/ab_rt.py $cfg "" --build $b 2>>gpurun_out/r2sc_ab.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg $b', d['sets'][0]['ms'])"
  done
done
done | tee gpurun_out/r2sc_ab.txt
for c in google8_ring google8_dgx1; do
  timeout 300 python tools/relay_timeline.py $c 10
done > gpurun_out/r2sc_timeline.txt 2> gpurun_out/r2sc_timeline.err
