#!/bin/bash
# relay forward timelines (stage boundaries) at the current defaults
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
for c in google8_ring google8_dgx1 reddit_dgx1; do
  timeout 300 python tools/relay_timeline.py $c 10
done > gpurun_out/r2sa_timeline.txt 2> gpurun_out/r2sa_timeline.err
timeout 300 python tools/relay_timeline.py google8_ring 10 claim_batch=1 >> gpurun_out/r2sa_timeline.txt 2>> gpurun_out/r2sa_timeline.err
timeout 300 python tools/relay_timeline.py google8_ring 10 geometry=1 >> gpurun_out/r2sa_timeline.txt 2>> gpurun_out/r2sa_timeline.err
tail -3 gpurun_out/r2sa_timeline.err
