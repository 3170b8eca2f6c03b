#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
for c in reddit_dgx1 google8_ring; do
  timeout 300 python tools/relay_timeline.py $c 10
  timeout 300 python tools/relay_timeline.py $c 10 leaf_split=2
done > gpurun_out/r2sn_timeline.txt 2> gpurun_out/r2sn_timeline.err
tail -3 gpurun_out/r2sn_timeline.err
