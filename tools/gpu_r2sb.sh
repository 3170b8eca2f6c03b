#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
for c in google8_ring google8_dgx1; do
  timeout 300 python tools/relay_timeline.py $c 10 | grep -A20 "per stage"
done > gpurun_out/r2sb_timeline.txt 2> gpurun_out/r2sb_timeline.err
tail -3 gpurun_out/r2sb_timeline.err
