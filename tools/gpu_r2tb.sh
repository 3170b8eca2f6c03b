#!/bin/bash
# source-level ncu of the Reddit dim-256 backward (staged folds): is its producer the bound?
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 ncu --set full --clock-control none --import-source on -k regex:executor --launch-skip 2 -c 1 \
  -o gpurun_out/r2tb_reddit_bwd python tools/one_launch.py reddit 1 1 3 > gpurun_out/r2tb.log 2>&1
ncu -i gpurun_out/r2tb_reddit_bwd.ncu-rep --page source --csv --print-source sass > gpurun_out/r2tb_reddit_bwd_sass.csv 2>/dev/null
rm -f gpurun_out/r2tb_reddit_bwd.ncu-rep
ls -la gpurun_out/r2tb*
