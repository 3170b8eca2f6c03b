#!/bin/bash
# source-level ncu of the Reddit dim-602 forward at the final code (dual producers)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 ncu --set full --clock-control none --import-source on -k regex:executor --launch-skip 2 -c 1 \
  -o gpurun_out/r2ts_reddit_fwd python tools/one_launch.py reddit 0 0 3 > gpurun_out/r2ts.log 2>&1
ncu -i gpurun_out/r2ts_reddit_fwd.ncu-rep --page source --csv --print-source sass > gpurun_out/r2ts_reddit_sass.csv 2>/dev/null
ncu -i gpurun_out/r2ts_reddit_fwd.ncu-rep --page raw --csv > gpurun_out/r2ts_reddit_raw.csv 2>/dev/null
rm -f gpurun_out/r2ts_reddit_fwd.ncu-rep
ls -la gpurun_out/r2ts*
