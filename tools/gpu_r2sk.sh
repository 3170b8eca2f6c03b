#!/bin/bash
# source-level ncu of the Reddit fwd602 and Com-Orkut forward launches at the current defaults
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
python tools/one_launch.py reddit 0 0 3 && python tools/one_launch.py orkut 0 0 3 || exit 1
for c in "reddit 0" "orkut 0"; do
  set -- $c
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:executor --launch-skip 2 -c 1 \
    -o gpurun_out/r2sk_$1_fwd python tools/one_launch.py $1 $2 0 3 > gpurun_out/r2sk_$1.log 2>&1
  ncu -i gpurun_out/r2sk_$1_fwd.ncu-rep --page source --csv --print-source sass > gpurun_out/r2sk_$1_sass.csv 2>/dev/null
  ncu -i gpurun_out/r2sk_$1_fwd.ncu-rep --page raw --csv > gpurun_out/r2sk_$1_raw.csv 2>/dev/null
done
ls -la gpurun_out/r2sk_*
