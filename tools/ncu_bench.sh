#!/bin/bash
# ncu evidence for the bench's executor launches (1 GPU).  Numbers printed under ncu are not bench values.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
TAG=${TAG:-r1}
make -s all > gpurun_out/build.log 2>&1 || exit 1
CFG=${CFG:-reddit}
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${TAG}_launches.csv \
  python bench.py --config $CFG --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-torch-baseline --no-per-rank > gpurun_out/${TAG}_launches_bench.json 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:executor -c ${NCU_COUNT:-3} \
  -o gpurun_out/${TAG}_prof -f \
  python bench.py --config $CFG --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-torch-baseline --no-per-rank > gpurun_out/${TAG}_prof_bench.log 2>&1
ls -la gpurun_out
