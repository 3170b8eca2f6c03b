#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2k_ab.jsonl; : > $O
for C in google8_dgx1 google8_ring reddit_dgx1; do
  for rep in 1 2; do
    for G in 0 2; do
      timeout 600 python tools/ab_rt.py $C --build geometry=$G "" >> $O 2>>gpurun_out/r2k_ab.err
    done
  done
done
cat $O | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    print(d['config'], d['build'], d['sets'][0]['ms'])
"
# source-level profile of the Com-Orkut forward (one launch), kept for reading here
timeout 900 ncu --set full --clock-control none --import-source on -k regex:executor -c 1 \
  -o gpurun_out/r2k_orkut_fwd -f python bench.py --config orkut --steps 1 --warmup 3 --e2e-steps 0 \
  --no-cpu-baseline --no-torch-baseline > gpurun_out/r2k_orkut_prof.log 2>&1
ncu -i gpurun_out/r2k_orkut_fwd.ncu-rep --page source --csv --print-source sass > gpurun_out/r2k_orkut_sass.csv 2>/dev/null
ncu -i gpurun_out/r2k_orkut_fwd.ncu-rep --page source --csv --print-source cuda > gpurun_out/r2k_orkut_src.csv 2>/dev/null
ls -la gpurun_out/r2k_orkut*; du -sh gpurun_out
