#!/bin/bash
# tiny config (register executor, latency-bound): CTA shape
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2tm_ab.txt; : > $O
for rep in 1 2; do
  for b in threads=512 ctas_per_sm=1 threads=256 threads=256,ctas_per_sm=1 threads=128,ctas_per_sm=1 small_launch_bytes=0; do
    timeout 300 python tools/ab_rt.py tiny "" --build $b 2>>gpurun_out/r2tm_ab.err | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('tiny', '$b'.ljust(28), d['sets'][0]['ms'])" >> $O
  done
done
python tools/launch_overhead.py tiny 50 >> $O 2>&1
cat $O
