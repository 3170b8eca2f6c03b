#!/bin/bash
# sustained bench (bench.py, soaked, power-capped) with and without dual producers
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2td_ab.txt; : > $O
for rep in 1 2; do
for cfg in orkut reddit google8; do
  for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/nodual.so; do
    DGCL_LIBRARY=$PWD/$L timeout 600 python bench.py --config $cfg --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-torch-baseline --no-per-rank 2>>gpurun_out/r2td_ab.err | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read())
print('$(basename $L)'.ljust(12), '$cfg'.ljust(8), 'step %.4f' % d['ms_per_step'], {k: round(v, 4) for k, v in d['ms_per_layer'].items()}, d['clocks']['sm_mhz'])" >> $O
  done
done
done
cat $O
