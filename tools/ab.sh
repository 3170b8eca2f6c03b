#!/bin/bash
# A/B: compare library builds (LIBS, default: build/ab/old.so and the in-tree one), same box
cd "$(dirname "$0")/.."
LIBS=${LIBS:-"build/ab/old.so paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so"}
for rep in 1 2; do
  for lib in $LIBS; do
    for C in ${CFGS:-reddit}; do
    DGCL_LIBRARY=$PWD/$lib timeout 600 python bench.py --config $C --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline 2>/dev/null | python3 -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$lib $C', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['ms_per_layer'].items()})"
    done
  done
done
