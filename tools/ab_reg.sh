#!/bin/bash
# A/B of library builds on the register (LDG/STG) executor: LIBS="a.so b.so" CFGS="orkut" OPTS="tma=0"
cd "$(dirname "$0")/.."
for rep in 1 2; do
  for C in ${CFGS:-orkut}; do
    for lib in ${LIBS:-paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so}; do
      DGCL_LIBRARY=$PWD/$lib timeout 600 python bench.py --config $C --steps 10 --warmup 3 --e2e-steps 0 \
        --no-cpu-baseline --no-torch-baseline $(for o in ${OPTS:-tma=0}; do echo --opt $o; done) 2>/dev/null |
        python3 -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$lib $C', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['ms_per_layer'].items()}, {k: round(v['frac'],3) for k,v in d['roofline']['per_kernel'].items()})"
    done
  done
done
