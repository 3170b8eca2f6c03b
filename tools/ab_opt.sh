#!/bin/bash
# A/B of library options on the same box: OPTS="fanout=0 fanout=1,geometry=2" CFGS="reddit orkut" tools/ab_opt.sh
cd "$(dirname "$0")/.."
for rep in 1 2; do
  for C in ${CFGS:-reddit}; do
    for o in ${OPTS:-fanout=0 fanout=1}; do
      timeout 600 python bench.py --config $C --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline \
        --no-torch-baseline $(echo "$o" | tr "," "\n" | sed "s/^/--opt /") 2>/dev/null | python3 -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$o $C', round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['ms_per_layer'].items()}, {k: round(v['frac'],3) for k,v in d['roofline']['per_kernel'].items()})"
    done
  done
done
