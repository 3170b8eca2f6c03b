#!/bin/bash
# bench.py on every BASELINE config (1-GPU loopback), one JSON line each -> gpurun_out/bench_all.jsonl
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || exit 1
: > gpurun_out/bench_all.jsonl
for C in ${CFGS:-tiny reddit google2 google4 google8 orkut google8_dgx1 google8_ring reddit_dgx1}; do
  timeout 900 python bench.py --config $C --steps ${STEPS:-10} --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-per-rank \
     ${EXTRA:-} >> gpurun_out/bench_all.jsonl 2> gpurun_out/bench_$C.err
  echo "$C rc=$?"
done
python3 - <<'PY'
import json
for line in open('gpurun_out/bench_all.jsonl'):
    d = json.loads(line)
    r = d['roofline']
    print(d['config']['config'], 'ms/step %.3f' % d['ms_per_step'], 'GB/s %.0f' % d['value'],
          {k: round(v, 3) for k, v in d['ms_per_layer'].items()},
          {k: round(v['frac'], 3) for k, v in r['per_kernel'].items()},
          {k: round(v['plan_frac'], 3) for k, v in r['per_kernel'].items() if 'plan_frac' in v},
          'stages', d['plan']['n_stages'], 'plan_s %.2f' % d['plan']['planner_seconds'],
          'gen_s %.1f' % d['plan']['graph_gen_s'])
PY
