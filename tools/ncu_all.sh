#!/bin/bash
# ncu --set full of every executor launch of one bench step, for every config (1 GPU loopback),
# plus the bench line of each (for the algorithmic bytes) -> gpurun_out/${TAG}_<cfg>_prof.ncu-rep
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
TAG=${TAG:-r2}
make -s all > gpurun_out/build.log 2>&1 || exit 1
for C in ${CFGS:-tiny reddit google2 google4 google8 orkut google8_dgx1 google8_ring reddit_dgx1}; do
  timeout 900 python bench.py --config $C --steps ${STEPS:-10} --warmup 3 --e2e-steps 0 --no-cpu-baseline \
     --no-torch-baseline ${EXTRA:-} > gpurun_out/${TAG}_${C}_bench.json 2> gpurun_out/${TAG}_${C}_bench.err
  N=$(python -c "import json;d=json.loads(open('gpurun_out/${TAG}_${C}_bench.json').read().splitlines()[-1]);print(len(d['ms_per_layer']))" 2>/dev/null || echo 3)
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:executor -c $N \
    -o gpurun_out/${TAG}_${C}_prof -f \
    python bench.py --config $C --steps 1 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-torch-baseline --no-per-rank ${EXTRA:-} \
    > gpurun_out/${TAG}_${C}_prof.log 2>&1
  echo "$C bench+ncu rc=$?"
done
# summaries on the box (gpurun_out/ must stay < 64 MiB): raw CSV pages + markdown, then the
# reports themselves are dropped (KEEP_REP=cfg keeps one)
mkdir -p gpurun_out/${TAG}_profiles
python tools/profile_summary.py ${TAG} "${CFGS// /,}" gpurun_out/${TAG}_profiles > /dev/null
for f in gpurun_out/${TAG}_*_prof.ncu-rep; do
  case "$f" in *"_${KEEP_REP:-none}_prof.ncu-rep") ;; *) rm -f "$f" ;; esac
done
du -sh gpurun_out
