#!/bin/bash
# Round-2 evidence pass on one GPU: tests + smoke, graded bench line, ncu launch list of the same
# command, every config's bench line + ncu --set full of every launch (summaries written here).
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
TAG=${TAG:-r2m}
TAG=$TAG PYT=2400 bash tools/gpu_tests.sh > gpurun_out/${TAG}_tests_summary.log 2>&1
grep -E "passed|failed" gpurun_out/${TAG}_pytest_gpu.log | tail -1
tail -1 gpurun_out/${TAG}_smoke.log
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${TAG}_launches.csv \
  python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-torch-baseline --no-per-rank > gpurun_out/${TAG}_launches_bench.json 2>&1
timeout 900 python bench.py --gpus 2 --share-gpu --config tiny --steps 3 --calls 10 > gpurun_out/${TAG}_bench_n2.json 2> gpurun_out/${TAG}_bench_n2.err
TAG=$TAG bash tools/ncu_all.sh > gpurun_out/${TAG}_ncu_all.log 2>&1
python - <<P
import json
d=json.loads(open("gpurun_out/${TAG}_bench.json").read().strip().splitlines()[-1])
print("bench", d["value"], d["ms_per_step"], d["roofline"]["frac"], d["ms_per_layer"], d["clocks"])
P
