#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
TAG=r2o PYT=2400 bash tools/gpu_tests.sh > /dev/null 2>&1
grep -E "passed|failed" gpurun_out/r2o_pytest_gpu.log | tail -1; tail -1 gpurun_out/r2o_smoke.log
timeout 900 python bench.py > gpurun_out/r2o_bench.json 2> gpurun_out/r2o_bench.err
STEPS=20 bash tools/bench_all.sh > gpurun_out/r2o_bench_all.log 2>&1; cp gpurun_out/bench_all.jsonl gpurun_out/r2o_bench_all.jsonl
tail -10 gpurun_out/r2o_bench_all.log
python - <<P
import json
d=json.loads(open("gpurun_out/r2o_bench.json").read().strip().splitlines()[-1])
print("bench", d["value"], d["ms_per_step"], d["roofline"]["frac"], d["ms_per_layer"], d["clocks"])
P
