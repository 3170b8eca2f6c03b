#!/bin/bash
# WIDE3 (3 x 64 KB) for single-producer WIDE launches: GPU suite, graded bench (per-rank numbers)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
TAG=r2to PYT=2400 bash tools/gpu_tests.sh > gpurun_out/r2to_tests_summary.log 2>&1
grep -E "passed|failed" gpurun_out/r2to_pytest_gpu.log | tail -1; tail -1 gpurun_out/r2to_smoke.log
timeout 900 python bench.py > gpurun_out/r2to_bench.json 2> gpurun_out/r2to_bench.err
python - <<'P'
import json
d=json.loads(open("gpurun_out/r2to_bench.json").read().strip().splitlines()[-1])
print("bench", d["value"], d["ms_per_step"], d["roofline"]["frac"], d["ms_per_layer"], d["per_rank_loopback"]["ms_per_layer"], d["clocks"])
P
