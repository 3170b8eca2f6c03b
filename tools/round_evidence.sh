#!/bin/bash
# Full evidence pass on one GPU: tests, smoke, bench (default), ncu (reddit), all configs.
cd "$(dirname "$0")/.."
TAG=${TAG:-r1f}
bash tools/gpu_check.sh > gpurun_out/${TAG}_check.log 2>&1
grep -E "passed|failed" gpurun_out/pytest_gpu.log | tail -2
tail -1 gpurun_out/smoke.log
cp gpurun_out/bench.json gpurun_out/${TAG}_bench.json
TAG=$TAG bash tools/ncu_bench.sh > /dev/null 2>&1
bash tools/bench_all.sh 2>&1 | tail -9
cp gpurun_out/bench_all.jsonl gpurun_out/${TAG}_bench_all.jsonl
