#!/bin/bash
# relay-plan work: GPU tests, stage timelines, relay-config bench lines
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
: > gpurun_out/relay_trace.log
for C in ${TRACE_CFGS:-google8_ring google8_dgx1 reddit_dgx1}; do
  timeout 300 python tools/relay_trace.py $C >> gpurun_out/relay_trace.log 2>&1
done
grep -E "launch|stage" gpurun_out/relay_trace.log | head -80
CFGS="${BENCH_CFGS:-google8_dgx1 google8_ring reddit_dgx1 google8 orkut}" bash tools/bench_all.sh 2>&1 | tail -6
