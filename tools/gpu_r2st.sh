#!/bin/bash
# compute-sanitizer memcheck + synccheck of the executor cases (incl. 1-KB rows: per-row relay
# stores, fan-out bulk stores, item orders)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1500 compute-sanitizer --tool memcheck python tools/sanitize_cases.py > gpurun_out/r2st_memcheck.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/r2st_memcheck.log
timeout 1500 compute-sanitizer --tool synccheck python tools/sanitize_cases.py > gpurun_out/r2st_synccheck.log 2>&1; echo "synccheck rc=$?" >> gpurun_out/r2st_synccheck.log
tail -16 gpurun_out/r2st_memcheck.log; tail -4 gpurun_out/r2st_synccheck.log
