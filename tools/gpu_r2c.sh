#!/bin/bash
# new GPU tests (overlap), relay stage traces, overlap timing, ncu of every config
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_gcn.py tests/test_gpu_exec.py -q -x -k "gcn or argument or wait" > gpurun_out/r2c_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r2c_pytest.log
tail -3 gpurun_out/r2c_pytest.log
for C in google8_ring google8_dgx1 reddit_dgx1; do
  timeout 300 python tools/relay_trace.py $C >> gpurun_out/r2c_relay_trace.log 2>&1
done
timeout 600 python examples/gcn_overlap.py > gpurun_out/r2c_overlap.json 2> gpurun_out/r2c_overlap.err
cat gpurun_out/r2c_overlap.json
TAG=r2c bash tools/ncu_all.sh
cat gpurun_out/r2c_relay_trace.log
