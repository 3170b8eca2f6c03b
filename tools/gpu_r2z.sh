#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
DGCL_RANDOM_CASES=300 timeout 2400 python -m pytest tests/test_gpu_exec.py -q -k "random_option" > gpurun_out/r2z_pytest.log 2>&1; tail -15 gpurun_out/r2z_pytest.log
