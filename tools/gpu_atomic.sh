#!/bin/bash
# Table 9 analogue: fixed-order (non-atomic) backward vs the atomic-add ablation, 1-GPU loopback
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
CFGS="${CFGS:-reddit google2 google8 orkut}" EXTRA="--opt atomic_backward=1 --no-torch-baseline" bash tools/bench_all.sh 2>&1 | tail -4
cp gpurun_out/bench_all.jsonl gpurun_out/atomic_bench.jsonl
