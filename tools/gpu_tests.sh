#!/bin/bash
# GPU tests (full suite incl. full-size every-row parity), smoke; box facts.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
TAG=${TAG:-r2}
nproc > gpurun_out/${TAG}_box.txt; free -g >> gpurun_out/${TAG}_box.txt
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout ${PYT:-3000} python -m pytest tests -m gpu -q ${PYTEST_ARGS:-} --durations=25 > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
tail -40 gpurun_out/${TAG}_pytest_gpu.log; tail -2 gpurun_out/${TAG}_smoke.log; cat gpurun_out/${TAG}_box.txt
