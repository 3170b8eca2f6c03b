mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_exec.py -x -q -k "trace or relay or tiny or host" > gpurun_out/pytest_exec.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_exec.log
tail -25 gpurun_out/pytest_exec.log
