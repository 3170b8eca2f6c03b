mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_exec.py -x -q > gpurun_out/pytest_exec.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_exec.log
tail -3 gpurun_out/pytest_exec.log
run() { # cfg opts...
  C=$1; shift
  timeout 600 python bench.py --config $C --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline --no-torch-baseline "$@" 2>/dev/null | python3 -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$C $*', round(d['ms_per_step'],3), {k: (round(v['ms'],3), round(v['frac'],3)) for k,v in d['roofline']['per_kernel'].items()})"
}
for C in google8_dgx1 reddit_dgx1 google8_ring; do
  for G in 0 1 2; do run $C --opt geometry=$G; done
  run $C --opt stage_fold=0
done
run reddit
run tiny
