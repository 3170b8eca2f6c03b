#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
for L in build/ab/h2.so build/ab/h3.so; do
  DGCL_LIBRARY=$PWD/$L timeout 900 python -m pytest tests/test_gpu_exec.py -q -x -k "uniform_loopback_fused or relay or per_rank" > gpurun_out/r2w_pytest_$(basename $L).log 2>&1; tail -1 gpurun_out/r2w_pytest_$(basename $L).log
done
O=gpurun_out/r2w_ab.jsonl; : > $O
for C in orkut google8 reddit google8_ring google4; do
  for rep in 1 2; do
    for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/h2.so build/ab/h3.so; do
      DGCL_LIBRARY=$PWD/$L timeout 600 python tools/ab_rt.py $C "" | sed "s#^{#{\"lib\": \"$L\", #" >> $O 2>>gpurun_out/r2w_ab.err
    done
  done
done
python - <<'P'
import json
for l in open("gpurun_out/r2w_ab.jsonl"):
    d=json.loads(l); print(d["lib"].split("/")[-1].ljust(10), d["config"].ljust(14), d["sets"][0]["ms"])
P
