#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2i_ab.jsonl; : > $O
for C in reddit google2 orkut google8_ring reddit_dgx1 google8; do
  for rep in 1 2; do
    for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/prev.so; do
      DGCL_LIBRARY=$PWD/$L timeout 600 python tools/ab_rt.py $C "" | sed "s#^{#{\"lib\": \"$L\", #" >> $O 2>>gpurun_out/r2i_ab.err
    done
  done
done
python - <<'P'
import json
for l in open("gpurun_out/r2i_ab.jsonl"):
    d=json.loads(l); print(d["lib"].split("/")[-1], d["config"], d["sets"][0]["ms"])
P
timeout 600 python examples/gcn_overlap.py > gpurun_out/r2i_overlap.json 2> gpurun_out/r2i_overlap.err; cat gpurun_out/r2i_overlap.json
timeout 900 python -m pytest tests/test_gpu_exec.py tests/test_gpu_multicast.py tests/test_gpu_gcn.py -q -x -k "uniform_loopback_fused or relay or per_rank or multicast or gcn or sixteen" > gpurun_out/r2i_pytest.log 2>&1; tail -3 gpurun_out/r2i_pytest.log
