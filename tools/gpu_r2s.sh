#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }


O=gpurun_out/r2t_ab.jsonl; : > $O
for C in reddit google2; do
  for rep in 1 2 3; do
    for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/r2o.so; do
      DGCL_LIBRARY=$PWD/$L timeout 600 python tools/ab_rt.py $C "" | sed "s#^{#{\"lib\": \"$L\", #" >> $O 2>>gpurun_out/r2t_ab.err
    done
  done
done
python - <<'P'
import json
for l in open("gpurun_out/r2t_ab.jsonl"):
    d=json.loads(l); print(d["lib"].split("/")[-1].ljust(10), d["config"].ljust(14), d["sets"][0]["ms"])
P
