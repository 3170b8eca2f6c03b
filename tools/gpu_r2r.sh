#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
compute-sanitizer --tool memcheck python tools/sanitize_cases.py > gpurun_out/r2r_memcheck.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/r2r_memcheck.log
compute-sanitizer --tool synccheck python tools/sanitize_cases.py > gpurun_out/r2r_synccheck.log 2>&1; echo "synccheck rc=$?" >> gpurun_out/r2r_synccheck.log
tail -12 gpurun_out/r2r_memcheck.log; tail -4 gpurun_out/r2r_synccheck.log
ncu --query-metrics 2>/dev/null | grep -i -E "nvl|nvlrx|nvltx" > gpurun_out/r2r_ncu_nvl_metrics.txt; wc -l gpurun_out/r2r_ncu_nvl_metrics.txt
O=gpurun_out/r2r_ab.jsonl; : > $O
for C in orkut google8 google8_ring reddit; do
  for rep in 1 2; do
    for L in paper_conf_eurosys_cai0wmcy21_b200/libdgcl.so build/ab/r2o.so build/ab/l0u2.so build/ab/l0u4.so; do
      DGCL_LIBRARY=$PWD/$L timeout 600 python tools/ab_rt.py $C "" | sed "s#^{#{\"lib\": \"$L\", #" >> $O 2>>gpurun_out/r2r_ab.err
    done
  done
done
python - <<'P'
import json
for l in open("gpurun_out/r2r_ab.jsonl"):
    d=json.loads(l); print(d["lib"].split("/")[-1].ljust(10), d["config"].ljust(14), d["sets"][0]["ms"])
P
