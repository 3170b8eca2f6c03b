#!/bin/bash
# tests + smoke + N=1 bench + spawned N=2 shared-GPU bench line
cd "$(dirname "$0")/.."
TAG=${TAG:-r2b} bash tools/gpu_tests.sh
timeout 900 python bench.py > gpurun_out/${TAG:-r2b}_bench.json 2> gpurun_out/${TAG:-r2b}_bench.err
timeout 900 python bench.py --gpus 2 --share-gpu --config google2 --steps 5 --calls 20 > gpurun_out/${TAG:-r2b}_bench2.json 2> gpurun_out/${TAG:-r2b}_bench2.err
python - <<'P'
import json,os
t=os.environ.get("TAG","r2b")
for f in ("bench","bench2"):
    try:
        d=json.loads(open("gpurun_out/%s_%s.json"%(t,f)).read().strip().splitlines()[-1])
        print(f, d["value"], d["ms_per_step"], d["roofline"]["frac"], d.get("cpu_baseline"))
    except Exception as e:
        print(f, "ERR", e)
P
tail -5 gpurun_out/${TAG:-r2b}_bench2.err
