#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
python -c "
import paper_conf_eurosys_cai0wmcy21_b200._abi as A, ctypes
L=A.lib(); v=ctypes.c_int32(0); L.dgcl_multicast_supported(0, ctypes.byref(v)); print('multicast supported', v.value)
buf=ctypes.create_string_buffer(256); st=L.dgcl_debug_multicast_selftest(0, 1<<21, buf, 256); print('selftest', st, buf.value.decode())
" > gpurun_out/r2f_mc.txt 2>&1
cat gpurun_out/r2f_mc.txt
O=gpurun_out/r2f_ab.jsonl; : > $O
for C in google2 google4 orkut google8 reddit google8_ring reddit_dgx1; do
  timeout 600 python tools/ab_rt.py $C "item_order=0" "item_order=2" "item_order=1" >> $O 2>>gpurun_out/r2f_ab.err
done
cat $O | python -c "
import json,sys
for l in sys.stdin:
    d=json.loads(l)
    print(d['config'], d['build'])
    for s in d['sets']: print('   ', s['opts'], s['ms'])
"
timeout 900 python -m pytest tests/test_gpu_exec.py -q -x -k "uniform_loopback_fused or relay or sixteen or tiny" > gpurun_out/r2f_pytest.log 2>&1; tail -3 gpurun_out/r2f_pytest.log
