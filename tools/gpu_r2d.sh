#!/bin/bash
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
O=gpurun_out/r2d_ab.jsonl; : > $O
for C in google2 orkut google8 reddit; do
  timeout 600 python tools/ab_rt.py $C "l2_policy=0" "l2_policy=1" "l2_policy=3" "l2_policy=5" "l2_policy=9" >> $O 2>>gpurun_out/r2d_ab.err
done
for C in google8_ring google8_dgx1 reddit_dgx1; do
  timeout 600 python tools/ab_rt.py $C "sys_scope=1,l2_policy=0" "sys_scope=0,l2_policy=0" "sys_scope=0,l2_policy=1" >> $O 2>>gpurun_out/r2d_ab.err
  timeout 600 python tools/ab_rt.py $C --build pipeline_blocks=4 "sys_scope=1" "sys_scope=0" >> $O 2>>gpurun_out/r2d_ab.err
done
: > gpurun_out/r2d_tail.log
for C in google2 orkut reddit google8; do
  timeout 300 python tools/tail_trace.py $C 0 >> gpurun_out/r2d_tail.log 2>&1
done
timeout 300 python tools/tail_trace.py google8 1 >> gpurun_out/r2d_tail.log 2>&1
cat $O; cat gpurun_out/r2d_tail.log; tail -5 gpurun_out/r2d_ab.err
