#!/bin/bash
# relay-plan stage timelines + multi-process bench on one shared GPU (torchrun, 2 ranks)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
for C in google8_ring google8_dgx1 reddit_dgx1; do
  timeout 300 python tools/relay_trace.py $C >> gpurun_out/relay_trace.log 2>&1
done
for C in tiny google2; do
  timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29511 bench.py --gpus 2 --share-gpu --config $C --steps 5 --warmup 3 \
    >> gpurun_out/multi_share.jsonl 2>> gpurun_out/multi_share.err
  echo "$C rc=$?" >> gpurun_out/multi_share.err
done
cat gpurun_out/relay_trace.log; tail -3 gpurun_out/multi_share.err; head -c 1500 gpurun_out/multi_share.jsonl
