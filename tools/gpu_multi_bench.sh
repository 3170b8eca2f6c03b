#!/bin/bash
# torchrun leg of bench.py on ONE GPU (--share-gpu: all ranks on cuda:0, gloo setup) + reference arm
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || exit 1
for N in 2 4; do
  timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node $N --master-addr 127.0.0.1 \
    --master-port $((29500 + N)) bench.py --gpus $N --share-gpu --config ${CFG:-tiny} --steps 3 --warmup 3 \
    > gpurun_out/multi_$N.json 2> gpurun_out/multi_$N.err
  echo "N=$N rc=$?"; tail -c 1500 gpurun_out/multi_$N.json; tail -3 gpurun_out/multi_$N.err
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/ref.json 2> gpurun_out/ref.err
echo "ref rc=$?"; cat gpurun_out/ref.json; tail -3 gpurun_out/ref.err
