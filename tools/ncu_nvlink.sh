#!/bin/bash
# NVLink bytes of the executor launches on a multi-GPU box (not runnable on the one-GPU gpurun
# boxes): rank 0 of `bench.py --gpus N` under ncu with the Blackwell NVLink counters
# (profiles/r2_ncu_nvlink_metric_names.txt), application replay so the peers' flag waits see
# every pass.  Other ranks run unprofiled.  Usage: N=8 CFG=reddit tools/ncu_nvlink.sh
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
N=${N:-8}; CFG=${CFG:-reddit}; TAG=${TAG:-nvl}
PORT=$((29600 + RANDOM % 1000))
for r in $(seq 0 $((N - 1))); do
  if [ "$r" = 0 ]; then PRE="ncu --replay-mode application --app-replay-match grid --clock-control none \
      --metrics nvltx__bytes_data_user.sum,nvlrx__bytes_data_user.sum,gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
      -k regex:executor -c 12 --csv --log-file gpurun_out/${TAG}_rank0.csv"; else PRE=""; fi
  RANK=$r LOCAL_RANK=$r WORLD_SIZE=$N MASTER_ADDR=127.0.0.1 MASTER_PORT=$PORT \
    $PRE python bench.py --gpus $N --config $CFG --steps 2 --warmup 3 --calls 10 --e2e-steps 0 \
    --no-cpu-baseline --no-p2p-baseline > gpurun_out/${TAG}_r$r.log 2>&1 &
done
wait
grep -E "nvltx|nvlrx" gpurun_out/${TAG}_rank0.csv | head -20
