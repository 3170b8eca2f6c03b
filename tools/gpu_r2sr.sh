#!/bin/bash
# why is one-group-at-a-time slow?  DRAM bytes / L2 hit rate of the Reddit fwd602 launch per order
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
make -s all > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
for om in 0 1 2; do
  timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,lts__t_sectors_srcunit_tex_op_read.sum,gpu__time_duration.sum,lts__t_sectors_op_write.sum \
    --clock-control none -k regex:executor --launch-skip 2 -c 1 --csv python tools/one_launch.py reddit 0 0 3 owner_major=$om 2>&1 | grep -E '"(dram|lts|gpu)__' | awk -F'","' -v om=$om '{print "owner_major=" om, $(NF-2), $NF}'
done > gpurun_out/r2sr_ncu.txt
cat gpurun_out/r2sr_ncu.txt
