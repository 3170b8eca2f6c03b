#!/bin/bash
# One-off probe of the GPU box (hardware facts for DESIGN.md).
set -x
nproc; free -g | head -2; nvidia-smi; nvidia-smi topo -m
python -c "import torch,os; print('devs', torch.cuda.device_count(), torch.cuda.get_device_name(0), 'affinity', len(os.sched_getaffinity(0)))"
ncu --query-metrics 2>/dev/null | grep -i -E "nvl|dram__bytes" | head -40
