#!/bin/bash
python -c "
import torch; p=torch.cuda.get_device_properties(0); print('persistingL2CacheMaxSize', getattr(p,'persisting_l2_cache_max_size', None), 'L2', p.L2_cache_size)"
for mb in 0 32 64 96; do
  for m in 1 2 4; do
    echo "== persist=$mb MB M=$m"
    SAM_L2_PERSIST_MB=$mb SAM_SUPER_TILE=$m timeout 200 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum --clock-control none -k regex:sam_scan_kernel -s 2 -c 1 python tools/prof_one.py i32 28 1 1 3 2>&1 | grep -E "bytes|duration"
  done
done
