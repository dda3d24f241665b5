#!/bin/bash
# quick experiment: super-tile size vs throughput and DRAM read bytes (i32 k1 2^28)
for m in 1 2 4; do
  echo "== SAM_SUPER_TILE=$m"
  SAM_SUPER_TILE=$m timeout 120 python tools/trace_tiles.py i32 30 1 1 2>&1 | head -1
  SAM_SUPER_TILE=$m timeout 200 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum --clock-control none -k regex:sam_scan_kernel -s 2 -c 1 python tools/prof_one.py i32 28 1 1 3 2>&1 | grep -E "bytes|duration"
done
