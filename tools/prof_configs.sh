#!/bin/bash
# ncu --set full of the scan kernel for a list of configs "dt:logn:k:s" (developer tool; outputs in gpurun_out/)
# usage: tools/prof_configs.sh TAG cfg1 cfg2 ...   (KEEP=1 keeps the .ncu-rep files; default: text summaries only)
tag=$1; shift
mkdir -p gpurun_out
for c in "$@"; do
  IFS=: read dt logn k s <<< "$c"
  out=gpurun_out/${tag}_${dt}_k${k}_s${s}
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:sam_scan_kernel -s 2 -c 1 \
     -o $out python tools/prof_one.py $dt $logn $k $s 3 > $out.log 2>&1
  python tools/ncu_summary.py $out.ncu-rep --src > $out.txt 2>&1
  python -c "import sys; sys.path.insert(0,'tools'); import ncu_summary as n; n.stall_table('$out.ncu-rep', 30)" >> $out.txt 2>&1
  ncu -i $out.ncu-rep --page raw --csv > $out.raw.csv 2>/dev/null
  [ "$KEEP" = "1" ] || rm -f $out.ncu-rep
done
