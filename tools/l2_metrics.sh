#!/bin/bash
# L2 hit/miss breakdown of one scan launch (developer tool): tools/l2_metrics.sh i32 30 1 1 out.csv
M=lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum,lts__t_sectors_srcunit_tex_op_write.sum,lts__t_sectors_op_read.sum,lts__t_sectors_op_read_lookup_hit.sum,lts__t_sectors_op_write.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_lookup_hit.sum,lts__t_sectors_lookup_miss.sum
ncu --metrics $M --clock-control none -k regex:sam_scan_kernel -s 2 -c 1 --csv python tools/prof_one.py $1 $2 $3 $4 3 > $5 2>&1
