#!/bin/bash
# A/B matrix of runtime knobs and library variants on the heavy configs (developer tool)
H="i32:28:2:1,i32:28:4:1,i64:28:2:1,i64:28:4:1,i64:28:8:1,i64:28:4:4,i64:28:2:8,i32:28:8:1,i32:28:3:1,i64:28:3:1"
V=paper_conf_pldi_malekiyb16_b200/lib/var
run() { echo "== $1"; shift; env "$@" timeout 150 python tools/sweep.py 2 $H; }
run "base land1 vfold1" X=1
run "base land1 vfold0" SAM_VFOLD=0
run "base land0" SAM_LAND=0
run "tr5" SAM_LIB_PATH=$V/libsam_tr5.so
run "lag12m3" SAM_LIB_PATH=$V/libsam_lag12m3.so
run "lag12m3 M=2" SAM_LIB_PATH=$V/libsam_lag12m3.so SAM_SUPER_TILE=2
run "m4" SAM_LIB_PATH=$V/libsam_m4.so
run "base land1 vfold1 (repeat)" X=1
