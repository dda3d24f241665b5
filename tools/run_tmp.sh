mkdir -p gpurun_out
SAM_LIB_PATH=paper_conf_pldi_malekiyb16_b200/lib/var/libsam_noks.so timeout 60 python tools/quick_check.py > gpurun_out/qc.txt 2>&1 || exit 1
F="i32:28:3:1,i32:28:4:1,i64:28:4:1,i32:28:8:1,i64:28:8:1,i64:28:4:4,i64:28:3:1"
(echo "== ks"; timeout 100 python tools/sweep.py 2 $F; echo "== noks"; SAM_LIB_PATH=paper_conf_pldi_malekiyb16_b200/lib/var/libsam_noks.so timeout 100 python tools/sweep.py 2 $F) > gpurun_out/sweep_ks.txt 2>&1
