mkdir -p gpurun_out
SAM_LIB_PATH=paper_conf_pldi_malekiyb16_b200/lib/var/libsam_er2.so timeout 60 python tools/quick_check.py > gpurun_out/qc.txt 2>&1 || exit 1
F="i32:30:1:1,i64:28:1:1,i32:28:2:1,i32:28:4:1,i64:28:4:1,i64:28:1:8,i32:28:1:3,i64:28:4:4,f32:28:1:4"
(echo "== base"; timeout 100 python tools/sweep.py 2 $F; echo "== er2"; SAM_LIB_PATH=paper_conf_pldi_malekiyb16_b200/lib/var/libsam_er2.so timeout 100 python tools/sweep.py 2 $F) > gpurun_out/sweep_er2.txt 2>&1
for v in base er2 base er2; do echo "== $v"; if [ $v = base ]; then timeout 200 python bench.py --no-e2e --no-cpu; else SAM_LIB_PATH=paper_conf_pldi_malekiyb16_b200/lib/var/libsam_$v.so timeout 200 python bench.py --no-e2e --no-cpu; fi; done > gpurun_out/bench_er2.txt 2>&1
