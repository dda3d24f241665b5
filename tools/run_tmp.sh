mkdir -p gpurun_out
timeout 60 python tools/quick_check.py > gpurun_out/qc.txt 2>&1 || exit 1
timeout 300 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/pt.txt 2>&1
F="i32:28:4:1,i32:28:5:1,i32:28:8:1,i64:28:3:1,i64:28:4:1,i64:28:4:4,i64:28:8:1"
echo "== base" > gpurun_out/sweep32.txt; timeout 100 python tools/sweep.py 2 $F >> gpurun_out/sweep32.txt 2>&1
echo "== old32" >> gpurun_out/sweep32.txt; SAM_LIB_PATH=paper_conf_pldi_malekiyb16_b200/lib/var/libsam_old32.so timeout 100 python tools/sweep.py 2 $F >> gpurun_out/sweep32.txt 2>&1
