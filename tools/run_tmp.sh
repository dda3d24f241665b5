mkdir -p gpurun_out
timeout 60 python tools/quick_check.py > gpurun_out/qc.txt 2>&1 || exit 1
SAM_COOP=1 timeout 60 python tools/quick_check.py >> gpurun_out/qc.txt 2>&1 || exit 1
timeout 200 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/pt.txt 2>&1
F="i32:30:1:1,i64:28:1:1,i32:28:2:1,i64:28:2:1,i32:28:4:1,i64:28:4:1,i32:28:8:1,i64:28:8:1,i64:28:4:4,i64:28:2:8,i64:28:1:8,i64:28:1:5"
for c in auto 1 0; do echo "== COOP=$c"; if [ $c = auto ]; then timeout 100 python tools/sweep.py 2 $F; else SAM_COOP=$c timeout 100 python tools/sweep.py 2 $F; fi; done > gpurun_out/sweepC.txt 2>&1
