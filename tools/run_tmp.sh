mkdir -p gpurun_out
timeout 60 python tools/quick_check.py > gpurun_out/qc.txt 2>&1 || exit 1
timeout 300 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/pt.txt 2>&1
timeout 200 python tools/sweep.py 2 > gpurun_out/sweep_ld.txt 2>&1
(echo "== M4"; SAM_SUPER_TILE=4 timeout 100 python tools/sweep.py 2 f32:28:1:4,i32:28:1:3,i32:28:1:2,i64:28:1:3,i64:28:1:8) >> gpurun_out/sweep_ld.txt 2>&1
timeout 200 python bench.py --no-e2e --no-cpu > gpurun_out/bench_ld.txt 2>&1
timeout 60 python tools/trace_tiles.py i32 30 1 1 > gpurun_out/trace12.txt 2>&1
