mkdir -p gpurun_out
timeout 60 python tools/quick_check.py > gpurun_out/qc.txt 2>&1 || exit 1
timeout 300 python -m pytest tests/test_parity_gpu.py tests/test_shard_gpu.py -x -q > gpurun_out/pt.txt 2>&1
F="i32:30:1:1,i64:28:1:1,i32:28:2:1,i64:28:4:1,i32:28:8:1,i64:28:1:8,i64:28:1:3,i64:28:4:4"
(echo "== coop"; timeout 100 python tools/sweep.py 3 $F; echo "== noncoop"; SAM_COOP=0 timeout 100 python tools/sweep.py 3 $F) > gpurun_out/sweep_chain.txt 2>&1
timeout 200 python bench.py --no-e2e --no-cpu > gpurun_out/bench_chain.txt 2>&1
SAM_COOP=0 timeout 200 python bench.py --no-e2e --no-cpu >> gpurun_out/bench_chain.txt 2>&1
timeout 60 python tools/trace_tiles.py i32 30 1 1 > gpurun_out/trace10.txt 2>&1
