mkdir -p gpurun_out
timeout 60 python tools/quick_check.py > gpurun_out/qc.txt 2>&1 || exit 1
timeout 300 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/pt.txt 2>&1
for i in 1 2; do timeout 200 python bench.py --no-e2e --no-cpu; done > gpurun_out/bench_ilp.txt 2>&1
timeout 100 python tools/sweep.py 2 i32:30:1:1,i64:28:1:1,f64:28:1:1 > gpurun_out/sweep_ilp.txt 2>&1
