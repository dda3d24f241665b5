mkdir -p gpurun_out
timeout 60 python tools/quick_check.py > gpurun_out/qc.txt 2>&1 || exit 1
timeout 300 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/pt.txt 2>&1
timeout 200 python tools/sweep.py 2 > gpurun_out/sweep_ch.txt 2>&1
timeout 200 python bench.py --no-e2e --no-cpu > gpurun_out/bench_ch.txt 2>&1
