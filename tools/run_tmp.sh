mkdir -p gpurun_out
timeout 60 python tools/quick_check.py > gpurun_out/qc.txt 2>&1 || exit 1
timeout 300 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/pt.txt 2>&1
timeout 200 python tools/sweep.py 3 > gpurun_out/sweep_m.txt 2>&1
timeout 200 python bench.py --no-e2e --no-cpu > gpurun_out/bench_m.txt 2>&1
timeout 200 python bench.py --config C4s8 --steps 20 --no-e2e --no-cpu >> gpurun_out/bench_m.txt 2>&1
