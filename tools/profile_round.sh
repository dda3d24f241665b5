#!/bin/bash
# Round evidence for profiles/ (developer tool): GPU tests, bench lines, sweep, ncu launch list of the
# bench command, full ncu capture of the scan kernel.  Outputs land in gpurun_out/.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > gpurun_out/gpu.txt
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.txt 2>&1
timeout 600 python bench.py > gpurun_out/bench_c2.jsonl 2> gpurun_out/bench_c2.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.jsonl 2>&1
rm -f gpurun_out/bench_configs.jsonl
for c in C3k8 C3i64k8 C4s8 C5; do timeout 300 python bench.py --config $c --steps 20 --no-e2e --no-cpu >> gpurun_out/bench_configs.jsonl 2>/dev/null; done
timeout 300 python tools/sweep.py 3 > gpurun_out/sweep.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:sam_ -c 20 --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sam_scan_kernel -s 8 -c 1 -o gpurun_out/prof_c2 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu > /dev/null 2>&1
ls -la gpurun_out
