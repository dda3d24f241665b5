#!/bin/bash
# Round evidence for profiles/ (developer tool): GPU tests, bench lines, ncu launch list of the bench
# command, full ncu captures of the scan kernel on the key configs, DRAM traffic of every sweep config,
# carry-scheme ablation.  Outputs land in gpurun_out/ (text only: .ncu-rep files are summarised and removed).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.limit --format=csv > gpurun_out/gpu.txt
lscpu | grep -E "Model name|^CPU\(s\)" >> gpurun_out/gpu.txt
if [ "$TESTS" != "0" ]; then
  timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.txt 2>&1; tail -3 gpurun_out/pytest_gpu.txt
fi
timeout 900 python bench.py > gpurun_out/bench.jsonl 2> gpurun_out/bench.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.jsonl 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:sam_ -c 20 --csv \
    --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu --no-sweep > /dev/null 2>&1
tools/prof_configs.sh full i32:30:1:1 i64:28:8:1 i64:28:4:4 i64:28:1:5 i32:28:4:1 i64:28:2:1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:sam_scan_kernel \
    --clock-control none --csv --log-file gpurun_out/ncu_sweep.csv python tools/ncu_sweep.py > gpurun_out/ncu_sweep.log 2>&1
timeout 600 python tools/ablation.py gpurun_out/ablation.json > gpurun_out/ablation.txt 2>&1
ls -la gpurun_out
# the dedicated state-pass kernel on north_star's multi-GPU config (C5 shard, 2^30 int64 k=4 s=4)
timeout 300 ncu --set full --clock-control none --import-source on -k regex:sam_state_kernel -s 2 -c 1 \
   -o gpurun_out/full_state_i64_k4_s4 python tools/prof_state.py i64 30 4 4 > gpurun_out/full_state.log 2>&1
python tools/ncu_summary.py gpurun_out/full_state_i64_k4_s4.ncu-rep > gpurun_out/full_state_i64_k4_s4.txt 2>&1
rm -f gpurun_out/full_state_i64_k4_s4.ncu-rep
timeout 600 python tools/state_bench.py > gpurun_out/state_bench.txt 2>&1
ls -la gpurun_out
