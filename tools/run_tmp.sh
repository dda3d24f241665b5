mkdir -p gpurun_out
F="i32:28:4:1,i64:28:4:1,i32:28:8:1,i64:28:8:1,i64:28:4:4,i64:28:2:8,i64:28:1:5"
for m in 6 2 1; do echo "== M=$m"; SAM_SUPER_TILE=$m timeout 100 python tools/sweep.py 2 $F; done > gpurun_out/sweepM2.txt 2>&1
for c in "i32 28 8 1" "i64 28 4 4"; do timeout 60 python tools/trace_tiles.py $c; done > gpurun_out/trace4.txt 2>&1
