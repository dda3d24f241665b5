mkdir -p gpurun_out
F="i32:28:1:2,i32:28:1:3,i32:28:1:4,i32:28:1:5,i32:28:1:8,i64:28:1:2,i64:28:1:3,i64:28:1:5,i64:28:1:8,i64:28:2:8,i64:28:4:4,i32:28:2:4"
for m in 3 4; do echo "== M=$m"; SAM_SUPER_TILE=$m timeout 150 python tools/sweep.py 3 $F; done > gpurun_out/sweep_tm.txt 2>&1
