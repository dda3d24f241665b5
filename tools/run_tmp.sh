mkdir -p gpurun_out
F="i32:28:1:3,i32:28:1:5,f32:28:1:3"
(for r in 1 2; do echo "== unset"; timeout 100 python tools/sweep.py 3 $F; echo "== M4"; SAM_SUPER_TILE=4 timeout 100 python tools/sweep.py 3 $F; echo "== M3"; SAM_SUPER_TILE=3 timeout 100 python tools/sweep.py 3 $F; done) > gpurun_out/sweep_odd.txt 2>&1
