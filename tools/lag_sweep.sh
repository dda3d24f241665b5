#!/bin/bash
# pipeline-depth sweep (developer tool): SAM_LAG values for the heavy configs; outputs in gpurun_out/
F=${F:-"i64:28:4:4,i64:28:8:1,i32:28:8:1,i64:28:4:1,i64:28:3:1,i32:28:6:1"}
for L in ${LAGS:-12 10 8 6 4}; do echo "== SAM_LAG=$L"; SAM_LAG=$L timeout 200 python tools/sweep.py 2 $F; done
