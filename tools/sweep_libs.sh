#!/bin/bash
# sweep.py over library variants (developer tool): tools/sweep_libs.sh "base lag16 lag20" [reps] [filter]
for v in $1; do echo "== $v"; if [ $v = base ]; then timeout 300 python tools/sweep.py ${2:-2} $3; else SAM_LIB_PATH=paper_conf_pldi_malekiyb16_b200/lib/var/libsam_$v.so timeout 300 python tools/sweep.py ${2:-2} $3; fi; done
