#!/bin/bash
# sweep.py under several values of one env var (developer tool): tools/sweep_env.sh VAR "v1 v2 ..." [reps]
for v in $2; do echo "== $1=$v"; env $1=$v timeout 300 python tools/sweep.py ${3:-2} $4; done
