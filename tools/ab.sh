#!/bin/bash
# A/B of library variants on the heavy configs (developer tool): tools/ab.sh "name:ENV=.. ENV=.." ...
H=${H:-"i32:28:1:1,i32:28:2:1,i32:28:4:1,i32:28:8:1,i64:28:1:1,i64:28:2:1,i64:28:4:1,i64:28:8:1,i64:28:4:4,i64:28:1:5,i64:28:2:8"}
for spec in "$@"; do
  name=${spec%%:*}; envs=${spec#*:}
  echo "== $name ($envs)"; env $envs timeout 300 python tools/sweep.py 2 $H
done
