#!/bin/bash
# carry-team count A/B on the sweep configs (developer tool)
H=${H:-"i32:30:1:1,i32:28:2:1,i32:28:4:1,i32:28:8:1,i64:28:1:1,i64:28:2:1,i64:28:4:1,i64:28:8:1,i64:28:4:4,i64:28:2:8,i64:28:1:5,i64:28:1:3,f32:28:1:4"}
for T in ${TEAMS:-1 2 4}; do echo "== SAM_TEAMS=$T"; SAM_TEAMS=$T timeout 200 python tools/sweep.py 2 $H; done
