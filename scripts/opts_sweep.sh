#!/bin/bash
# run-option sweep on config 2 (exploration): EXP_OPTS per line
export PYTHONPATH=$PWD
while read -r o; do
  echo "opts $o"
  EXP_OPTS=$o REPS=1 timeout 300 python scripts/exp_time.py 2 ${Q:-c4,diamond,k4,tailed_triangle} "-" 2>&1 | grep -v "^$"
done <<< "${SWEEP:-chunk=8
chunk=2
chunk=32
chunk=128}"
