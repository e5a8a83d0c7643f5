#!/bin/bash
# tau sweep (Tables II/III, :510-518) on config 2: 1 ms, 10 ms (default), 100 ms, no splitting
export PYTHONPATH=$PWD
for t in 1.0 10.0 100.0 -1.0; do
  echo "tau_ms $t"
  EXP_OPTS=tau_ms=$t REPS=1 timeout 300 python scripts/exp_time.py 2 ${Q:-c4,diamond,k4,tailed_triangle} "-" 2>&1 | grep -v "^$"
done
