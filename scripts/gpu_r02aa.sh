#!/bin/bash
# tau sweep on C2 (five queries) and C3 k5 with this round's kernel.
export PYTHONPATH=$PWD
mkdir -p gpurun_out
{
for t in 3 10 30 100; do
  echo "== tau $t"
  TAU=$t timeout 900 python scripts/variant_time.py 2 c4,diamond,tailed_triangle,k4,triangle 5 1
  TAU=$t timeout 900 python scripts/variant_time.py 3 k5 3 1
done
} > gpurun_out/tau_r02aa.log 2>&1
grep -v "^lib" gpurun_out/tau_r02aa.log
