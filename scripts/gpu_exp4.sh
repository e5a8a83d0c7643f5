#!/bin/bash
# default build vs occupancy variants (variants/minN.so = __launch_bounds__(128, N)) on config 2
export PYTHONPATH=$PWD
Q=${Q:-triangle,c4,diamond,tailed_triangle,k4}
timeout 300 python scripts/exp_time.py 2 $Q "-" > gpurun_out/exp4_default.log 2>&1
for v in ${VARIANTS:-min8 min12}; do
  TDFS_LIB=$PWD/variants/$v.so timeout 300 python scripts/exp_time.py 2 $Q "-" > gpurun_out/exp4_$v.log 2>&1
done
tail -n 6 gpurun_out/exp4_*.log
