#!/bin/bash
# hash index / occupancy experiments on config 2, then the full -m gpu suite and a bench line
export PYTHONPATH=$PWD
Q=${Q:-triangle,c4,diamond,tailed_triangle,k4}
timeout 300 python scripts/exp_time.py 2 $Q "-;-|64;-|16" > gpurun_out/exp2_default.log 2>&1
for v in min8 min12; do
  TDFS_LIB=$PWD/variants/$v.so timeout 200 python scripts/exp_time.py 2 $Q "-" > gpurun_out/exp2_$v.log 2>&1
done
cat gpurun_out/exp2_*.log
bash scripts/gpu_check.sh ${1:-s3b}
