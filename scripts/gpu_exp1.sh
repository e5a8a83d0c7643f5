#!/bin/bash
export PYTHONPATH=$PWD
mkdir -p gpurun_out
timeout 900 python scripts/exp_time.py 2 c4,k4,diamond,tailed_triangle,triangle "TDFS_COOP=0|32;-|32;-;TDFS_FCAP=512;TDFS_FCAP=128;TDFS_LF_COST=3;TDFS_LF_COST=12" > gpurun_out/exp1.log 2>&1
cat gpurun_out/exp1.log | tail -40
timeout 1500 python -m pytest tests -m gpu -q -rfE --timeout 300 --timeout-method=signal -p no:cacheprovider \
  --deselect tests/test_gpu_configs.py > gpurun_out/gputests_exp1.log 2>&1
tail -30 gpurun_out/gputests_exp1.log
