#!/bin/bash
# variant timing on config 2 (EXP_VARIANTS), then the -m gpu suite + bench (gpu_check.sh)
export PYTHONPATH=$PWD
Q=${Q:-triangle,c4,diamond,tailed_triangle,k4}
timeout 400 python scripts/exp_time.py 2 $Q "${EXP_VARIANTS:--}" > gpurun_out/exp_${1:-x}.log 2>&1
cat gpurun_out/exp_${1:-x}.log
[ -n "${SKIP_CHECK:-}" ] || bash scripts/gpu_check.sh ${1:-x}
