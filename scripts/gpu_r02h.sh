#!/bin/bash
export PYTHONPATH=$PWD
bash scripts/gpu_check.sh r02h
for q in c4 diamond tailed_triangle k4 triangle; do :; done
PYTHONPATH=$PWD timeout 600 python scripts/variant_time.py 2 c4,diamond,tailed_triangle,k4,triangle 3 1 0 deg > gpurun_out/degorder_c2.log 2>&1; cat gpurun_out/degorder_c2.log
PYTHONPATH=$PWD timeout 600 python scripts/variant_time.py 3 k5,house 1 1 0 deg > gpurun_out/degorder_c3.log 2>&1; cat gpurun_out/degorder_c3.log
bash scripts/gpu_r02g.sh
