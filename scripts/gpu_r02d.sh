#!/bin/bash
export PYTHONPATH=$PWD
bash scripts/gpu_check.sh r02d
REPS=3 bash scripts/variants.sh 2 c4,diamond,tailed_triangle,k4,triangle base min8 min10 min16 > gpurun_out/variants_r02d.log 2>&1; cat gpurun_out/variants_r02d.log
