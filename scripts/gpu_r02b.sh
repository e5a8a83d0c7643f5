#!/bin/bash
export PYTHONPATH=$PWD
bash scripts/gpu_check.sh r02b
timeout 900 python scripts/configs_probe.py 3 house,c5 64 0 0 10 > gpurun_out/probe3_range.log 2>&1; cat gpurun_out/probe3_range.log
timeout 900 python scripts/configs_probe.py 3 house,c5 64 0 0 10 256 > gpurun_out/probe3_norange.log 2>&1; cat gpurun_out/probe3_norange.log
bash scripts/profile_src.sh r02b c4 16; python scripts/src_regions.py gpurun_out/src_r02b_c4.ncu-rep 40 > gpurun_out/src_r02b_c4.txt 2>&1
