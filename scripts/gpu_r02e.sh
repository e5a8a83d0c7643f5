#!/bin/bash
export PYTHONPATH=$PWD
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > gpurun_out/gputests_r02e.log 2>&1
grep -E "^(FAILED|ERROR)|passed|failed|Timeout" gpurun_out/gputests_r02e.log | tail -30
for mb in 32 64 96 256 1024; do PYTHONPATH=$PWD timeout 300 python scripts/variant_time.py 2 c4,diamond,tailed_triangle,k4 2 1 $mb; done > gpurun_out/hubmb_r02e.log 2>&1; cat gpurun_out/hubmb_r02e.log
timeout 900 python scripts/configs_probe.py 3 house,c5,k5 64 0 0 10 0 stats > gpurun_out/probe3_stats.log 2>&1; cat gpurun_out/probe3_stats.log
