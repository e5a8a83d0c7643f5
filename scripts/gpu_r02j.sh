#!/bin/bash
export PYTHONPATH=$PWD
timeout 900 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider -k "shard or partitioned or degree_order or two_ranks" > gpurun_out/gputests_r02j.log 2>&1
grep -E "^(FAILED|ERROR)|passed|failed|Timeout" gpurun_out/gputests_r02j.log | tail -10
P=scripts/configs_probe.py
timeout 1200 python $P 4 prism,w5 8 0,1,2,3,4,5,6,7 2 > gpurun_out/imb_c4_blk.log 2>&1; cat gpurun_out/imb_c4_blk.log
timeout 900 python $P 5 k4 8 0,1,2,3,4,5,6,7 2 > gpurun_out/imb_c5_blk.log 2>&1; cat gpurun_out/imb_c5_blk.log
timeout 600 python $P 2 c4,diamond,k4 8 0,1,2,3,4,5,6,7 2 > gpurun_out/imb_c2_blk.log 2>&1; cat gpurun_out/imb_c2_blk.log
timeout 600 python $P 2 c4,diamond,k4 8 0,1,2,3,4,5,6,7 0 > gpurun_out/imb_c2_rr.log 2>&1; cat gpurun_out/imb_c2_rr.log
