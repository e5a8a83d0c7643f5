#!/bin/bash
export PYTHONPATH=$PWD
timeout 900 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider -k "enumerate_to_rank or deep_range or trace or stream" > gpurun_out/gputests_r02f.log 2>&1
grep -E "^(FAILED|ERROR)|passed|failed|Timeout" gpurun_out/gputests_r02f.log | tail -10
REPS=3 bash scripts/variants.sh 2 c4,diamond,tailed_triangle,k4,triangle base f512t0 f256t1 f256t0 f128t0 f256t0m10 > gpurun_out/variants_r02f.log 2>&1; cat gpurun_out/variants_r02f.log
bash scripts/sanitize.sh r02
