#!/bin/bash
# Diagnostics run: verbose -m gpu suite with durations, then a source-level capture of one query.
export PYTHONPATH=$PWD
TAG=${1:-x}
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -v -rA --durations=30 --timeout 900 --timeout-method=thread \
  -p no:cacheprovider > gpurun_out/gputests_${TAG}_full.log 2>&1
grep -E "PASSED|FAILED|ERROR|Timeout|passed|failed|s call" gpurun_out/gputests_${TAG}_full.log | tail -60
if [ -n "${SRCQ:-}" ]; then bash scripts/profile_src.sh ${TAG} ${SRCQ} ${SRCW:-16}; fi
