#!/bin/bash
# ncu evidence for the matching kernel (run under gpurun, 1 GPU).
#   launches.csv : every kernel launch of a 1-step bench with its device time
#   prof_<q>.ncu-rep : --set full capture of the matching kernel for query <q>
set -u
export PYTHONPATH=$PWD
TAG=${1:-r01}
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e \
  > gpurun_out/launches_${TAG}.out 2>&1
echo "launch list rc=$?"
for q in ${QUERIES:-k4 diamond}; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:tdfs_kernel -s 1 -c 1 \
    -o gpurun_out/prof_${TAG}_${q} -f python bench.py --steps 1 --warmup 0 --queries $q --no-cpu-baseline --no-e2e \
    > gpurun_out/prof_${TAG}_${q}.out 2>&1
  echo "full capture $q rc=$?"
done
