#!/bin/bash
# Round evidence for profiles/ (one GPU):
#  (1) launch list of a 1-step bench (every kernel's device time; cold-cache, serialised under ncu);
#  (2) ncu --set full of each query's timed matching launch (one ncu process per query, kernel replay,
#      -s 1 skips the STATS launch), with source;
#  (3) the L2 read-peak microbenchmark;  (4) scripts/ncu_summary.py -> gpurun_out/ncu_full_summary.json
#   profile_round.sh TAG [CONFIG] [QUERIES]
set -u
export PYTHONPATH=$PWD
TAG=${1:-r02}
CFG=${2:-2}
QS=${3:-triangle,c4,diamond,tailed_triangle,k4}
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${TAG}.csv python bench.py --config $CFG --steps 1 --warmup 0 --no-cpu-baseline --no-e2e \
  --queries $QS > gpurun_out/launches_${TAG}.out 2>&1
echo "launch list rc=$?"
for q in ${QS//,/ }; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:tdfs_kernel -s 1 -c 1 \
    -o gpurun_out/full_${TAG}_${q} -f python bench.py --config $CFG --steps 1 --warmup 0 --no-cpu-baseline --no-e2e \
    --queries $q > gpurun_out/full_${TAG}_${q}.out 2>&1
  echo "full capture $q rc=$?"
done
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/l2_peak scripts/l2_peak.cu && /tmp/l2_peak > gpurun_out/l2_peak_${TAG}.json
cat gpurun_out/l2_peak_${TAG}.json
python scripts/ncu_summary.py $TAG $CFG $QS
