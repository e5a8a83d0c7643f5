#!/bin/bash
# Stream C (hub x hub leaves: popcount of the AND of both bitmap rows over F's id range) at per-word cost 1/2/4
# vs off (pad = the same tree with stream C compiled out) on C2, C4 (1/64 shard), C5 (1/16 shard, tau 100 ms).
export PYTHONPATH=$PWD
mkdir -p gpurun_out
REPS=5 bash scripts/variants.sh 2 c4,diamond,tailed_triangle,k4 pad and1 and2 and4 > gpurun_out/var_c2_r02q.log 2>&1
grep -v "^lib" gpurun_out/var_c2_r02q.log
{
for v in pad and1 and2 and4; do
  echo "== $v"
  TAU=100 PYTHONPATH=/tmp/var_$v:$PWD timeout 900 python scripts/variant_time.py 5 k4 1 16
  TAU=1 PYTHONPATH=/tmp/var_$v:$PWD timeout 900 python scripts/variant_time.py 4 prism,w5 1 64
  PYTHONPATH=/tmp/var_$v:$PWD timeout 900 python scripts/variant_time.py 3 k5,house 1 64
done
} > gpurun_out/c345_r02q.log 2>&1
grep -v "^lib" gpurun_out/c345_r02q.log
# C5 k4 --set full capture (1/16 shard, tau 100 ms) of the committed kernel (in-tree libtdfs.so)
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:tdfs_kernel -s 1 -c 1 \
  -o gpurun_out/full_r02q_c5_k4 -f python bench.py --config 5 --profile-shard-world 16 --steps 1 --warmup 0 \
  --no-cpu-baseline --no-e2e --queries k4 > gpurun_out/full_r02q_c5_k4.out 2>&1; echo "c5 capture rc=$?"
