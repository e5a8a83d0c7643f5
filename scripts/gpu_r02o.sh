#!/bin/bash
# (1) old (HEAD kernel) vs new (one DFS call site, warp context in shared memory) vs new at 10 blocks/SM on C2;
# (2) C5 k4 (1/16 shard): range tasks for the reused leaf-parent level (rlr) vs per-sibling tasks, tau 1/10/100 ms;
# (3) ncu DRAM bytes + L2 hit of base vs the evict_last hub-bitmap hint (h1) on C5 k4 1/16 and C4 prism 1/64.
export PYTHONPATH=$PWD
mkdir -p gpurun_out
REPS=5 bash scripts/variants.sh 2 triangle,c4,diamond,tailed_triangle,k4 old base mb10 rlr > gpurun_out/var_c2_r02o.log 2>&1
grep -v "^lib" gpurun_out/var_c2_r02o.log
for v in h1; do
  d=/tmp/var_$v; rm -rf $d && mkdir -p $d/paper_conf_icde_yuan0ha0024_b200
  cp paper_conf_icde_yuan0ha0024_b200/*.py $d/paper_conf_icde_yuan0ha0024_b200/; cp variants/$v.so $d/paper_conf_icde_yuan0ha0024_b200/libtdfs.so
done
{
for v in old base rlr; do
  for t in 1 10 100; do echo "== $v tau $t"; TAU=$t PYTHONPATH=/tmp/var_$v:$PWD timeout 900 python scripts/variant_time.py 5 k4 1 16; done
done
for v in old base; do echo "== $v C4"; PYTHONPATH=/tmp/var_$v:$PWD timeout 900 python scripts/variant_time.py 4 prism,w5 3 64; done
} > gpurun_out/c45_r02o.log 2>&1
grep -v "^lib" gpurun_out/c45_r02o.log
for v in base h1; do
  PYTHONPATH=/tmp/var_$v:$PWD timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum \
    --clock-control none -k regex:tdfs_kernel --csv --log-file gpurun_out/ncu_l2hint_${v}_c5.csv python scripts/variant_time.py 5 k4 1 16 > /dev/null 2>&1
  PYTHONPATH=/tmp/var_$v:$PWD timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum \
    --clock-control none -k regex:tdfs_kernel --csv --log-file gpurun_out/ncu_l2hint_${v}_c4.csv python scripts/variant_time.py 4 prism 1 64 > /dev/null 2>&1
  echo "ncu $v rc=$?"
done
