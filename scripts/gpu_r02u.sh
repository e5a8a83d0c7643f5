#!/bin/bash
# Hub minimum degree 256 (base) vs 128 / 64 (variants md128 / md64) on C2 at 256 / 512 MB budgets, and C5 k4 1/16 at 1 GB.
export PYTHONPATH=$PWD
mkdir -p gpurun_out
for v in base md128 md64; do
  d=/tmp/var_$v; rm -rf $d && mkdir -p $d/paper_conf_icde_yuan0ha0024_b200
  cp paper_conf_icde_yuan0ha0024_b200/*.py $d/paper_conf_icde_yuan0ha0024_b200/
  if [ "$v" = base ]; then cp paper_conf_icde_yuan0ha0024_b200/libtdfs.so $d/paper_conf_icde_yuan0ha0024_b200/;
  else cp variants/$v.so $d/paper_conf_icde_yuan0ha0024_b200/libtdfs.so; fi
done
{
for v in base md128 md64; do
  for mb in 256 512; do
    echo "== $v hub_mb $mb"; PYTHONPATH=/tmp/var_$v:$PWD timeout 900 python scripts/variant_time.py 2 c4,diamond,tailed_triangle,k4,triangle 3 1 $mb
  done
  echo "== $v C5"; TAU=100 PYTHONPATH=/tmp/var_$v:$PWD timeout 900 python scripts/variant_time.py 5 k4 1 16 1024
done
} > gpurun_out/hubdeg_r02u.log 2>&1
grep -v "^lib" gpurun_out/hubdeg_r02u.log
