#!/bin/bash
# Time variant builds of libtdfs.so (variants/NAME.so, built here with build.py defines) on one
# config: each runs from a private copy of the package so the in-tree library stays untouched.
#   variants.sh CFG QUERIES NAME1 NAME2 ...   (NAME "base" = the in-tree library)
CFG=$1; QS=$2; shift 2
for v in "$@"; do
  d=/tmp/var_$v
  rm -rf $d && mkdir -p $d/paper_conf_icde_yuan0ha0024_b200
  cp paper_conf_icde_yuan0ha0024_b200/*.py $d/paper_conf_icde_yuan0ha0024_b200/
  if [ "$v" = base ]; then cp paper_conf_icde_yuan0ha0024_b200/libtdfs.so $d/paper_conf_icde_yuan0ha0024_b200/;
  else cp variants/$v.so $d/paper_conf_icde_yuan0ha0024_b200/libtdfs.so; fi
  echo "== $v"
  PYTHONPATH=$d:$PWD timeout 900 python scripts/variant_time.py $CFG $QS ${REPS:-3}
done
