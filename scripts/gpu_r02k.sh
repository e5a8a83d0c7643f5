#!/bin/bash
export PYTHONPATH=$PWD
for v in base lf1024 lf2048; do
  d=/tmp/var_$v; rm -rf $d && mkdir -p $d/paper_conf_icde_yuan0ha0024_b200
  cp paper_conf_icde_yuan0ha0024_b200/*.py $d/paper_conf_icde_yuan0ha0024_b200/
  if [ "$v" = base ]; then cp paper_conf_icde_yuan0ha0024_b200/libtdfs.so $d/paper_conf_icde_yuan0ha0024_b200/; else cp variants/$v.so $d/paper_conf_icde_yuan0ha0024_b200/libtdfs.so; fi
  echo "== $v"
  PYTHONPATH=$d:$PWD timeout 600 python scripts/variant_time.py 4 prism,w5 1 64
  PYTHONPATH=$d:$PWD timeout 600 python scripts/variant_time.py 4 prism,w5 1 1
  PYTHONPATH=$d:$PWD timeout 600 python scripts/variant_time.py 2 k4,diamond,c4 2 1
done
timeout 900 python scripts/configs_probe.py 4 prism 8 0,1,2,3,4,5,6,7 0 1 0
