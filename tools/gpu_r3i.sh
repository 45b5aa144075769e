#!/bin/bash
for v in F_nc1 F_wm17 F_wmr120 F_wmr128; do
  export BANDLU_LIB=$PWD/variants_build/lib_$v.so
  echo "== $v"
  for a in "2 32 1024 5000 16" "2 3 256 10000 4"; do timeout 120 python tools/time_trsT.py $a | grep "'N'"; done
done
