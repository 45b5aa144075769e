#!/bin/bash
for v in g16 g16r g32 g32r; do
  echo "== $v"
  BANDLU_LIB=$PWD/variants_build/lib_F_$v.so python tools/time_trf.py 2 32 1024 5000 rows cols 2>&1 | tail -2
  BANDLU_LIB=$PWD/variants_build/lib_F_$v.so python tools/time_trf.py 4 4 193 512 rows cols 2>&1 | tail -1
  BANDLU_LIB=$PWD/variants_build/lib_F_$v.so python tools/time_trf.py 4 4 512 10000 rows cols 2>&1 | tail -2
done
BANDLU_LIB=$PWD/variants_build/lib_F_g16.so timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "cols or trf_parity_small" 2>&1 | tail -2
