#!/bin/bash
for v in g16 g16r g32r g16s; do
  echo "== $v"; BANDLU_LIB=$PWD/variants_build/lib_F_$v.so python tools/dbg_cols.py 2>&1 | grep ipiv | head -3
  BANDLU_LIB=$PWD/variants_build/lib_F_$v.so python tools/time_trf.py 2 32 1024 5000 rows cols 2>&1 | tail -1
done
