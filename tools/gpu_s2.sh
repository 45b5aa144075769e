#!/bin/bash
# full ncu capture of the C3 factorization, base and the G8/R2 variant, raw metric pages exported
OUT=gpurun_out; NCU=/tmp/ncu; mkdir -p $OUT $NCU
for v in base g8r2m12; do
  BANDLU_LIB=$PWD/variants_build/lib_$v.so timeout 600 ncu --set full --clock-control none --import-source on -k regex:gbtrf_rows -c 1 -o $NCU/s2_$v python tools/prof_step.py C3 > $OUT/s2_ncu_$v.log 2>&1
  ncu -i $NCU/s2_$v.ncu-rep --page raw --csv > $OUT/s2_raw_$v.csv 2>/dev/null
  ncu -i $NCU/s2_$v.ncu-rep --page details --csv > $OUT/s2_details_$v.csv 2>/dev/null
done
ls -la $OUT
