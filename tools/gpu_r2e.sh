#!/bin/bash
# latency profile of the factorization kernel at low occupancy (C3 shard of 8 GPUs: 1250 matrices)
OUT=gpurun_out; mkdir -p $OUT
PROF_BATCH=1250 PROF_TWO=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:gbtrf_rows -c 1 -o $OUT/lat_1250 python tools/prof_step.py C3 > $OUT/ncu_lat.log 2>&1
ncu -i $OUT/lat_1250.ncu-rep --page source --csv --print-source sass > $OUT/src_lat_1250.csv 2>/dev/null
ncu -i $OUT/lat_1250.ncu-rep --page raw --csv > $OUT/raw_lat_1250.csv 2>/dev/null
rm -f $OUT/lat_1250.ncu-rep
gzip -f $OUT/src_lat_1250.csv
ls -la $OUT | tail -5
