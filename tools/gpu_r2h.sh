#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gbtrf_tpm -c 1 -o $OUT/tpm python tools/prof_trf.py 10 10 512 1250 tpm > $OUT/ncu_tpm.log 2>&1
ncu -i $OUT/tpm.ncu-rep --page source --csv --print-source sass > $OUT/src_tpm.csv 2>/dev/null
ncu -i $OUT/tpm.ncu-rep --page raw --csv > $OUT/raw_tpm.csv 2>/dev/null
rm -f $OUT/tpm.ncu-rep; gzip -f $OUT/src_tpm.csv; tail -2 $OUT/ncu_tpm.log
