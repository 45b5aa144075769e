#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gbtrf_wide -c 1 -o /tmp/wide -f python tools/prof_step.py C5W > /tmp/wide.log 2>&1; echo "ncu rc=$?"
ncu -i /tmp/wide.ncu-rep --page raw --csv > $OUT/raw_wide.csv
ncu -i /tmp/wide.ncu-rep --page source --csv > $OUT/src_wide.csv
