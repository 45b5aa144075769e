#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
for K in gbtrs_t_kernel gbtrs_window_kernel; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$K -c 1 -o /tmp/$K -f python tools/time_trsT.py 10 10 512 10000 1 > /tmp/$K.log 2>&1; echo "ncu rc=$?"
ncu -i /tmp/$K.ncu-rep --page raw --csv > $OUT/raw_$K.csv
ncu -i /tmp/$K.ncu-rep --page source --csv > $OUT/src_$K.csv
ncu -i /tmp/$K.ncu-rep --page details --csv > $OUT/det_$K.csv
done
ls -la $OUT
