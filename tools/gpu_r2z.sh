#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 300 python tools/l2gran.py 128 64 32 0 128
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:gbtrs_bwd -c 2 python tools/l2gran.py 32 128 2>&1 | grep -E "gbtrs_bwd|dram__|gpu__time" | head -12
