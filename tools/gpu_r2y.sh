#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/pytest_y.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_y.log
timeout 300 python tools/time_trsN.py trs 10,10,512,10000 32,32,2048,3000 2,3,256,200000 10,7,512,25000
timeout 300 python tools/time_trsN.py trfs 32,32,32,200000 32,32,512,12000 10,10,512,10000
