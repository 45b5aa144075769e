#!/bin/bash
# full GPU suite + transposed timings on the default build
OUT=gpurun_out; mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/pytest_t.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_t.log
for a in "10 10 512 10000 1" "2 32 1024 5000 16" "1 1 256 10000 1" "32 32 512 2000 1" "4 4 193 512 1" "5 9 300 4000 2"; do
  timeout 300 python tools/time_trsT.py $a
done > $OUT/trsT_times.txt 2>&1
cat $OUT/trsT_times.txt
