#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "trf_parity" > $OUT/pytest_tpm.log 2>&1; echo "pytest rc=$?"; tail -5 $OUT/pytest_tpm.log
for b in 1250 10000; do timeout 120 python tools/time_trf.py 10 10 512 $b rows tpm; done
