#!/bin/bash
# transposed ring solve: parity + timing
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "transposed" 2>&1 | tail -5
timeout 300 python tools/time_trsT.py 10 10 512 10000 1
timeout 300 python tools/time_trsT.py 2 32 1024 5000 16
timeout 300 python tools/time_trsT.py 1 1 256 10000 1
timeout 300 python tools/time_trsT.py 32 32 512 2000 1
timeout 300 python tools/time_trsT.py 4 4 193 512 1
