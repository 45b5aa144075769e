#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
export BANDLU_JIT_CACHE=/tmp/bandlu_jit; mkdir -p $BANDLU_JIT_CACHE
timeout 900 python -m pytest tests -m gpu -x -q -k "jit" > $OUT/pytest_jit.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_jit.log
timeout 900 python tools/jit_bench.py 512 1.5 > $OUT/jit_bench.txt 2>&1; cat $OUT/jit_bench.txt
