#!/bin/bash
# session check: smoke, GPU tests, default bench, one full ncu capture of the C3 step
OUT=gpurun_out; NCU=/tmp/ncu; mkdir -p $OUT $NCU
export BANDLU_JIT_CACHE=/tmp/bandlu_jit; mkdir -p $BANDLU_JIT_CACHE
python -c "import __graft_entry__ as g; g.smoke()" > $OUT/s1_smoke.log 2>&1; tail -1 $OUT/s1_smoke.log
timeout 900 python -m pytest tests -m gpu -q -x > $OUT/s1_pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 $OUT/s1_pytest_gpu.log
python bench.py > $OUT/s1_bench.json 2> $OUT/s1_bench.err; echo "bench rc=$?"; cut -c1-400 $OUT/s1_bench.json
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gbtrf_rows -c 1 -o $NCU/s1_C3 python tools/prof_step.py C3 > $OUT/s1_ncu.log 2>&1
ncu -i $NCU/s1_C3.ncu-rep --page source --csv --print-source sass > $OUT/s1_src_C3.csv 2>/dev/null
ls -la $OUT
