#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT/san
export BANDLU_JIT_CACHE=/tmp/bandlu_jit; mkdir -p $BANDLU_JIT_CACHE
timeout 1200 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 $OUT/pytest_gpu.log
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py > $OUT/san/$tool.log 2>&1; echo "$tool rc=$?"; grep -E "SUMMARY|sanitize" $OUT/san/$tool.log
done
