#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu.log
for b in 1250 2500 3552 5000 10000; do
 for p in auto two fused; do
  timeout 300 python bench.py --batch $b --plan $p --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/s_${b}_$p.json 2>$OUT/s_${b}_$p.err; echo "C3 batch $b $p $(python tools/summ.py $OUT/s_${b}_$p.json)"
 done
done
