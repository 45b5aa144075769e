#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_gpu.log
for v in fast slow; do for b in 1250 10000; do for p in two fused; do
  BANDLU_LIB=$PWD/variants_build/lib_$v.so timeout 300 python bench.py --batch $b --plan $p --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/v_${v}_${b}_$p.json 2>$OUT/v_${v}_${b}_$p.err; echo "$v batch $b $p $(python tools/summ.py $OUT/v_${v}_${b}_$p.json)"
done; done; done
