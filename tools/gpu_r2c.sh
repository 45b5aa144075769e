#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 600 python -m pytest tests -m gpu -x -q -k "fused or trfs or gbsv or full" > $OUT/pytest_fused.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_fused.log
bash tools/var_bench.sh
for c in PELE C2 C1 XGC; do
  timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/b_$c.json 2>$OUT/b_$c.err; echo "fused $c $(python tools/summ.py $OUT/b_$c.json)"
  timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu --e2e-steps 0 --two-launch > $OUT/b2_$c.json 2>$OUT/b2_$c.err; echo "two $c $(python tools/summ.py $OUT/b2_$c.json)"
done
