#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
BANDLU_LIB=$PWD/variants_build/lib_F_nb2.so timeout 900 python -m pytest tests -m gpu -x -q -k "trf_parity or trfs or fused or gbsv or full" > $OUT/pytest_nb2.log 2>&1; echo "pytest nb2 rc=$?"; tail -2 $OUT/pytest_nb2.log
for v in nb1 nb2 nb1 nb2; do for b in 10000 1250; do
  BANDLU_LIB=$PWD/variants_build/lib_$v.so timeout 300 python bench.py --batch $b --steps 30 --warmup 3 --no-cpu --e2e-steps 0 --plan two > $OUT/v_$v.json 2>$OUT/v_$v.err; echo "$v $b $(python tools/summ.py $OUT/v_$v.json | sed 's/parity={[^}]*}//')"
done; done
