#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -x -q -k "32-32 or 32,32 or wide" > $OUT/pytest_wide.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_wide.log
for v in wide1 wide2; do
  BANDLU_LIB=$PWD/variants_build/lib_F_$v.so timeout 600 python bench.py --config C5 --c5-ns 128,512,2048 --steps 5 --warmup 3 --no-cpu --fill 0.05 > $OUT/w_$v.json 2>$OUT/w_$v.err
  python -c "
import json; d=json.loads(open('$OUT/w_$v.json').read().strip().splitlines()[-1])
for p in d['sweep']:
    if p['kl']==32: print('$v', p['n'], round(p['ms_per_step'],3), [round(x,3) for x in p['kernel_ms']], round(p['hbm_gbs']), p['parity_bad'])
"
done
