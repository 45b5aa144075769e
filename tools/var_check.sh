#!/bin/bash
# For each experiment build in variants_build/list.txt: parity of the forced
# variant ($VARIANT, default 4 = ROWS) on a few shapes, then the C3 bench.
for v in $(cat variants_build/list.txt); do
  export BANDLU_LIB=$PWD/variants_build/lib_$v.so
  echo "== $v"
  for shape in "512 512 10 10 300 1" "70 70 10 10 37 1" "40 64 10 10 9 1" "64 40 10 10 9 1"; do
    timeout 120 python tools/quick_check.py $shape ${VARIANT:-4} 2>&1 | tail -2
  done
  timeout 120 python tools/fused_check.py 512 10 10 64 2>&1 | tail -1
  timeout 120 python tools/fused_check.py 37 10 10 33 2>&1 | tail -1
  for c in ${CFGS:-C3}; do
    timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/var_${v}_$c.json 2> gpurun_out/var_${v}_$c.err
    echo "$v $c $(python tools/summ.py gpurun_out/var_${v}_$c.json)"
  done
done
