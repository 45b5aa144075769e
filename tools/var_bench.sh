#!/bin/bash
# bench every experiment build in variants_build/list.txt on $CFGS (no parity checks)
for v in $(cat variants_build/list.txt); do
  for c in ${CFGS:-C3}; do
    BANDLU_LIB=$PWD/variants_build/lib_$v.so timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > gpurun_out/var_${v}_$c.json 2> gpurun_out/var_${v}_$c.err
    echo "$v $c $(python tools/summ.py gpurun_out/var_${v}_$c.json)"
  done
done
