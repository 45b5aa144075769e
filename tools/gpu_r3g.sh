#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
for v in F_c4base F_c4a F_c4b F_c4c; do
  export BANDLU_LIB=$PWD/variants_build/lib_$v.so
  timeout 300 python bench.py --config C4 --steps 10 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/c4_$v.json 2>$OUT/c4_$v.err
  echo "$v $(python tools/summ.py $OUT/c4_$v.json | sed 's/parity={[^}]*}//' | cut -c1-220)"
  timeout 300 python tools/time_trsN.py trfs 2,32,1024,1000 2,32,2048,2500 2,32,256,20000
done
