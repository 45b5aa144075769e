#!/bin/bash
# C3 factorization: resident warps per SM vs the number of 'rounds' of the batch
OUT=gpurun_out; mkdir -p $OUT
for v in $(cat variants_build/list.txt); do
  export BANDLU_LIB=$PWD/variants_build/lib_$v.so
  timeout 300 python bench.py --config C3 --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/var_${v}_C3.json 2> $OUT/var_${v}_C3.err
  echo "$v $(python tools/summ.py $OUT/var_${v}_C3.json | sed 's/parity={[^}]*}//' | cut -c1-200)"
  for b in 3552 4736 5032 7104; do PROF=1 timeout 120 python tools/time_chunks.py $b 512 10 10 2>/dev/null | sed "s/^/  $v /" ; done
done
