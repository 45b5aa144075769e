#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
export BANDLU_LIB=$PWD/variants_build/lib_F_thr.so
for b in 10000 40000; do timeout 120 python tools/time_trf.py 1 1 256 $b rows thread; done
timeout 120 python tools/time_trf.py 2 2 64 100 rows thread
timeout 120 python tools/time_trf.py 4 4 193 512 rows thread
timeout 300 python bench.py --config C2 --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/thr_c2.json 2>&1; python tools/summ.py $OUT/thr_c2.json | sed 's/parity={[^}]*}//'
