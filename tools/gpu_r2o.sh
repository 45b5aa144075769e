#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
for b in 10000 40000; do timeout 120 python tools/time_trf.py 1 1 256 $b rows thin; done
timeout 120 python tools/time_trf.py 4 4 193 512 rows thin
for c in C2 C1 XGC; do for p in auto thin; do
  timeout 300 python bench.py --config $c --plan $p --steps 30 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/t_$c_$p.json 2>$OUT/t_err.txt; echo "$c $p $(python tools/summ.py $OUT/t_$c_$p.json | sed 's/parity={[^}]*}//')"; tail -2 $OUT/t_err.txt
done; done
