#!/bin/bash
# fused-kernel experiments at C3: prefetch depth / y placement variants, the two-launch plan, ncu of the fused kernel
OUT=gpurun_out; mkdir -p $OUT
bash tools/var_bench.sh
timeout 300 python bench.py --steps 20 --warmup 3 --no-cpu --e2e-steps 0 --two-launch > $OUT/bench_c3_two.json 2>$OUT/bench_c3_two.err
echo "two-launch $(python tools/summ.py $OUT/bench_c3_two.json)"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gbtr -c 1 -o $OUT/full_fused_C3 python tools/prof_step.py C3 > $OUT/ncu_fused.log 2>&1
ncu -i $OUT/full_fused_C3.ncu-rep --page source --csv --print-source sass > $OUT/src_fused_C3.csv 2>/dev/null
python tools/sass_hist.py $OUT/src_fused_C3.csv 40 > $OUT/sass_hist_fused_C3.txt 2>/dev/null
ncu -i $OUT/full_fused_C3.ncu-rep --page details --csv > $OUT/details_fused_C3.csv 2>/dev/null
rm -f $OUT/src_fused_C3.csv
ls -la $OUT
