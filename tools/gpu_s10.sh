#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -q > $OUT/s10_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $OUT/s10_pytest.log
grep -E "^FAILED" $OUT/s10_pytest.log | head -20
for c in C1 C2 XGC; do timeout 300 python bench.py --config $c --steps 30 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/s10_bench_$c.json 2>$OUT/s10_bench_$c.err; python tools/summ.py $OUT/s10_bench_$c.json | cut -c1-250; done
for b in 10000 2500; do timeout 300 python bench.py --config C2 --batch $b --steps 30 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/s10_C2_$b.json 2>/dev/null; python tools/summ.py $OUT/s10_C2_$b.json | cut -c1-200; done
