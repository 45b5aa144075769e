#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -q > $OUT/s8_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $OUT/s8_pytest.log
grep -E "^FAILED" $OUT/s8_pytest.log | head -20
for c in C4 C2; do timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/s8_bench_$c.json 2>$OUT/s8_bench_$c.err; python tools/summ.py $OUT/s8_bench_$c.json | cut -c1-250; done
