#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -q > $OUT/s7_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $OUT/s7_pytest.log
grep -E "^FAILED" $OUT/s7_pytest.log | head -20
for c in C1 C2 XGC; do timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/s7_bench_$c.json 2>$OUT/s7_bench_$c.err; python tools/summ.py $OUT/s7_bench_$c.json | cut -c1-250; done
