#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -q > $OUT/s9_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $OUT/s9_pytest.log
grep -E "^FAILED" $OUT/s9_pytest.log | head -20
for c in C4 C2 C1; do timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/s9_bench_$c.json 2>$OUT/s9_bench_$c.err; python tools/summ.py $OUT/s9_bench_$c.json | cut -c1-250; done
for cfg in "1 1 256 10000" "2 3 512 10000" "1 1 256 1250" "2 32 1024 5000"; do python tools/time_trf.py $cfg rows cols 2>&1 | tail -2; done
