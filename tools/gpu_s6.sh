#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -q > $OUT/s6_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/s6_pytest.log
grep -E "^FAILED" $OUT/s6_pytest.log | head -20
for cfg in "1 1 256 10000" "2 2 64 100" "2 3 512 10000" "3 2 512 10000" "0 3 512 10000" "3 0 512 10000" "1 1 256 1250"; do
  python tools/time_trf.py $cfg rows window cols 2>&1 | tail -3
done
for c in C1 C2 XGC; do timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/s6_bench_$c.json 2>$OUT/s6_bench_$c.err; python tools/summ.py $OUT/s6_bench_$c.json | cut -c1-250; done
