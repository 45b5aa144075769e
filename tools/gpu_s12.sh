#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -q > $OUT/s12_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $OUT/s12_pytest.log
grep -E "^FAILED" $OUT/s12_pytest.log | head -20
for c in C4 C2; do timeout 300 python bench.py --config $c --steps 30 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/s12_bench_$c.json 2>$OUT/s12_bench_$c.err; python tools/summ.py $OUT/s12_bench_$c.json | cut -c1-220; done
timeout 300 python bench.py --config C4 --trans T --steps 10 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/s12_bench_C4T.json 2>/dev/null; python tools/summ.py $OUT/s12_bench_C4T.json | cut -c1-220
for cfg in "1 1 256 10000" "2 3 512 10000" "2 32 1024 5000"; do python tools/time_trf.py $cfg rows cols 2>&1 | tail -2; done
