#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -q > $OUT/s11_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $OUT/s11_pytest.log
grep -E "^FAILED" $OUT/s11_pytest.log | head -20
for c in C4 C2 C1; do timeout 300 python bench.py --config $c --steps 30 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/s11_bench_$c.json 2>$OUT/s11_bench_$c.err; python tools/summ.py $OUT/s11_bench_$c.json | cut -c1-220; done
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-cpu --fill 0.1 --parity-sample 256 > $OUT/s11_C5.json 2>$OUT/s11_C5.err; python tools/summ.py $OUT/s11_C5.json | cut -c1-200
