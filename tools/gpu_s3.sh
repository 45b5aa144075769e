#!/bin/bash
# column-owner kernel: parity tests, forced-variant factorization timing, bench lines
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "cols or trf_parity_small or planted or ties or padded or batch_tail" > $OUT/s3_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/s3_pytest.log
grep -E "FAILED|Error|assert" $OUT/s3_pytest.log | head -20
for cfg in "1 1 256 10000" "2 32 1024 5000" "2 2 64 100" "4 4 193 512" "2 3 512 10000"; do
  python tools/time_trf.py $cfg rows cols 2>&1 | tail -2
done
for c in C1 C2 C4 XGC; do timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/s3_bench_$c.json 2>$OUT/s3_bench_$c.err; python tools/summ.py $OUT/s3_bench_$c.json | cut -c1-300; done
