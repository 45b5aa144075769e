#!/bin/bash
# quick GPU pass: gpu tests, C3 bench (fused plan and the two-launch plan for comparison)
OUT=gpurun_out; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $OUT/smi.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -15 $OUT/pytest_gpu.log
timeout 600 python bench.py --steps 20 --warmup 3 --e2e-steps 2 > $OUT/bench_c3.json 2> $OUT/bench_c3.err; echo "bench rc=$?"
tail -3 $OUT/bench_c3.err
python tools/summ.py $OUT/bench_c3.json
