#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 300 python tools/time_trsT.py 10 10 512 10000 1
timeout 300 python tools/time_trsT.py 2 32 1024 5000 16
timeout 300 python tools/time_trsT.py 1 1 256 10000 1
timeout 1500 python bench.py --config C5 --steps 5 --warmup 3 --no-cpu --fill 0.1 --parity-sample 4096 > $OUT/bench_C5_p1024.json 2> $OUT/bench_C5_p1024.err; echo "C5 rc=$?"; tail -2 $OUT/bench_C5_p1024.err
python -c "
import json; d=json.loads(open('$OUT/bench_C5_p1024.json').read().strip().splitlines()[-1]); print(d['value'], d['roofline']['frac'], d['parity'], min(p['parity_checked'] for p in d['sweep']))"
