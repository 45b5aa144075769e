#!/bin/bash
# full GPU suite + solves + C5 (32,32) points after adopting the block solve for nrhs == 1
OUT=gpurun_out; mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/pytest_w.log 2>&1; echo "pytest rc=$?"; tail -3 $OUT/pytest_w.log
for a in "10 10 512 10000 1" "2 32 1024 5000 16" "32 32 512 2000 1" "5 9 300 4000 1" "16 16 512 4000 1"; do
  timeout 120 python tools/time_trsT.py $a
done
timeout 900 python bench.py --config C5 --steps 5 --warmup 3 --no-cpu --fill 0.1 > $OUT/bench_C5_w.json 2> $OUT/bench_C5_w.err; echo "C5 rc=$?"
python tools/summ.py $OUT/bench_C5_w.json | cut -c1-200
python - <<'PY'
import json
d=json.loads(open('gpurun_out/bench_C5_w.json').read().strip().splitlines()[-1])
by={}
for p in d['sweep']: by.setdefault((p['kl'],p['ku']),[]).append(p)
for k,v in by.items(): print(k, 'ms=%.1f'%sum(p['ms_per_step'] for p in v), 'GB/s %.0f-%.0f'%(min(p['hbm_gbs'] for p in v), max(p['hbm_gbs'] for p in v)), v[-1]['kernels'], ['%.2f'%x for x in v[-1]['kernel_ms']])
PY
