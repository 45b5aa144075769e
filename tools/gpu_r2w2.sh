#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
for v in F_blk F_blk_ub8; do
  export BANDLU_LIB=$PWD/variants_build/lib_$v.so
  timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "trs or gbsv or trfs or fused or full or jit" > $OUT/pytest_$v.log 2>&1; echo "$v pytest rc=$? $(tail -1 $OUT/pytest_$v.log)"
  for a in "10 10 512 10000 1" "32 32 512 2000 1" "32 32 32 379356 1"; do timeout 120 python tools/time_trsT.py $a | grep "'N'"; done
  timeout 900 python bench.py --config C5 --steps 5 --warmup 3 --no-cpu --fill 0.1 --parity-sample 64 > $OUT/bench_C5_$v.json 2> $OUT/bench_C5_$v.err; echo "C5 rc=$?"
  python - $v <<'PY'
import json,sys
d=json.loads(open('gpurun_out/bench_C5_%s.json'%sys.argv[1]).read().strip().splitlines()[-1])
print(d['value'], d['roofline']['frac'], d['parity'])
by={}
for p in d['sweep']: by.setdefault((p['kl'],p['ku']),[]).append(p)
for k,v in by.items(): print(k, 'ms=%.1f'%sum(p['ms_per_step'] for p in v), 'bwd ms', ' '.join('%.2f'%p['kernel_ms'][-1] for p in v))
PY
done
