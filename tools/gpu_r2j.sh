#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT/san
nvcc -gencode arch=compute_100a,code=sm_100a -O3 tools/probes/dfma_peak.cu -o /tmp/dfma && /tmp/dfma > $OUT/dfma_peak.json; cat $OUT/dfma_peak.json
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py > $OUT/san/$tool.log 2>&1; echo "$tool rc=$?"; tail -4 $OUT/san/$tool.log
done
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_gpu.log
timeout 1200 python bench.py --config C5 --steps 5 --warmup 3 --no-cpu --fill 0.1 > $OUT/bench_C5.json 2> $OUT/bench_C5.err; echo "C5 rc=$?"; tail -2 $OUT/bench_C5.err
python -c "
import json; d=json.loads(open('$OUT/bench_C5.json').read().strip().splitlines()[-1]); print(d['value'], d['roofline']['frac'], d['parity'])
for p in d['sweep']: print(p['kl'],p['ku'],p['n'],p['batch_per_gpu'],round(p['ms_per_step'],3),round(p['hbm_gbs']),p['kernels'],p['parity_bad'])
"
