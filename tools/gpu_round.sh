#!/bin/bash
# One GPU session: tests, default bench (C3 + cpu_baseline), per-config benches,
# ncu launch list of the bench command, full ncu capture of both kernels at C3/C2/C4,
# summarised on the box (gpurun_out/prof/) -- only the C3 report comes back (64 MiB cap).
set -x
OUT=gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1
timeout 900 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.log 2>&1
python bench.py > $OUT/bench_default.json 2> $OUT/bench_default.err
for c in C1 C2 C4 XGC PELE; do python bench.py --config $c --steps 30 --warmup 3 --no-cpu > $OUT/bench_$c.json 2>$OUT/bench_$c.err; done
python bench.py --config C5 --steps 10 --warmup 3 --no-cpu > $OUT/bench_C5.json 2> $OUT/bench_C5.err
python bench.py --impl reference --steps 4 > $OUT/bench_reference.json 2>$OUT/bench_reference.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_c3.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu > $OUT/ncu_launch_bench.log 2>&1
for c in C3 C2 C4; do
  ncu --set full --clock-control none --import-source on -k regex:gbtr -c 2 -o $OUT/full_$c python tools/prof_step.py $c > $OUT/ncu_full_$c.log 2>&1
done
mkdir -p $OUT/prof; cp profiles/ncu_summary.json $OUT/prof/ 2>/dev/null
PROF_DIR=$OUT/prof python tools/make_profiles.py r01 C3 C2 C4 > /dev/null
ncu -i $OUT/full_C3.ncu-rep --page source --csv --print-source sass > $OUT/src_C3.csv 2>/dev/null
python tools/sass_hist.py $OUT/src_C3.csv 40 > $OUT/prof/sass_hist_C3.txt 2>/dev/null
rm -f $OUT/full_C2.ncu-rep $OUT/full_C4.ncu-rep $OUT/src_C3.csv
tail -3 $OUT/pytest_gpu.log; cat $OUT/smoke.log | tail -2
python tools/summ.py $OUT/bench_default.json $OUT/bench_C*.json
