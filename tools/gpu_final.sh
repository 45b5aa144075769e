#!/bin/bash
# Round-2 closing measurement: smoke, GPU tests, every bench config (C3 default + cpu baseline + e2e,
# reference arm, C1 C2 C4 XGC PELE, strong-scaling shard sizes, --trans T, C5 sweep), the ncu launch
# list of the C3 bench, full ncu captures of every config's kernels, SASS histograms.
OUT=gpurun_out/final; NCU=/tmp/ncu; mkdir -p $OUT/prof $NCU
export BANDLU_JIT_CACHE=/tmp/bandlu_jit; mkdir -p $BANDLU_JIT_CACHE
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 $OUT/pytest_gpu.log
python bench.py > $OUT/bench_default.json 2> $OUT/bench_default.err; echo "bench rc=$?"
python bench.py --impl reference --steps 4 > $OUT/bench_reference.json 2>$OUT/bench_reference.err
for c in C1 C2 C4 XGC PELE; do timeout 600 python bench.py --config $c --steps 30 --warmup 3 --no-cpu > $OUT/bench_$c.json 2>$OUT/bench_$c.err; done
for b in 5000 2500 1250; do timeout 600 python bench.py --batch $b --scaling strong --steps 30 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/bench_C3_b$b.json 2>$OUT/bench_C3_b$b.err; done
timeout 600 python bench.py --config C3 --trans T --steps 20 --warmup 3 --no-cpu > $OUT/bench_C3T.json 2>$OUT/bench_C3T.err
timeout 600 python bench.py --config C4 --trans T --steps 10 --warmup 3 --no-cpu > $OUT/bench_C4T.json 2>$OUT/bench_C4T.err
timeout 1500 python bench.py --config C5 --steps 5 --warmup 3 --no-cpu --fill 0.1 --parity-sample 1024 > $OUT/bench_C5.json 2>$OUT/bench_C5.err; echo "C5 rc=$?"
python tools/summ.py $OUT/bench_default.json $OUT/bench_reference.json $OUT/bench_C*.json $OUT/bench_XGC.json $OUT/bench_PELE.json | cut -c1-260
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $NCU/launches_c3.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu > $OUT/ncu_launch_bench.log 2>&1
cp $NCU/launches_c3.csv $OUT/launches_c3.csv
for c in C3 C2 C4 C5W C3T; do
  if [ "$c" = "C3T" ]; then extra="PROF_SEPARATE=1"; else extra=""; fi
  env $extra timeout 900 ncu --set full --clock-control none --import-source on -k regex:gbtr -c 2 -o $NCU/full_$c python tools/prof_step.py $c > $OUT/ncu_full_$c.log 2>&1
done
cp profiles/ncu_summary.json $OUT/prof/ 2>/dev/null
NCU_DIR=$NCU PROF_DIR=$OUT/prof python tools/make_profiles.py r02 C3 C2 C4 C5W C3T > /dev/null
for c in C3 C4 C5W; do
  ncu -i $NCU/full_$c.ncu-rep --page source --csv --print-source sass > $NCU/src_$c.csv 2>/dev/null
  python tools/sass_hist.py $NCU/src_$c.csv 40 > $OUT/prof/sass_hist_$c.txt 2>/dev/null
done
head -60 $OUT/prof/r02_summary.md
