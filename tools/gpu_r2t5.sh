#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 600 python bench.py --config C3 --trans T --steps 20 --warmup 3 > $OUT/bench_C3T.json 2> $OUT/bench_C3T.err; echo "C3T rc=$?"; tail -2 $OUT/bench_C3T.err
timeout 600 python bench.py --config C4 --trans T --steps 10 --warmup 3 --no-cpu > $OUT/bench_C4T.json 2> $OUT/bench_C4T.err; echo "C4T rc=$?"
timeout 600 python bench.py --config C3 --trans T --impl reference --steps 5 --warmup 3 > $OUT/bench_C3T_ref.json 2> $OUT/bench_C3T_ref.err; echo "ref rc=$?"
python tools/summ.py $OUT/bench_C3T.json $OUT/bench_C4T.json $OUT/bench_C3T_ref.json | cut -c1-330
