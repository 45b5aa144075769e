#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/pytest_r3d.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/pytest_r3d.log
timeout 1200 compute-sanitizer --tool memcheck python tools/sanitize.py > $OUT/san_mem.log 2>&1; echo "memcheck rc=$?"; tail -3 $OUT/san_mem.log
timeout 1200 compute-sanitizer --tool racecheck python tools/sanitize.py > $OUT/san_race.log 2>&1; echo "racecheck rc=$?"; tail -3 $OUT/san_race.log
timeout 1200 compute-sanitizer --tool synccheck python tools/sanitize.py > $OUT/san_sync.log 2>&1; echo "synccheck rc=$?"; tail -3 $OUT/san_sync.log
timeout 900 python bench.py --config C5 --steps 5 --warmup 3 --no-cpu --fill 0.1 --parity-sample 1100 > $OUT/bench_C5_r3.json 2> $OUT/bench_C5_r3.err; echo "C5 rc=$?"
python tools/summ.py $OUT/bench_C5_r3.json | cut -c1-200
