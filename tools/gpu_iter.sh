# quick GPU iteration: parity tests matching $1 (pytest -k), then benches for configs $2..
OUT=gpurun_out
K="$1"; shift
timeout 900 python -m pytest tests -m gpu -q -x -k "$K" > $OUT/pytest_iter.log 2>&1; tail -3 $OUT/pytest_iter.log
for c in "$@"; do timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu --e2e-steps 0 > $OUT/bench_$c.json 2>$OUT/bench_$c.err; python tools/summ.py $OUT/bench_$c.json; tail -2 $OUT/bench_$c.err; done
