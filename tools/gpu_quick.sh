OUT=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $OUT/smi.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -x > $OUT/pytest_gpu.log 2>&1
python bench.py --steps 30 --warmup 3 > $OUT/bench_default.json 2> $OUT/bench_default.err
for c in C2 C4 C5; do timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu > $OUT/bench_$c.json 2>$OUT/bench_$c.err; done
tail -3 $OUT/pytest_gpu.log; tail -2 $OUT/smoke.log; cat $OUT/bench_default.json
