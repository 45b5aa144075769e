#!/bin/bash
# time the C3 factorization (dgbtrf, rows kernel) of every experiment build in variants_build/list.txt;
# "same" = bitwise equal to the first build's factors and pivots
A=${TRF_ARGS:-10 10 512 10000}
python - $A <<'PY'
import os, sys, subprocess
sys.path.insert(0, os.getcwd())
names = open("variants_build/list.txt").read().split()
for v in names:
    r = subprocess.run([sys.executable, "tools/time_trf_lib.py", *sys.argv[1:], v], capture_output=True, text=True)
    print(v, (r.stdout.strip().splitlines() or [r.stderr[-300:]])[-1])
PY
