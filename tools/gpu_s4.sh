#!/bin/bash
OUT=gpurun_out; mkdir -p $OUT
./tools/probes/lat_probe_bin
python tools/dbg_cols.py 2>&1 | grep ipiv
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "cols or trf_parity_small or planted or ties or padded or batch_tail" > $OUT/s4_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $OUT/s4_pytest.log
grep -E "^FAILED|^E  " $OUT/s4_pytest.log | head -10
for cfg in "1 1 256 10000" "2 32 1024 5000" "2 2 64 100" "4 4 193 512" "2 3 512 10000" "1 1 256 1250"; do
  python tools/time_trf.py $cfg rows cols 2>&1 | tail -2
done
