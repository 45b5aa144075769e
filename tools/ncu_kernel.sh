# ncu --set full of one kernel (regex $2) in one bench step at config $1; raw + source csv into gpurun_out/
OUT=gpurun_out; C=$1; K=$2; TAG=${3:-$1}
ncu --set full --clock-control none --import-source on -k regex:$K -c 1 -o $OUT/full_$TAG python tools/prof_step.py $C > $OUT/ncu_$TAG.log 2>&1
ncu -i $OUT/full_$TAG.ncu-rep --page raw --csv > $OUT/raw_$TAG.csv
ncu -i $OUT/full_$TAG.ncu-rep --page source --csv --print-source sass > $OUT/src_$TAG.csv
python tools/ncu_summary.py $OUT/full_$TAG.ncu-rep
