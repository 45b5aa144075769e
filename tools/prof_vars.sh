# ncu full capture of the factorization kernel of each experiment build named in $VARS
for v in ${VARS:-r1g16}; do
  BANDLU_LIB=$PWD/variants_build/lib_$v.so ncu --set full --clock-control none --import-source on -k regex:gbtrf -c 1 -o gpurun_out/var_$v python tools/prof_step.py C3 > gpurun_out/ncu_var_$v.log 2>&1
done
ls -la gpurun_out/*.ncu-rep
