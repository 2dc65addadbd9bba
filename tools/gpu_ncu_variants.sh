# ncu --set full of the sweep kernel (C5 random, 2nd launch) for each lib in $LIBS
mkdir -p gpurun_out
for L in $LIBS; do
  name=$(basename $L .so)
  TSP2OPT_LIB=$L timeout 600 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 1 -c 1 -o gpurun_out/ncu_${name}_${CFG:-C5}_${TOUR:-random} -f python tools/profile_sweep.py ${CFG:-C5} ${TOUR:-random} 2 > gpurun_out/ncu_${name}.log 2>&1; echo $name $?
done
