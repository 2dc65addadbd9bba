# ncu --set full of the NEXT-4 kernels and the incremental list sweep (one launch each, mid local search)
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pruned_sweep -s 300 -c 1 -o gpurun_out/ncu_pruned_C5 -f python tools/exp_pruned.py C5 2 8 > gpurun_out/ncu_a.log 2>&1; echo a=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep25_list -s 300 -c 1 -o gpurun_out/ncu_sweep25_C5 -f python tools/exp_25opt.py C5 > gpurun_out/ncu_b.log 2>&1; echo b=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_list_kernel -s 300 -c 1 -o gpurun_out/ncu_inc_C5 -f python tools/exp_incremental.py C5:mf 3 > gpurun_out/ncu_c.log 2>&1; echo c=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cull_kernel -s 300 -c 1 -o gpurun_out/ncu_cull_C5 -f python tools/exp_incremental.py C5:mf 3 > gpurun_out/ncu_d.log 2>&1; echo d=$?
ls -la gpurun_out/*.ncu-rep
