mkdir -p gpurun_out
timeout 900 ncu --set full --cache-control none --clock-control none --import-source on -k regex:cull_kernel --launch-skip 4000 --launch-count 1 -o gpurun_out/cull_mid -f python tools/exp_incremental.py C5:mf 3 > gpurun_out/ncu_cm.log 2>&1; echo a=$?
timeout 900 ncu --set full --cache-control none --clock-control none --import-source on -k regex:box_kernel --launch-skip 4000 --launch-count 1 -o gpurun_out/box_mid -f python tools/exp_incremental.py C5:mf 3 > gpurun_out/ncu_bm.log 2>&1; echo b=$?
