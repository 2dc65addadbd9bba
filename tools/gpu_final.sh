# launch lists (one configuration each) and ncu of the default incremental search
bash tools/gpu.sh "launches:r02_launches_C5_value:python,tools/bench_step.py,C5,0,5" "launches:r02_launches_C5_hilbert_ls1:python,tools/ls_once.py,C5,hilbert" "launches:r02_launches_C3_random_ls1:python,tools/ls_once.py,C3,random"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:inc_ls1_kernel -c 1 -o gpurun_out/r02_inc_ls1_C5_hilbert -f python tools/ls_once.py C5 hilbert > gpurun_out/r02_inc_ls1_C5_hilbert.log 2>&1
echo "ncu inc_ls1 rc=$?"
python tools/ncu_summary.py gpurun_out/r02_inc_ls1_C5_hilbert.ncu-rep > gpurun_out/r02_inc_ls1_C5_hilbert.txt 2>&1
