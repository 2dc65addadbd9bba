# ncu --set full of the dense sweep (C5 random, bench workload) and of the two-barrier incremental
# search (C5 Hilbert local search, one launch), with source; launch list of the C5 Hilbert search
export EXP_NO_LS=1
bash tools/gpu.sh "ncu:r02_sweep_C5_src:sweep_kernel:python,tools/exp_dense.py,ncu" "ncu:r02_inc_ls2_C5_hilbert:inc_ls2_kernel:python,tools/ls_once.py,C5,hilbert" "launches:r02_launches_C5_hilbert_ls2:python,tools/ls_once.py,C5,hilbert"
for r in r02_sweep_C5_src r02_inc_ls2_C5_hilbert; do
  ncu -i gpurun_out/$r.ncu-rep --page source --csv --print-source sass > gpurun_out/$r.source.csv 2>/dev/null
done
