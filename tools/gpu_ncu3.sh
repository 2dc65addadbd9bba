# ncu --set full of (1) the dense sweep in the middle of the C3 random-start search (launch 3000) and
# (2) the two-barrier incremental search kernel (C5 Hilbert, its single launch); source pages as CSV
mkdir -p gpurun_out
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 3000 -c 1 -o gpurun_out/r02_sweep_C3_mid -f python tools/ls_once.py C3 random > gpurun_out/r02_sweep_C3_mid.log 2>&1
echo "ncu C3 rc=$?"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:inc_ls2_kernel -c 1 -o gpurun_out/r02_inc_ls2_C5_hilbert -f python tools/ls_once.py C5 hilbert > gpurun_out/r02_inc_ls2_C5_hilbert.log 2>&1
echo "ncu inc rc=$?"
for r in r02_sweep_C3_mid r02_inc_ls2_C5_hilbert; do
  python tools/ncu_summary.py gpurun_out/$r.ncu-rep > gpurun_out/$r.txt 2>&1
  ncu -i gpurun_out/$r.ncu-rep --page source --csv --print-source sass > gpurun_out/$r.source.csv 2>/dev/null
done
