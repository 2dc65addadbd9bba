for r in 3 4 6 10; do TSP2OPT_AUTO_INC_RHO=$r timeout 600 python tools/exp_c3.py rho$r 2>&1 | tail -1 | tee -a gpurun_out/exp_c3.jsonl; done
timeout 900 python tools/exp_c3_switch.py 2>&1 | tee gpurun_out/exp_c3_switch_ls1.jsonl
