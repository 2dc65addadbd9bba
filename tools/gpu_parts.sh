TSP2OPT_LIB=$PWD/paper_conf_ipps_rockis13_b200/libtsp2opt_acq.so timeout 400 python tools/exp_inc_parts.py ls1_acqrel 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl
timeout 400 python tools/exp_inc_parts.py ls1_fence 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl
