for K in 4 2 1; do TSP2OPT_INC_PART=$K timeout 900 python tools/exp_inc_parts.py ls2x_part$K 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl; done
for K in 4 2; do TSP2OPT_INC_PART_BOUND=0 TSP2OPT_INC_PART=$K timeout 900 python tools/exp_inc_parts.py ls2x_nobound_part$K 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl; done
TSP2OPT_LIB=$PWD/paper_conf_ipps_rockis13_b200/libtsp2opt_phase.so timeout 600 python tools/exp_phases2.py 2>&1 | tee -a gpurun_out/phases2.jsonl
