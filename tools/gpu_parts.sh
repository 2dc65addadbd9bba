timeout 400 python tools/exp_inc_parts.py ls1_final 2>&1 | tail -1 | tee -a gpurun_out/exp_inc_parts.jsonl
timeout 300 python tools/exp_c3.py ls1_final 2>&1 | tail -1 | tee -a gpurun_out/exp_c3.jsonl
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 600 -k "golden or switches or fullsize or first or p2p" 2>&1 | tail -2
