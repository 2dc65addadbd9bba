#!/bin/bash
# One parametrised driver for gpurun calls (replaces the round-1 one-off scripts):
#   gpurun -- 'bash tools/gpu.sh TASK [TASK ...]'
# Tasks (each writes under gpurun_out/ and echoes one status line):
#   smoke                 __graft_entry__.smoke()
#   tests[:EXPR]          pytest -m gpu (optionally -k EXPR)
#   exp:LIB1,LIB2,...     tools/exp_dense.py per in-tree build (default | base | <variant>)
#   ubench                tools/ubench/pipes.cu pipe rates
#   sanitize[:TOOLS]      compute-sanitizer over tools/sanitize_run.py modes
#   bench[:ARGS]          python bench.py (ARGS with commas for spaces)
#   launches:NAME:CMD     ncu launch list (gpu__time_duration) of CMD (commas for spaces) -> NAME.csv/.txt
#   ncu:NAME:REGEX:CMD    ncu --set full of the first REGEX launch after one skip -> NAME.ncu-rep + .txt
#   py:CMD                any python command (commas for spaces)
#   env:K=V               export K=V for the tasks that follow
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for task in "$@"; do
  kind="${task%%:*}"; arg="${task#*:}"; [ "$arg" = "$task" ] && arg=""
  case "$kind" in
    smoke) timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
           echo "smoke rc=$? $(tail -1 gpurun_out/smoke.log)";;
    tests) k=(); [ -n "$arg" ] && k=(-k "$arg")
           timeout 2400 python -m pytest tests -m gpu -q -x --timeout 900 --durations=15 "${k[@]}" > gpurun_out/pytest_gpu.log 2>&1
           echo "tests rc=$? $(tail -1 gpurun_out/pytest_gpu.log)";;
    exp) for lib in ${arg//,/ }; do
           so=paper_conf_ipps_rockis13_b200/libtsp2opt.so; [ "$lib" != default ] && so=paper_conf_ipps_rockis13_b200/libtsp2opt_$lib.so
           TSP2OPT_LIB=$PWD/$so timeout 900 python tools/exp_dense.py $lib 2>&1 | tail -1 | tee -a gpurun_out/exp.jsonl
         done;;
    ubench) nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/pipes tools/ubench/pipes.cu && /tmp/pipes > gpurun_out/ubench_pipes.txt 2>&1
           echo "ubench rc=$?";;
    sanitize) TOOLS="${arg//,/ }" bash tools/gpu_sanitize.sh;;
    bench) timeout 1800 python bench.py ${arg//,/ } > gpurun_out/bench.log 2> gpurun_out/bench.err
           echo "bench rc=$? $(tail -c 300 gpurun_out/bench.log)";;
    launches) name="${arg%%:*}"; cmd="${arg#*:}"
           timeout 1800 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/$name.csv ${cmd//,/ } > gpurun_out/$name.log 2>&1
           echo "launches $name rc=$?"; python tools/launch_summary.py gpurun_out/$name.csv > gpurun_out/$name.txt 2>&1;;
    ncu) name="${arg%%:*}"; rest="${arg#*:}"; rx="${rest%%:*}"; cmd="${rest#*:}"
           timeout 1800 ncu --set full --clock-control none --import-source on -k regex:$rx -s 1 -c 1 -o gpurun_out/$name -f ${cmd//,/ } > gpurun_out/$name.log 2>&1
           echo "ncu $name rc=$?"; python tools/ncu_summary.py gpurun_out/$name.ncu-rep > gpurun_out/$name.txt 2>&1;;
    env) export "$arg"; echo "env $arg";;
    py) timeout 2400 python ${arg//,/ } 2>&1 | tail -40; echo "py rc=${PIPESTATUS[0]}";;
    *) echo "unknown task $task";;
  esac
done
