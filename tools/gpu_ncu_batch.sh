# ncu --set full of one batched-LS launch (n=${NB:-100}, B=${BB:-4736})
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:batch_ls -c 1 \
  -o gpurun_out/batch_ls_${NB:-100} -f python tools/profile_batch.py ${NB:-100} ${BB:-4736} > gpurun_out/ncu_batch.log 2>&1
echo ncu=$?; tail -3 gpurun_out/ncu_batch.log
