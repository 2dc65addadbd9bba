# full GPU test suite + ncu of the batched kernel (current auto layout)
mkdir -p gpurun_out
bash tools/gpu_tests.sh
NB=100 BB=4736 bash tools/gpu_ncu_batch.sh
NB=1002 BB=592 bash tools/gpu_ncu_batch.sh
