bash tools/gpu_round.sh $1 > gpurun_out/round_$1.log 2>&1
bash tools/ncu_kernels.sh $1 > gpurun_out/ncu_kernels_$1.log 2>&1
