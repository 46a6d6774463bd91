bash tools/check_decode.sh > gpurun_out/check_decode.txt 2>&1
bash tools/scratch_abn.sh u2 head u2 > /dev/null 2>&1
