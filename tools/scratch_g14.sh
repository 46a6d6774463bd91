bash tools/scratch_abn.sh g1 head g1 u1 > /dev/null 2>&1
cp gpurun_out/abn.log gpurun_out/abn_g14.log
bash tools/scratch_ncu.sh head mix text
bash tools/scratch_ncu.sh g1 mix text
