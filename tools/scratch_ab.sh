# usage: bash tools/scratch_ab.sh NAME [pytest-k-expr]: A/B decode timing main vs liblzr_NAME.so, then parity tests on NAME
V=$1
for r in 1 2; do
python tools/dec_time.py mix text zeroruns random 2>&1 | tail -1
LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_$V.so python tools/dec_time.py mix text zeroruns random 2>&1 | tail -1
done > gpurun_out/ab_$V.log
LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_$V.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q ${2:+-k "$2"} 2>&1 | tail -15 > gpurun_out/par_$V.log
LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_$V.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:lzr_decode_kernel -s 1 -c 1 \
  -f -o gpurun_out/${V}_text python tools/prof_encode.py --cls text --mib 256 --decode > /dev/null 2>&1
