mkdir -p gpurun_out
bash tools/ab.sh main wc2 wc4 wc8 > gpurun_out/g13_ab.log 2>&1
LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_wc4.so timeout 600 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -1 >> gpurun_out/g13_ab.log
cat gpurun_out/g13_ab.log
