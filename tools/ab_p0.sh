bash tools/ab.sh main p0p 2>&1
LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_p0p.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_lazy.py -q -x 2>&1 | tail -1
