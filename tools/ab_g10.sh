bash tools/ab.sh tbbase main g10 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_lazy.py -q -x 2>&1 | tail -1
LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_g10.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -1
