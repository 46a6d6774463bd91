bash tools/ab.sh sbbase sbrt 2>&1
AB_ARGS="--parse 1 mix" bash tools/ab.sh sbbase sbrt 2>&1 | head -2
LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_sbrt.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -1
