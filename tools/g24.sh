AB_ARGS="--parse 1" bash tools/ab.sh nopar main 2>&1
bash tools/ab.sh nopar main 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_lazy.py -q -x 2>&1 | tail -1
