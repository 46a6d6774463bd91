for r in 1 2 3; do timeout 300 python tools/e2e_sweep.py 8,16,32 2>&1 | tail -3 | tr '\n' ' '; echo; done
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "host or batch" 2>&1 | tail -1
