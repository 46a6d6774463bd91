for sets in 3 4 5; do for r in 1 2; do echo -n "sets=$sets "; LZR_HOST_SETS=$sets timeout 300 python tools/e2e_sweep.py 12,16,24 2>&1 | tail -3 | tr '\n' ' '; echo; done; done
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -1
