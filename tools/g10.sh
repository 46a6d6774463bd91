mkdir -p gpurun_out
for r in 1 2; do for sets in 3 4 6; do for sp in 1 2; do echo -n "sets=$sets split=$sp: "; LZR_HOST_SETS=$sets LZR_HOST_SPLIT=$sp timeout 300 python tools/e2e_sweep.py 8,16,32 2>&1 | tail -3 | tr '\n' ' '; echo; done; done; done > gpurun_out/g10_e2e.log 2>&1
LZR_HOST_SPLIT=2 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k host 2>&1 | tail -1 >> gpurun_out/g10_e2e.log
cat gpurun_out/g10_e2e.log
