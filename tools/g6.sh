mkdir -p gpurun_out
timeout 300 python tools/batch_probe.py > gpurun_out/g6_batch_probe.log 2>&1
for sp in 0 1; do for r in 1 2; do echo -n "split=$sp "; LZR_HOST_SPLIT=$sp timeout 300 python tools/e2e_sweep.py 8,16,32 2>&1 | tail -n 3 | tr '\n' ' '; echo; done; done > gpurun_out/g6_e2e.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "host" 2>&1 | tail -2 >> gpurun_out/g6_e2e.log
cat gpurun_out/g6_batch_probe.log gpurun_out/g6_e2e.log
