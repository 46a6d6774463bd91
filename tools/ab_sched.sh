# decode GB/s per class with and without the costliest-first schedule (alternating), then the decode tests
for r in 1 2; do
LZR_DEC_SCHED=0 python tools/dec_time.py mix text zeroruns random 2>&1 | tail -1
LZR_DEC_SCHED=1 python tools/dec_time.py mix text zeroruns random 2>&1 | tail -1
done > gpurun_out/ab_sched.log
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -3 > gpurun_out/par_sched.log
