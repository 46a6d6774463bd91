mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -n 3 > gpurun_out/g8_pytest.log
bash tools/ab.sh main > gpurun_out/g8_ab.log 2>&1
timeout 300 python tools/batch_probe.py 64,32,16,8 > gpurun_out/g8_batch.log 2>&1
for r in 1 2; do timeout 300 python tools/e2e_sweep.py 8,16,32 2>&1 | tail -3; done >> gpurun_out/g8_batch.log
timeout 600 python bench.py --no-cpu > gpurun_out/g8_bench.log 2>&1
cat gpurun_out/g8_pytest.log gpurun_out/g8_ab.log gpurun_out/g8_batch.log; tail -c 700 gpurun_out/g8_bench.log
