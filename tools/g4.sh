mkdir -p gpurun_out
nproc > gpurun_out/g4_nproc.log
timeout 1500 python -m pytest tests -m gpu -q -x -rf --durations=8 2>&1 | tail -n 30 > gpurun_out/g4_pytest.log
timeout 600 python bench.py > gpurun_out/g4_bench.log 2>&1
for W in 1024 256; do timeout 300 python bench.py --window $W --no-cpu --no-e2e > gpurun_out/g4_bench_w$W.log 2>&1; done
tail -n 12 gpurun_out/g4_pytest.log; for f in gpurun_out/g4_bench*.log; do echo $f; python -c "import json,sys; l=json.loads(open('$f').read().strip().splitlines()[-1]); print(l['value'], l['config'].get('compression_ratio'), l.get('cpu_fast'), l.get('integration'))"; done
