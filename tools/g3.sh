mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_lazy.py -q -x -rf 2>&1 | tail -n 30 > gpurun_out/g3_pytest.log
for c in mix text zeroruns; do timeout 300 python bench.py --parse lazy --cls $c --no-cpu --no-e2e > gpurun_out/g3_bench_lazy_$c.log 2>&1; done
timeout 300 python bench.py --no-cpu --no-e2e > gpurun_out/g3_bench_greedy.log 2>&1
tail -n 3 gpurun_out/g3_pytest.log; for f in gpurun_out/g3_bench_*.log; do echo $f; python -c "import json,sys; l=json.loads(open('$f').read().strip().splitlines()[-1]); print(l['value'], l['config'].get('compression_ratio'))"; done
