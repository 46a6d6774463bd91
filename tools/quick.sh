# quick GPU iteration: parity tests, then bench mix/text/zeroruns (device-resident only)
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -n 5 > gpurun_out/q_pytest.log
for c in mix text zeroruns random; do
  timeout 300 python bench.py --cls $c --no-cpu --no-e2e --no-decode 2>&1 | tail -n 1 > gpurun_out/q_bench_$c.json
done
cat gpurun_out/q_pytest.log
for c in mix text zeroruns random; do python -c "import json,sys; d=json.load(open('gpurun_out/q_bench_$c.json')); print('$c', d['value'], d['roofline']['avg_launch_ms'])" 2>&1 | tail -n 1; done
