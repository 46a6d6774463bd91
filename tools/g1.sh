mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/g1_smi.log
timeout 1500 python -m pytest tests -m gpu -q -rf 2>&1 | tail -n 30 > gpurun_out/g1_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g1_smoke.log 2>&1
timeout 600 python bench.py > gpurun_out/g1_bench.log 2>&1
tail -n 5 gpurun_out/g1_pytest.log gpurun_out/g1_smoke.log gpurun_out/g1_bench.log
