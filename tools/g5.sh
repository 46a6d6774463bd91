mkdir -p gpurun_out
bash tools/sanitize_lazy.sh > gpurun_out/g5_sanitize_lazy.txt 2>&1
bash tools/ncu_bench.sh r01e
python tools/ncu_summarize.py r01e > gpurun_out/g5_ncu_summ.log 2>&1 || true
timeout 600 python bench.py > gpurun_out/g5_bench.log 2>&1
cat gpurun_out/g5_sanitize_lazy.txt; tail -c 1500 gpurun_out/g5_bench.log
