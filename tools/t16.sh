timeout 900 python bench.py --config 5 > gpurun_out/bench_cfg5.log 2>&1; tail -n 2 gpurun_out/bench_cfg5.log
timeout 600 python bench.py --no-cpu --no-e2e > gpurun_out/bench_cfg2.log 2>&1; tail -n 1 gpurun_out/bench_cfg2.log
timeout 900 ncu --set full --import-source on -k regex:"sha1|index_insert|index_lookup|gather" -c 4 -f -o gpurun_out/dedup_r01 python bench.py --config 5 --steps 1 --warmup 0 --no-cpu --bytes-per-rank 4294967296 > gpurun_out/ncu_dedup.log 2>&1; tail -n 3 gpurun_out/ncu_dedup.log
