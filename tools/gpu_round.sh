# full round check: gpu tests, smoke, default bench, reference arm, config-3/5, lazy,
# torchrun N=1, self-launched N=2 (gloo, shared GPU), ncu launch list + encode capture
R=${1:-r02a}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi_$R.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -n 5 > gpurun_out/pytest_gpu_$R.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$R.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_default_$R.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_$R.log 2>&1
for C in 4096 8192 16384 32768 65536; do timeout 600 python bench.py --config 3 --chunk-size $C --steps 3 --no-cpu --no-e2e > gpurun_out/bench_cfg3_${C}_$R.log 2>&1; done
timeout 900 python bench.py --config 5 --steps 5 > gpurun_out/bench_cfg5_$R.log 2>&1
timeout 600 python bench.py --parse lazy --no-cpu --no-per-class > gpurun_out/bench_lazy_$R.log 2>&1
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 1 --steps 5 --warmup 3 --no-cpu --no-per-class > gpurun_out/bench_torchrun1_$R.log 2>&1
timeout 600 python bench.py --gpus 2 --backend gloo --steps 5 --warmup 3 --no-cpu --no-per-class --no-e2e > gpurun_out/bench_gloo2_$R.log 2>&1
bash tools/ncu_bench.sh $R
tail -n 3 gpurun_out/pytest_gpu_$R.log gpurun_out/smoke_$R.log
for f in gpurun_out/bench_*_$R.log; do echo "$f: $(tail -n 1 $f | cut -c1-160)"; done
