# gpu tests + smoke + default bench + decode capture of the current tree (one gpurun call)
R=${1:-r02i}
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -n 3 > gpurun_out/pytest_gpu_$R.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$R.log 2>&1
timeout 600 python bench.py > gpurun_out/bench_default_$R.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lzr_decode_kernel -s 1 -c 1 \
  -f -o gpurun_out/dec_mix_$R python tools/prof_encode.py --cls mix --mib 256 --decode > /dev/null 2>&1
