# ncu --set full of the decode, scan and compact kernels on the bench workload
# (256 MiB mix, C = 4 KiB) and of the big-chunk encode kernel (C = 64 KiB)
R=${1:-r02}
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lzr_decode_kernel -s 1 -c 1 \
  -f -o gpurun_out/dec_mix_$R python tools/prof_encode.py --cls mix --mib 256 --decode > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none -k regex:lzr_compact_kernel -s 1 -c 1 \
  -f -o gpurun_out/compact_mix_$R python tools/prof_encode.py --cls mix --mib 256 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none -k regex:lzr_scan_kernel -s 1 -c 1 \
  -f -o gpurun_out/scan_mix_$R python tools/prof_encode.py --cls mix --mib 256 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lzr_encode -s 1 -c 1 \
  -f -o gpurun_out/enc64k_mix_$R python tools/prof_encode.py --cls mix --mib 256 --chunk-size 65536 > /dev/null 2>&1
ls -la gpurun_out/*_$R.ncu-rep
