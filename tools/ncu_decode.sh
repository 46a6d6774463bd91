#!/bin/bash
# ncu --set full of the decode kernel (N1) on 64 MiB of a class
for c in "$@"; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:lzr_decode_kernel -s 1 -c 1 \
    -o gpurun_out/dec_$c -f python tools/prof_encode.py --cls $c --mib 64 --decode > gpurun_out/ncu_dec_$c.log 2>&1
done
