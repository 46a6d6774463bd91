#!/bin/bash
# ncu --set full of the encode kernel for each input class (64 MiB each)
for c in "$@"; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:lzr_encode -s 1 -c 1 \
    -o gpurun_out/enc_$c -f python tools/prof_encode.py --cls $c --mib 64 > gpurun_out/ncu_$c.log 2>&1
done
