# usage: bash tools/ncu_decode.sh VARIANT cls...: ncu --set full of the decode kernel on 256 MiB of each class
V=$1; shift
for c in "$@"; do
LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_$V.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:lzr_decode_kernel -s 1 -c 1 \
  -f -o gpurun_out/${V}_$c python tools/prof_encode.py --cls $c --mib 256 --decode > /dev/null 2>&1
done
