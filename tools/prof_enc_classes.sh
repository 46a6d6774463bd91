mkdir -p gpurun_out
for c in text zeroruns; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lzr_encode -s 2 -c 1 \
  -f -o gpurun_out/enc_$c python tools/prof_encode.py --cls $c --mib 64 --iters 3 > gpurun_out/ncu_enc_$c.log 2>&1
done
ls -la gpurun_out
