#!/bin/bash
# compute-sanitizer on the decode kernel only (--kernel-name regex): memcheck,
# racecheck, synccheck, initcheck over every class at 4 KiB, mix at 8 / 64 KiB,
# and a corrupted-stream decode (run under gpurun)
out=gpurun_out/sanitize_dec
mkdir -p $out
for tool in memcheck racecheck synccheck initcheck; do
  for cls in mix text zeroruns random; do
    timeout 900 compute-sanitizer --tool $tool --kernel-name regex:lzr_decode --error-exitcode 9 \
      python tools/prof_encode.py --cls $cls --mib 4 --iters 1 --decode > $out/${tool}_${cls}.log 2>&1
    echo "$tool $cls rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_${cls}.log | tail -1)"
  done
  for C in 8192 65536; do
    timeout 900 compute-sanitizer --tool $tool --kernel-name regex:lzr_decode --error-exitcode 9 \
      python tools/prof_encode.py --cls mix --mib 4 --iters 1 --decode --chunk-size $C > $out/${tool}_mix$C.log 2>&1
    echo "$tool mix C=$C rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_mix$C.log | tail -1)"
  done
  timeout 900 compute-sanitizer --tool $tool --kernel-name regex:lzr_decode --error-exitcode 9 \
    python -m pytest tests/test_gpu_parity.py -m gpu -q -k "corruption or fuzz or without_error" > $out/${tool}_corrupt.log 2>&1
  echo "$tool corrupt/fuzz tests rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|passed|failed' $out/${tool}_corrupt.log | tail -2 | tr '\n' ' ')"
done
