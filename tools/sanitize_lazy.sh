#!/bin/bash
# compute-sanitizer over the lazy-parse compress + decompress path (R21)
out=gpurun_out/sanitize_lazy
mkdir -p $out
for tool in memcheck racecheck synccheck initcheck; do
  for cls in mix zeroruns; do
    timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 \
      python tools/prof_encode.py --cls $cls --mib 2 --iters 1 --decode --parse 1 > $out/${tool}_${cls}.log 2>&1
    echo "$tool lazy $cls rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_${cls}.log | tail -1)"
  done
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 \
    python tools/prof_encode.py --cls mix --mib 2 --iters 1 --decode --chunk-size 8192 --parse 1 > $out/${tool}_mix8k.log 2>&1
  echo "$tool lazy mix C=8192 rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_mix8k.log | tail -1)"
done
