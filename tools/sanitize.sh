#!/bin/bash
# compute-sanitizer over the compress + decompress path on small inputs (run under gpurun)
out=gpurun_out/sanitize
mkdir -p $out
for tool in memcheck racecheck synccheck initcheck; do
  for cls in mix zeroruns text; do
    timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 \
      python tools/prof_encode.py --cls $cls --mib 2 --iters 1 --decode > $out/${tool}_${cls}.log 2>&1
    echo "$tool $cls rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_${cls}.log | tail -1)"
  done
done
