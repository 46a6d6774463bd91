#!/bin/bash
# racecheck + synccheck on a launch large enough for the 3 CTAs x 3 groups shape
# (>= 12 chunk waves: 64 MiB = 16384 chunks of 4 KiB)
out=gpurun_out/sanitize_big
mkdir -p $out
for tool in racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 \
    python tools/prof_encode.py --cls mix --mib 64 --iters 1 > $out/${tool}_mix64.log 2>&1
  echo "$tool mix 64 MiB rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_mix64.log | tail -1)"
done
