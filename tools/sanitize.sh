#!/bin/bash
# compute-sanitizer over the compress + decompress path (4 KiB and 8 KiB chunks)
# and the dedup path on small inputs (run under gpurun)
out=gpurun_out/sanitize
mkdir -p $out
for tool in memcheck racecheck synccheck initcheck; do
  for cls in mix zeroruns text; do
    timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 \
      python tools/prof_encode.py --cls $cls --mib 2 --iters 1 --decode > $out/${tool}_${cls}.log 2>&1
    echo "$tool $cls rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_${cls}.log | tail -1)"
  done
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 \
    python tools/prof_encode.py --cls mix --mib 2 --iters 1 --decode --chunk-size 8192 > $out/${tool}_mix8k.log 2>&1
  echo "$tool mix C=8192 rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_mix8k.log | tail -1)"
  # 16- and 32-warp groups (C = 16 / 32 KiB: L2 walk bitmaps)
  for C in 16384 32768; do
    timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 \
      python tools/prof_encode.py --cls mix --mib 2 --iters 1 --decode --chunk-size $C > $out/${tool}_mix$C.log 2>&1
    echo "$tool mix C=$C rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_mix$C.log | tail -1)"
  done
  # big chunks (C = 64 KiB: 16-bit index, L2 walk bitmaps) and the lazy parse
  timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 \
    python tools/prof_encode.py --cls mix --mib 4 --iters 1 --decode --chunk-size 65536 > $out/${tool}_mix64k.log 2>&1
  echo "$tool mix C=65536 rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_mix64k.log | tail -1)"
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 \
    python tools/prof_encode.py --cls mix --mib 2 --iters 1 --decode --parse 1 > $out/${tool}_lazy.log 2>&1
  echo "$tool mix lazy rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_lazy.log | tail -1)"
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/prof_dedup.py > $out/${tool}_dedup.log 2>&1
  echo "$tool dedup rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' $out/${tool}_dedup.log | tail -1)"
done
