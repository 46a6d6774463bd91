timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -n 1
for C in 4096 8192 16384 32768; do
  M=512; [ $C = 4096 ] && M=256
  echo -n "C=$C "; timeout 300 python tools/ab_time.py --chunk-size $C --mib $M --reps 3 mix text zeroruns random 2>&1 | tail -n 1
done
