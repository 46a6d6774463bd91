timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -n 3
bash tools/ab.sh base main
for C in 8192 32768; do
  AB_ARGS="--chunk-size $C --mib 512 --reps 3 mix text zeroruns" bash tools/ab.sh base main 2>&1 | head -n 2 | sed "s/^/C=$C /"
done
