for s in 1 2 4 8; do LZR_ENCODE_SPLITS=$s timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -n 1; done
for C in 8192 16384 32768; do
  AB_ARGS="--chunk-size $C --mib 512 --reps 3 mix text zeroruns" bash tools/ab_env.sh LZR_ENCODE_SPLITS=1 LZR_ENCODE_SPLITS=2 LZR_ENCODE_SPLITS=4 LZR_ENCODE_SPLITS=8 2>&1 | head -n 4 | sed "s/^/C=$C /"
done
