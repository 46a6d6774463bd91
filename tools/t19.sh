for v in k8b k8c; do LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -n 1; done
for C in 8192 32768; do
  AB_ARGS="--chunk-size $C --mib 512 --reps 3 mix text zeroruns" bash tools/ab.sh main k8b k8c 2>&1 | head -n 3 | sed "s/^/C=$C /"
done
