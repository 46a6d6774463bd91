bash tools/ab.sh old main 2>&1
for C in 8192 32768; do AB_ARGS="--chunk-size $C mix" bash tools/ab.sh old main 2>&1 | sed "s/^/C=$C /"; done
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -1
