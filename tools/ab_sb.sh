bash tools/ab.sh main 2>&1
AB_ARGS="--chunk-size 8192 mix" bash tools/ab.sh main 2>&1 | head -1
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -1
