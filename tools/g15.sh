for C in 8192 16384 32768; do AB_ARGS="--chunk-size $C mix text" bash tools/ab.sh old main 2>&1 | sed "s/^/C=$C /"; done
