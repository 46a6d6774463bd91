for C in 8192 16384 32768; do AB_ARGS="--chunk-size $C mix text zeroruns" bash tools/ab.sh p8base p8 2>&1 | sed "s/^/C=$C /"; done
bash tools/ab.sh p8base p8 2>&1
for s in 1 2; do LZR_ENCODE_SPLITS=$s LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_p8.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -1; done
