# usage: bash tools/ab_decode.sh PARITY_VARIANT V1 V2 ...: decode timing of the variants (alternating, 2 rounds), parity tests on the first
P=$1; shift
for r in 1 2; do for V in "$@"; do
LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_$V.so python tools/dec_time.py mix text zeroruns random 2>&1 | tail -1
done; done > gpurun_out/abn.log
LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_$P.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q 2>&1 | tail -15 > gpurun_out/par_$P.log
