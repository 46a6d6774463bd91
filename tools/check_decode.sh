#!/bin/bash
# Bounds-checked decoder (-DLZR_DEC_CHECK: every shared-memory access of the
# rebuild traps unless inside the chunk and reading only final bytes) over the
# decode parity, corruption and fuzz tests and 256 MiB of every class (run
# under gpurun; compute-sanitizer is not available on the GPU pool)
python tools/build_variant.py chk paper_conf_pact_map17_b200/csrc/decode.cu -DLZR_DEC_CHECK > /dev/null 2>&1 || exit 3
LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_chk.so timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_lazy.py -m gpu -q 2>&1 | tail -3
LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_chk.so timeout 600 python tools/dec_time.py mix text zeroruns random cr2 2>&1 | tail -2
for C in 8192 16384 65536; do
  LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_chk.so timeout 600 python tools/prof_encode.py --cls mix --mib 64 --decode --chunk-size $C 2>&1 | tail -1
done
