for r in 1 2; do for v in d4 d2; do LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_$v.so timeout 300 python tools/dec_time.py 2>&1 | tail -1; done; done
