for r in 1 2; do for v in d2 d1; do LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_$v.so timeout 300 python tools/dec_time.py mix text zeroruns random 2>&1 | tail -1; done; done
