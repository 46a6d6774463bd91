for c in text mix zeroruns; do LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_timing.so timeout 300 python tools/phase_times.py --cls $c 2>&1 | tail -16; done
