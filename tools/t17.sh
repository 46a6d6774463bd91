LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_timing.so timeout 300 python tools/phase_times.py --cls text > gpurun_out/phase_text2.txt 2>&1
timeout 600 ncu --set full --import-source on -k regex:lzr_encode -s 1 -c 1 -o gpurun_out/enc_text2 -f python tools/prof_encode.py --cls text --mib 64 > gpurun_out/ncu_text2.log 2>&1
