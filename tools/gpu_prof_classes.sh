# per-class phase timing (instrumented build) + ncu full captures of encode
for c in text zeroruns; do
  LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_timing.so timeout 300 python tools/phase_times.py --cls $c > gpurun_out/phase_$c.txt 2>&1
done
bash tools/ncu_classes.sh text zeroruns
