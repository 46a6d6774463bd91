mkdir -p gpurun_out
bash tools/ab.sh main k4b9 k4b4 > gpurun_out/g7_ab.log 2>&1
for v in main k4b9; do
  if [ $v = main ]; then L=paper_conf_pact_map17_b200/liblzr.so; else L=paper_conf_pact_map17_b200/liblzr_$v.so; fi
  echo "== $v"; LZR_LIBRARY=$L timeout 300 python tools/batch_probe.py 2>&1 | grep -E "(16|8|64) MiB"
  LZR_LIBRARY=$L timeout 300 python tools/e2e_sweep.py 16,32 2>&1 | tail -2
  LZR_LIBRARY=$L timeout 300 python tools/e2e_sweep.py 16,32 2>&1 | tail -2
done > gpurun_out/g7_batch.log 2>&1
cat gpurun_out/g7_ab.log gpurun_out/g7_batch.log
