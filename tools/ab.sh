# usage: bash tools/ab.sh name1 name2 ...   (paper_conf_pact_map17_b200/liblzr_<name>.so; "main" = liblzr.so)
for r in 1 2; do
for v in "$@"; do
  if [ "$v" = main ]; then L=paper_conf_pact_map17_b200/liblzr.so; else L=paper_conf_pact_map17_b200/liblzr_$v.so; fi
  LZR_LIBRARY=$L timeout 300 python tools/ab_time.py ${AB_ARGS:-} 2>&1 | tail -n 1
done
done
