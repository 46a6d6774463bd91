# usage: bash tools/ab_env.sh "ENV=VAL ..." "ENV=VAL ..." ...   (main library, env variants)
for r in 1 2; do
for v in "$@"; do
  echo -n "[$v] "; env $v timeout 300 python tools/ab_time.py ${AB_ARGS:-} 2>&1 | tail -n 1
done
done
