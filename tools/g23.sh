AB_ARGS="--parse 1" bash tools/ab.sh nopar main 2>&1
