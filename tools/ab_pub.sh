bash tools/ab.sh main pub32 pub128 pub256 2>&1
