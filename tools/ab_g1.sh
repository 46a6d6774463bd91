bash tools/ab.sh main g1all 2>&1
