bash tools/ab.sh main wc2 wc11 wc12 wc31 2>&1
