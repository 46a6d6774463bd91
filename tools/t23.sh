python tools/pcie_probe.py
for s in 3 4 6; do echo "sets=$s"; LZR_HOST_SETS=$s timeout 300 python tools/e2e_sweep.py 8,16,32,64; done
