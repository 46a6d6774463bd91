mkdir -p gpurun_out
for sets in 3 4 6 8; do for sp in 0 1; do echo -n "sets=$sets split=$sp: "; LZR_HOST_SETS=$sets LZR_HOST_SPLIT=$sp timeout 300 python tools/e2e_sweep.py 8,16,32 2>&1 | tail -3 | tr '\n' ' '; echo; done; done > gpurun_out/g9_e2e.log 2>&1
timeout 200 python tools/pcie_probe.py > gpurun_out/g9_pcie.log 2>&1
cat gpurun_out/g9_e2e.log gpurun_out/g9_pcie.log
