"""Per-phase cycle breakdown of the encode kernel (instrumented build).
usage: LZR_LIBRARY=paper_conf_pact_map17_b200/liblzr_timing.so python tools/phase_times.py --cls text"""
import argparse, ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import synth
import paper_conf_pact_map17_b200 as lzr

NAMES = ["loop/copy-out", "stage", "histogram", "scan|cb", "scatter|runs", "bucket flags",
         "slot+cand", "walk", "chain zero", "chain", "totals", "encode passes"]
ap = argparse.ArgumentParser()
ap.add_argument("--cls", default="text")
ap.add_argument("--mib", type=int, default=64)
a = ap.parse_args()
n = a.mib << 20
p = lzr.Params()
x = torch.empty(n, dtype=torch.uint8, device="cuda")
synth.fill_device(x, 4096, a.cls)
ws = lzr.Workspace(n, p, x.device)
L = lzr.lib()
buf = (ctypes.c_ulonglong * (16 * 4 * 2))()
lzr.compress(x, p, ws=ws); torch.cuda.synchronize()
L.lzr_debug_phase_times(buf)
lzr.compress(x, p, ws=ws); torch.cuda.synchronize()
L.lzr_debug_phase_times(buf)
t = np.array(buf, dtype=np.float64).reshape(16, 4, 2)
N = n // 4096
tot = t.sum()
print(f"class {a.cls}: cycles per chunk per warp (work / wait), K=4")
for i, nm in list(enumerate(NAMES)) + [(14, "scan part 1")]:
    w = t[i, :, 0] / N
    z = t[i, :, 1] / N
    print(f"{i:2d} {nm:14s} " + "  ".join(f"w{k}:{w[k]:7.0f}/{z[k]:6.0f}" for k in range(4)))
ph = list(range(12)) + [14]
print("total work", t[ph, :, 0].sum() / N / 4, "wait", t[ph, :, 1].sum() / N / 4)
print("best_match: cycles/chunk/warp", [round(t[12, k, 0] / N) for k in range(4)],
      "calls/chunk/warp", [round(t[12, k, 1] / N, 1) for k in range(4)],
      "walk iterations/chunk/warp", [round(t[13, k, 1] / N, 1) for k in range(4)])
