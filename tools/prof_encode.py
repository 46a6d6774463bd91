"""Profiling driver: generate one class on the device and run the compress
path a few times (for ncu / compute-sanitizer captures; not a bench)."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import synth
import paper_conf_pact_map17_b200 as lzr

ap = argparse.ArgumentParser()
ap.add_argument("--cls", default="mix")
ap.add_argument("--mib", type=int, default=64)
ap.add_argument("--iters", type=int, default=2)
ap.add_argument("--chunk-size", type=int, default=4096)
ap.add_argument("--decode", action="store_true")
ap.add_argument("--parse", type=int, default=0)  # 0 greedy, 1 lazy (R21)
a = ap.parse_args()
n = a.mib << 20
p = lzr.Params(chunk_size=a.chunk_size, parse=a.parse)
x = torch.empty(n, dtype=torch.uint8, device="cuda")
synth.fill_device(x, a.chunk_size, a.cls)
ws = lzr.Workspace(n, p, x.device)
for _ in range(a.iters):
    out, sizes, offs, total = lzr.compress(x, p, ws=ws)
    if a.decode:
        y, err = lzr.decompress(out, sizes, offs, n, p)
torch.cuda.synchronize()
if a.decode:  # the round trip must hold (bounds-checked builds run this too)
    assert int(err.item()) == 0 and torch.equal(y, x), "decode round trip failed"
print("total", int(total.item()), "CR", n / int(total.item()), "round trip ok" if a.decode else "")
