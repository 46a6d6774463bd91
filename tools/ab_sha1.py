"""A/B timing of lzr_fingerprint_chunks (LZR_LIBRARY build), 4 GiB mix, GB/s."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_pact_map17_b200 as lzr
n = 4 << 30
x = torch.empty(n, dtype=torch.uint8, device="cuda")
synth.fill_device(x, 4096, "mix")
fp = torch.empty((n // 4096, 20), dtype=torch.uint8, device="cuda")
for _ in range(2):
    lzr.fingerprint(x, 4096, out=fp)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda.synchronize()
e0.record()
for _ in range(5):
    lzr.fingerprint(x, 4096, out=fp)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 5
print(os.path.basename(os.environ.get("LZR_LIBRARY", "liblzr.so")), f"sha1 {n / ms / 1e6:.1f} GB/s")
