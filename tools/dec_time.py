"""A/B timing of the decompression path (N1) for one library build (LZR_LIBRARY):
output GB/s over classes.  usage: LZR_LIBRARY=... [LZR_DEC_SCHED=0] python tools/dec_time.py [cls...]
(LZR_DEC_SCHED=0: chunks in index order instead of the costliest-first schedule)"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_pact_map17_b200 as lzr
n = 256 << 20
p = lzr.Params()
sched = os.environ.get("LZR_DEC_SCHED", "1") != "0"
x = torch.empty(n, dtype=torch.uint8, device="cuda")
ws = lzr.Workspace(n, p, x.device)
y = torch.empty_like(x)
res = []
for c in (sys.argv[1:] or ["mix", "text", "zeroruns"]):
    synth.fill_device(x, 4096, c)
    out, sizes, offs, total = lzr.compress(x, p, ws=ws)
    for _ in range(3):
        lzr.decompress(out, sizes, offs, n, p, out=y, schedule=sched)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(10):
        lzr.decompress(out, sizes, offs, n, p, out=y, schedule=sched)
    e1.record()
    torch.cuda.synchronize()
    assert torch.equal(y, x)
    res.append(f"{c}:{n / (e0.elapsed_time(e1) / 10) / 1e6:.1f}")
print(os.path.basename(os.environ.get("LZR_LIBRARY", "liblzr.so")), "sched" if sched else "index-order",
      " ".join(res), flush=True)
