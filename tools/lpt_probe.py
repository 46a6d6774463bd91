"""Probe: how much of the encode launch is the end-of-queue tail?  Times the
compression of the 256 MiB mix as generated vs the same chunks reordered so
that the costliest class (text) comes first and the cheapest (raw) last
(chunk cost taken from a first compression: compressed-and-not-raw chunks with
CR < 3 first).  Not a bench; one GPU."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_pact_map17_b200 as lzr
n = 256 << 20
C = 4096
p = lzr.Params()
x = torch.empty(n, dtype=torch.uint8, device="cuda")
synth.fill_device(x, C, "mix")
ws = lzr.Workspace(n, p, x.device)
out, sizes, offs, total = lzr.compress(x, p, ws=ws)
s = sizes.view(torch.int32).long() if sizes.dtype != torch.int64 else sizes
cr = C / s.clamp(min=1).double()
key = torch.where(s >= C, torch.full_like(cr, 1e9), cr)  # raw last, then by CR ascending
order = torch.argsort(key)
xp = x.view(-1, C)[order].reshape(-1).contiguous()

def t(inp, reps=10):
    for _ in range(3):
        lzr.compress(inp, p, ws=ws)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(reps):
        lzr.compress(inp, p, ws=ws)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps

for r in range(2):
    a, b = t(x), t(xp)
    print(f"as generated {a:.3f} ms ({n / a / 1e6:.1f} GB/s)   costly-first {b:.3f} ms ({n / b / 1e6:.1f} GB/s)")

# the same for the decoder (index order, no schedule): decompression of the two compressed streams
oa, sa, fa, ta = lzr.compress(x, p)
ob, sb, fb, tb = lzr.compress(xp, p)
y = torch.empty_like(x)


def td(o, s_, f, reps=10):
    for _ in range(3):
        lzr.decompress(o, s_, f, n, p, out=y, schedule=False)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(reps):
        lzr.decompress(o, s_, f, n, p, out=y, schedule=False)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


for r in range(2):
    a, b = td(oa, sa, fa), td(ob, sb, fb)
    print(f"decode: as generated {a:.3f} ms ({n / a / 1e6:.1f} GB/s)   costly-first {b:.3f} ms ({n / b / 1e6:.1f} GB/s)")
