"""A/B timing of the compress path for one library build (LZR_LIBRARY) over classes.
usage: LZR_LIBRARY=... python tools/ab_time.py [--mib 256] [--reps 10] [--chunk-size 4096] cls..."""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_pact_map17_b200 as lzr
ap = argparse.ArgumentParser()
ap.add_argument("cls", nargs="*", default=["mix", "text", "zeroruns"])
ap.add_argument("--mib", type=int, default=256)
ap.add_argument("--reps", type=int, default=10)
ap.add_argument("--chunk-size", type=int, default=4096)
ap.add_argument("--parse", type=int, default=0)  # 1 = lazy (R21)
a = ap.parse_args()
n = a.mib << 20
p = lzr.Params(chunk_size=a.chunk_size, parse=a.parse)
x = torch.empty(n, dtype=torch.uint8, device="cuda")
ws = lzr.Workspace(n, p, x.device)
res = []
for c in a.cls:
    synth.fill_device(x, a.chunk_size, c)
    for _ in range(3):
        lzr.compress(x, p, ws=ws)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(a.reps):
        lzr.compress(x, p, ws=ws)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / a.reps
    res.append(f"{c}:{n / ms / 1e6:.2f}")
print(os.path.basename(os.environ.get("LZR_LIBRARY", "liblzr.so")), " ".join(res), flush=True)
