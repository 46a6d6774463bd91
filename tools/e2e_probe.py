"""Debug probe: compress_host after the same device work bench.py does first."""
import ctypes, sys, time
sys.path.insert(0, ".")
import torch
import synth, paper_conf_pact_map17_b200 as lzr
C = int(sys.argv[1]); n = int(sys.argv[2]) << 20; batch = int(sys.argv[3]) << 20
mode = sys.argv[4] if len(sys.argv) > 4 else "plain"
p = lzr.Params(chunk_size=C)
x = torch.empty(n, dtype=torch.uint8, device="cuda"); synth.fill_device(x, C, "mix")
if mode in ("ws", "dec"):
    ws = lzr.Workspace(n, p, x.device)
    for i in range(3):
        t = time.time()
        lzr.compress_encode(x, p, ws); torch.cuda.synchronize(); print("enc", i, time.time() - t, flush=True)
        lzr.compress_compact(x, p, ws); torch.cuda.synchronize(); print("cmp", i, time.time() - t, flush=True)
    print("device compress ok", flush=True)
    if mode == "dec":
        out, err = lzr.decompress(ws.out, ws.sizes[: ws.N], ws.offsets[: ws.N], n, p)
        torch.cuda.synchronize(); print("decode ok", int(err.item()), flush=True)
hx = x.cpu().pin_memory()
scratch = torch.empty(lzr.lib().lzr_compress_host_scratch_bytes(batch, ctypes.byref(p.c())), dtype=torch.uint8, device="cuda")
for i in range(3):
    t = time.time(); out = lzr.compress_host(hx, p, batch, scratch); print("host", i, time.time() - t, out[3], flush=True)
