"""e2e (host buffers) throughput vs batch size through lzr_compress_host."""
import ctypes, statistics, sys, time
sys.path.insert(0, ".")
import torch
import synth, paper_conf_pact_map17_b200 as lzr
n = 256 << 20
p = lzr.Params()
x = torch.empty(n, dtype=torch.uint8, device="cuda"); synth.fill_device(x, 4096, "mix")
hx = x.cpu().pin_memory()
h_out = torch.empty(n, dtype=torch.uint8, pin_memory=True)
N = n // 4096
h_sizes = torch.empty(N, dtype=torch.int32, pin_memory=True)
h_offs = torch.empty(N, dtype=torch.int64, pin_memory=True)
for mb in [int(v) for v in sys.argv[1].split(",")]:
    b = mb << 20
    scratch = torch.empty(lzr.lib().lzr_compress_host_scratch_bytes(b, ctypes.byref(p.c())), dtype=torch.uint8, device="cuda")
    lzr.compress_host(hx, p, b, scratch, h_out, h_sizes, h_offs)
    ts = []
    for _ in range(5):
        t = time.perf_counter(); lzr.compress_host(hx, p, b, scratch, h_out, h_sizes, h_offs); ts.append(time.perf_counter() - t)
    print(mb, "MiB batches:", round(n / statistics.median(ts) / 1e9, 2), "GB/s", flush=True)
    del scratch
