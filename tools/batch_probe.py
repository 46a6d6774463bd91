"""Device-only cost of batching: compress 256 MiB as k batches (one stream, or
round-robin over 4 streams) vs one launch -- separates the per-batch kernel
tail from PCIe effects in the e2e pipeline."""
import sys
sys.path.insert(0, ".")
import torch
import synth, paper_conf_pact_map17_b200 as lzr
n = 256 << 20
p = lzr.Params()
x = torch.empty(n, dtype=torch.uint8, device="cuda"); synth.fill_device(x, 4096, "mix")
for mb in [int(v) for v in (sys.argv[1] if len(sys.argv) > 1 else "256,64,32,16,8").split(",")]:
    b = mb << 20
    k = n // b
    for ns in (1, 4):
        streams = [torch.cuda.Stream() for _ in range(ns)]
        wss = [lzr.Workspace(b, p, x.device) for _ in range(ns)]
        def run():
            for i in range(k):
                s = streams[i % ns]
                with torch.cuda.stream(s):
                    lzr.compress(x[i * b:(i + 1) * b], p, ws=wss[i % ns])
        for _ in range(2):
            run()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for s in streams:
            s.wait_event(e0)
        for _ in range(5):
            run()
        for s in streams:
            ev = torch.cuda.Event(); ev.record(s); torch.cuda.current_stream().wait_event(ev)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 5
        print(f"batch {mb:4d} MiB x {k:3d}, {ns} stream(s): {n / ms / 1e6:.1f} GB/s", flush=True)
