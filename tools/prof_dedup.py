"""Driver for compute-sanitizer / ncu: dedup_compress (SHA-1, index, gather,
compress) of a small dedup-2.0 stream, plus the routing kernels with 3 owners."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_pact_map17_b200 as lzr
C, N = 4096, 600
x = torch.empty(N * C + 100, dtype=torch.uint8, device="cuda")
synth.fill_device(x, C, "mix_dedup")
res = lzr.dedup_compress(x, lzr.Params())
fp = res["fp"]
R = 3
cnt = lzr.owner_counts(fp, R).to(torch.int64)
base = torch.zeros(R, dtype=torch.int64, device="cuda")
base[1:] = torch.cumsum(cnt, 0)[:-1]
sfp, sg, slot = lzr.route(fp, 0, R, base)
idx = lzr.DedupIndex.for_chunks(fp.shape[0])
back, _ = idx.index_gidx(sfp, sg)
i2, u2 = lzr.unroute(back, slot, 0)
torch.cuda.synchronize()
assert torch.equal(i2, res["index"])
print("unique", res["n_unique"], "of", fp.shape[0])
