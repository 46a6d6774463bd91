"""Instruction / stall-sample shares of the encode kernel by phase (line ranges of
encode.cu) from an ncu source page: python tools/phase_prof.py cs.csv"""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
RANGES = [("lcp/run helpers", 109, 176), ("best_match_runs", 192, 228), ("best_match", 229, 319),
          ("walk_segment", 320, 437), ("setup/stage", 438, 530), ("histogram", 531, 580),
          ("hist scan|zero|cb", 581, 616), ("scatter|run ends", 617, 649), ("bucket flags", 650, 656),
          ("slot+cand", 657, 679), ("walk call", 680, 689), ("chain", 690, 725), ("totals", 726, 764),
          ("encode passes", 765, 832), ("copy-out", 833, 845)]
agg = {}
cur = None; h = None
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        cur = r[1].split("/")[-1]; continue
    if r[0] == "Line No":
        h = r; ie = h.index("Instructions Executed"); ss = h.index("Warp Stall Sampling (All Samples)"); continue
    try:
        li = int(r[0])
    except ValueError:
        continue
    def num(x):
        try:
            return float(x)
        except ValueError:
            return 0.0
    inst = num(r[ie]); smp = num(r[ss])
    name = cur
    if cur == "encode.cu":
        name = next((nm for nm, a, b in RANGES if a <= li <= b), "encode.cu other")
    a = agg.setdefault(name, [0.0, 0.0]); a[0] += inst; a[1] += smp
ti = sum(v[0] for v in agg.values()); ts = sum(v[1] for v in agg.values())
print(f"total warp-inst {ti:.3e}  samples {ts:.0f}")
for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{k:22s} inst {v[0]/ti*100:5.1f}%  stall-samples {v[1]/ts*100:5.1f}%")
