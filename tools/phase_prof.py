"""Instruction / stall-sample shares of the encode kernel by phase (line ranges of
encode.cu) from an ncu source page: python tools/phase_prof.py cs.csv"""
import csv, sys
import os
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from phase_ranges import ranges, phase_of
rows = list(csv.reader(open(sys.argv[1])))
RS = ranges()
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
        name = phase_of(li, RS)
    a = agg.setdefault(name, [0.0, 0.0]); a[0] += inst; a[1] += smp
ti = sum(v[0] for v in agg.values()); ts = sum(v[1] for v in agg.values())
print(f"total warp-inst {ti:.3e}  samples {ts:.0f}")
for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{k:22s} inst {v[0]/ti*100:5.1f}%  stall-samples {v[1]/ts*100:5.1f}%")
